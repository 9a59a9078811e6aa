# IPC halo stress after the creation/connect ordering fix: quiet device, then under a competing context
timeout 900 python -m pytest tests/test_gpu_partition.py -m gpu -q 2>&1 | tail -1
timeout 600 python tools/ipc_stress.py 30 2>&1 | tail -3
(timeout 400 python bench.py --config uniform512 --steps 4000 --warmup 3 --no-cpu-baseline > /dev/null 2>&1 &)
sleep 20
timeout 600 python tools/ipc_stress.py 20 2>&1 | tail -3
