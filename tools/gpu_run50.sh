(timeout 700 python bench.py --config uniform512 --steps 8000 --warmup 3 --no-cpu-baseline > /dev/null 2>&1 &)
sleep 15
timeout 600 python tools/ipc_diag.py 40 0 2>&1 | tail -8
timeout 500 python tools/ipc_diag.py 30 1 2>&1 | tail -8
