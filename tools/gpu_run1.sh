set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/r01b_pytest_gpu.txt
bash tools/profile_round.sh r01b
for c in sphere3 cavity4_kbc uniform512; do timeout 300 python bench.py --config $c --no-cpu-baseline > gpurun_out/r01b_bench_$c.json 2>/dev/null; done
