timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_partition.py tests/test_gpu_schedule_ckpt.py -m gpu -x -q 2>&1 | tail -2
timeout 1500 python -m pytest tests/test_gpu_fullsize.py -m gpu -q 2>&1 | grep -E "assert|Error|passed|failed" | head -20
BENCH_ARGS="--config tunnel4" VARIANTS="liblbmr nozs" bash tools/gpu_variants.sh
BENCH_ARGS="--config sphere3" VARIANTS="liblbmr nozs" bash tools/gpu_variants.sh
BENCH_ARGS="--config cavity4_kbc" VARIANTS="liblbmr nozs" bash tools/gpu_variants.sh
BENCH_ARGS="--config sphere_tab1_s3" VARIANTS="liblbmr nozs" bash tools/gpu_variants.sh
