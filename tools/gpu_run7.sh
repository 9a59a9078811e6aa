timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_schedule_ckpt.py -m gpu -x -q 2>&1 | tail -2
BENCH_ARGS="--config tunnel4" VARIANTS="liblbmr" bash tools/gpu_variants.sh
BENCH_ARGS="--config tunnel4 --precision fp64" VARIANTS="liblbmr" bash tools/gpu_variants.sh
BENCH_ARGS="--config cavity4_bgk" VARIANTS="liblbmr" bash tools/gpu_variants.sh
BENCH_ARGS="--config cavity4_kbc" VARIANTS="liblbmr kbcf3" bash tools/gpu_variants.sh
BENCH_ARGS="--config cavity4_kbc --precision fp64" VARIANTS="liblbmr" bash tools/gpu_variants.sh
BENCH_ARGS="--config sphere_tab1_s3" VARIANTS="liblbmr" bash tools/gpu_variants.sh
BENCH_ARGS="--config sphere3" VARIANTS="liblbmr" bash tools/gpu_variants.sh
