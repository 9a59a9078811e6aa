timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
for c in tunnel4 sphere3 cavity4_kbc; do BENCH_ARGS="--config $c" VARIANTS="liblbmr" bash tools/gpu_variants.sh; done
BENCH_ARGS="--config sphere_tab1_s3" VARIANTS="liblbmr" bash tools/gpu_variants.sh
