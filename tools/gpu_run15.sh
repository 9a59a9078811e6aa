for o in 0 1 2 3; do LBMR_ORDER=$o BENCH_ARGS="--config tunnel4" VARIANTS="liblbmr" bash tools/gpu_variants.sh | sed "s/^/order$o /"; done
BENCH_ARGS="--config tunnel4" VARIANTS="nofill" bash tools/gpu_variants.sh
for o in 0 1 3; do LBMR_ORDER=$o BENCH_ARGS="--config sphere3" VARIANTS="liblbmr" bash tools/gpu_variants.sh | sed "s/^/order$o /"; done
