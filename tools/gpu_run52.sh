# D3Q19 fp32 occupancy re-sweep on the quarter-block build (cfg5 default, then cfg3)
for r in 1 2; do VARIANTS="occ6 occ5" bash tools/gpu_variants.sh; done
for r in 1 2; do BENCH_ARGS="--config sphere3" VARIANTS="occ6 occ5" bash tools/gpu_variants.sh; done
