# timing experiment: cost of the special path (ALLPLAIN: every warp plain; NOSLOW: no bounce/records) — wrong results, timing only
for c in tunnel4 sphere3 cavity4_kbc cavity4_bgk; do echo "== $c"; BENCH_ARGS="--config $c" VARIANTS="liblbmr allplain noslow" bash tools/gpu_variants.sh; done
echo "== sphere_tab1_s3 fp64"; BENCH_ARGS="--config sphere_tab1_s3" VARIANTS="liblbmr allplain noslow" bash tools/gpu_variants.sh
