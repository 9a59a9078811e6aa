# 128-thread CTAs for every variant (nt128all) vs fp64 KBC only (liblbmr)
for c in tunnel4 sphere3 cavity4_kbc cavity4_bgk uniform512; do echo "== $c"; BENCH_ARGS="--config $c" VARIANTS="liblbmr nt128all liblbmr nt128all" bash tools/gpu_variants.sh; done
for c in tunnel4 sphere_tab1_s3; do echo "== $c fp64"; BENCH_ARGS="--config $c --precision fp64" VARIANTS="liblbmr nt128all" bash tools/gpu_variants.sh; done
echo "== sphere_tab1_s3 fp32"; BENCH_ARGS="--config sphere_tab1_s3 --precision fp32" VARIANTS="liblbmr nt128all" bash tools/gpu_variants.sh
