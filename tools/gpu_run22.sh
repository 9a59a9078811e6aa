# KBC occupancy re-sweep after the moment-form collision
for c in cavity4_kbc sphere_tab1_s3; do
  echo "== $c fp32"; BENCH_ARGS="--config $c --precision fp32" VARIANTS="liblbmr kbcf5 kbcf3" bash tools/gpu_variants.sh
  echo "== $c fp64"; BENCH_ARGS="--config $c --precision fp64" VARIANTS="liblbmr kbcd3" bash tools/gpu_variants.sh
done
