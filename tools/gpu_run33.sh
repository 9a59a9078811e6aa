# D3Q19 special-path order: base (HEAD~3) vs info-first + double wall velocity (dvel) vs early for all lattices (early)
for c in tunnel4 sphere3; do echo "== $c"; BENCH_ARGS="--config $c" VARIANTS="base dvel early base dvel early" bash tools/gpu_variants.sh; done
echo "== cavity4_kbc"; BENCH_ARGS="--config cavity4_kbc" VARIANTS="dvel early" bash tools/gpu_variants.sh
