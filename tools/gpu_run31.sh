# skip the bounce-union load in warps without special cells
for c in tunnel4 sphere3; do echo "== $c"; BENCH_ARGS="--config $c" VARIANTS="base liblbmr base liblbmr" bash tools/gpu_variants.sh; done
echo "== cavity4_kbc"; BENCH_ARGS="--config cavity4_kbc" VARIANTS="base liblbmr" bash tools/gpu_variants.sh
ncu --set full --clock-control none --import-source on -k regex:level_step -s 17 -c 1 -o gpurun_out/r31_L1_new \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline --profile-steps 1 > /dev/null 2>&1
