# experiment: upper bound of the slow-link path, cfg4 profile
for c in tunnel4 cavity4_kbc cavity4_bgk; do
  BENCH_ARGS="--config $c" VARIANTS="liblbmr noslow" bash tools/gpu_variants.sh
done
timeout 300 python bench.py --config cavity4_kbc --precision fp64 --no-cpu-baseline > gpurun_out/r01b_bench_cavity4_kbc_fp64.json 2>/dev/null
tail -1 gpurun_out/r01b_bench_cavity4_kbc_fp64.json | cut -c1-300
ncu --set full --clock-control none --import-source on -k regex:level_step -s 15 -c 4 -o gpurun_out/prof_cfg4kbc python bench.py --config cavity4_kbc --steps 2 --warmup 3 --no-cpu-baseline --profile-steps 1 > gpurun_out/ncu_cfg4kbc.log 2>&1
tail -1 gpurun_out/ncu_cfg4kbc.log
