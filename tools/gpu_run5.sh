timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "kbc or tab1 or random" 2>&1 | tail -2
BENCH_ARGS="--config cavity4_kbc" VARIANTS="liblbmr" bash tools/gpu_variants.sh
BENCH_ARGS="--config cavity4_kbc --precision fp64" VARIANTS="liblbmr" bash tools/gpu_variants.sh
BENCH_ARGS="--config sphere_tab1_s3" VARIANTS="liblbmr" bash tools/gpu_variants.sh
ncu --set full --clock-control none --import-source on -k regex:level_step -s 15 -c 1 -o gpurun_out/prof_cfg4kbc_r5 python bench.py --config cavity4_kbc --steps 2 --warmup 3 --no-cpu-baseline --profile-steps 1 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:level_step -s 7 -c 1 -o gpurun_out/prof_tab1s3_r5 python bench.py --config sphere_tab1_s3 --steps 2 --warmup 3 --no-cpu-baseline --profile-steps 1 > /dev/null 2>&1
ls gpurun_out
