timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/r01c_pytest_gpu.txt
cat gpurun_out/r01c_pytest_gpu.txt | tail -3
BENCH_ARGS="--config tunnel4" VARIANTS="liblbmr noslow" bash tools/gpu_variants.sh
BENCH_ARGS="--config cavity4_bgk" VARIANTS="liblbmr noslow" bash tools/gpu_variants.sh
BENCH_ARGS="--config cavity4_kbc" VARIANTS="liblbmr noslow kbcf2 kbcf4" bash tools/gpu_variants.sh
BENCH_ARGS="--config cavity4_kbc --precision fp64" VARIANTS="liblbmr kbcd2" bash tools/gpu_variants.sh
BENCH_ARGS="--config sphere_tab1_s3" VARIANTS="liblbmr kbcd2" bash tools/gpu_variants.sh
for s in unfused nograph unfused_nograph; do BENCH_ARGS="--config tunnel4 --schedule $s" VARIANTS="liblbmr" bash tools/gpu_variants.sh; done
