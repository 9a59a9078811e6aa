# ci after the pulls + wall velocity in kernel precision; D3Q19 fp32 at 5 CTAs/SM; repeated A/B
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r26_pytest.log 2>&1; tail -3 gpurun_out/r26_pytest.log
for c in tunnel4 sphere3 cavity4_kbc; do echo "== $c"; BENCH_ARGS="--config $c" VARIANTS="base liblbmr q19f5 base liblbmr" bash tools/gpu_variants.sh; done
