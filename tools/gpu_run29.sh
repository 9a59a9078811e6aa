# bounce-union masks in a per-special-block array (256-byte block record restored)
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r29_pytest.log 2>&1; tail -3 gpurun_out/r29_pytest.log
for c in tunnel4 sphere3 cavity4_kbc; do echo "== $c"; BENCH_ARGS="--config $c" VARIANTS="base liblbmr base liblbmr" bash tools/gpu_variants.sh; done
for c in cavity4_kbc sphere_tab1_s3; do echo "== $c fp64"; BENCH_ARGS="--config $c --precision fp64" VARIANTS="base liblbmr" bash tools/gpu_variants.sh; done
