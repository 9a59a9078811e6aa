# early bounce for D3Q27 only (D3Q19 back to the info-first order)
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r32_pytest.log 2>&1; tail -3 gpurun_out/r32_pytest.log
for c in tunnel4 sphere3 cavity4_kbc cavity4_bgk; do echo "== $c"; BENCH_ARGS="--config $c" VARIANTS="base liblbmr base liblbmr" bash tools/gpu_variants.sh; done
for c in cavity4_kbc sphere_tab1_s3; do echo "== $c fp64"; BENCH_ARGS="--config $c --precision fp64" VARIANTS="base liblbmr" bash tools/gpu_variants.sh; done
echo "== tunnel4 fp64"; BENCH_ARGS="--config tunnel4 --precision fp64" VARIANTS="base liblbmr" bash tools/gpu_variants.sh
