# early bounce copies (per-warp bounce-union mask in the block record): parity + A/B
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r25_pytest.log 2>&1; tail -3 gpurun_out/r25_pytest.log
for c in tunnel4 sphere3 cavity4_kbc cavity4_bgk; do echo "== $c"; BENCH_ARGS="--config $c" VARIANTS="base liblbmr" bash tools/gpu_variants.sh; done
for c in sphere_tab1_s3 cavity4_kbc; do echo "== $c fp64"; BENCH_ARGS="--config $c --precision fp64" VARIANTS="base liblbmr" bash tools/gpu_variants.sh; done
