# bounce word loaded with the fluid/special masks (no extra round trip before the pulls)
for c in tunnel4 sphere3 cavity4_kbc; do echo "== $c"; BENCH_ARGS="--config $c" VARIANTS="base liblbmr base liblbmr" bash tools/gpu_variants.sh; done
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_schedule_ckpt.py -m gpu -x -q 2>&1 | tail -2
