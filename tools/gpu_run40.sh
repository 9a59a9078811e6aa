# 128-thread CTAs everywhere (default now) vs 64-thread CTAs; full gpu suite on the default
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r40_pytest.log 2>&1; tail -3 gpurun_out/r40_pytest.log
for c in tunnel4 sphere3 cavity4_kbc uniform512; do echo "== $c"; BENCH_ARGS="--config $c" VARIANTS="liblbmr nt64all liblbmr nt64all" bash tools/gpu_variants.sh; done
echo "== sphere_tab1_s3 fp64"; BENCH_ARGS="--config sphere_tab1_s3 --precision fp64" VARIANTS="liblbmr nt64all" bash tools/gpu_variants.sh
