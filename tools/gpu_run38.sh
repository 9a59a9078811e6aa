# fp64 KBC with 128-thread CTAs (quarter blocks): 4 or 5 CTAs/SM
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edge.py -m gpu -x -q 2>&1 | tail -2
for c in sphere_tab1_s3 cavity4_kbc; do echo "== $c fp64"; BENCH_ARGS="--config $c --precision fp64" VARIANTS="liblbmr nt128m4 nt128m5 liblbmr nt128m5" bash tools/gpu_variants.sh; done
LBMR_LIB=$PWD/paper_conf_ipps_mahmoudsm24_b200/_lib/exp/nt128m5.so timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "kbc or tab1 or random" 2>&1 | tail -2
