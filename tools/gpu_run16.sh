LBMR_LIB=$PWD/paper_conf_ipps_mahmoudsm24_b200/_lib/exp/fillfirst.so timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "tunnel or cavity2 or random" 2>&1 | tail -1
BENCH_ARGS="--config tunnel4" VARIANTS="liblbmr fillfirst nofill" bash tools/gpu_variants.sh
BENCH_ARGS="--config sphere3" VARIANTS="liblbmr fillfirst nofill" bash tools/gpu_variants.sh
BENCH_ARGS="--config cavity4_kbc" VARIANTS="liblbmr fillfirst nofill" bash tools/gpu_variants.sh
