LBMR_LIB=$PWD/paper_conf_ipps_mahmoudsm24_b200/_lib/exp/pipe.so timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q 2>&1 | tail -2
BENCH_ARGS="--config tunnel4" VARIANTS="liblbmr pipe" bash tools/gpu_variants.sh
BENCH_ARGS="--config tunnel4 --precision fp64" VARIANTS="liblbmr pipe q19d3" bash tools/gpu_variants.sh
BENCH_ARGS="--config cavity4_bgk" VARIANTS="liblbmr pipe" bash tools/gpu_variants.sh
BENCH_ARGS="--config cavity4_kbc" VARIANTS="liblbmr pipe" bash tools/gpu_variants.sh
BENCH_ARGS="--config cavity4_kbc --precision fp64" VARIANTS="liblbmr pipe" bash tools/gpu_variants.sh
BENCH_ARGS="--config sphere_tab1_s3" VARIANTS="liblbmr pipe" bash tools/gpu_variants.sh
BENCH_ARGS="--config uniform512" VARIANTS="liblbmr pipe" bash tools/gpu_variants.sh
