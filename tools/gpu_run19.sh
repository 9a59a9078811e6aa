# coalescence gather in (q, ghost) order with SoA candidate slots: parity + A/B vs HEAD build + launch list
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r19_pytest.log 2>&1; tail -3 gpurun_out/r19_pytest.log
for c in tunnel4 sphere3 cavity4_kbc sphere_tab1_s3; do echo "== $c"; BENCH_ARGS="--config $c" VARIANTS="base liblbmr" bash tools/gpu_variants.sh; done
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r19_launches.csv \
    python bench.py --steps 3 --warmup 3 --no-cpu-baseline --profile-steps 1 > /dev/null 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r19_launches_base.csv \
    env LBMR_LIB=$PWD/paper_conf_ipps_mahmoudsm24_b200/_lib/exp/base.so python bench.py --steps 3 --warmup 3 --no-cpu-baseline --profile-steps 1 > /dev/null 2>&1
