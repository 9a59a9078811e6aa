# KBC moment form: parity errors (KBC cases, both builds), full gpu suite, A/B benches
cat > /tmp/kbcerr.py <<'PY'
import sys; sys.path.insert(0,'.')
import lbm_inputs as I
from tests._parity import errors, gpu_run, oracle_run
for name, p, steps in [("kbcmini", I.cavity4_kbc("mini"), 20), ("tab1s1", I.sphere_tab1(1), 3)]:
    o = oracle_run(p, steps)
    for prec in (1, 0):
        er, eu = errors(gpu_run(p, steps, prec), o)
        print(f"{name:8s} steps={steps:3d} {'fp64' if prec else 'fp32'} err_rho={er:.3e} err_u={eu:.3e}", flush=True)
PY
echo "== new"; timeout 600 python /tmp/kbcerr.py
echo "== base"; LBMR_LIB=$PWD/paper_conf_ipps_mahmoudsm24_b200/_lib/exp/base.so timeout 600 python /tmp/kbcerr.py
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r21_pytest.log 2>&1; tail -3 gpurun_out/r21_pytest.log
for c in cavity4_kbc sphere_tab1_s3 sphere_tab1_s1; do for p in fp32 fp64; do echo "== $c $p"; BENCH_ARGS="--config $c --precision $p" VARIANTS="base liblbmr" bash tools/gpu_variants.sh; done; done
