# staged KBC (cp.async pulls into the shared-memory column, collision from there) + bounce copies after the pulls
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
timeout 600 python /tmp/kbcerr.py
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r28_pytest.log 2>&1; tail -3 gpurun_out/r28_pytest.log
echo "== tunnel4"; BENCH_ARGS="--config tunnel4" VARIANTS="base liblbmr base liblbmr" bash tools/gpu_variants.sh
for c in cavity4_kbc sphere_tab1_s3; do
  echo "== $c fp64"; BENCH_ARGS="--config $c --precision fp64" VARIANTS="base nostaged liblbmr stD3" bash tools/gpu_variants.sh
  echo "== $c fp32"; BENCH_ARGS="--config $c --precision fp32" VARIANTS="base nostaged liblbmr stF8" bash tools/gpu_variants.sh
done
