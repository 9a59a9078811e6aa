import sys; sys.path.insert(0,'.')
import lbm_inputs as I
from tests._parity import errors, gpu_run, oracle_run
for name, p, steps in [("cav2", I.cavity2(), 100), ("cav2r", I.cavity2("r"), 20), ("sphere4", I.sphere3(scale=4), 20),
                       ("kbcmini", I.cavity4_kbc("mini"), 6), ("tunnel5", I.tunnel4(scale=5), 4),
                       ("rand33", I.random_balanced(33, n=(9,11,10), levels=4, p_refine=0.5), 6)]:
    o = oracle_run(p, steps)
    for prec in (1, 0):
        er, eu = errors(gpu_run(p, steps, prec), o)
        print(f"{name:8s} steps={steps:3d} {'fp64' if prec else 'fp32'} err_rho={er:.3e} err_u={eu:.3e}", flush=True)
