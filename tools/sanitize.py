"""Short runs for compute-sanitizer (T15): cfg1 cavity (2 levels), a random
2:1 grid with BC leaves, and a 2-slab partition, fp32 and fp64."""
import os, sys
sys.path.insert(0, os.getcwd())
import lbm_inputs as I
from paper_conf_ipps_mahmoudsm24_b200 import lbmr
for prec in (lbmr.FP32, lbmr.FP64):
    for prob in (I.cavity2("r"), I.random_balanced(33, n=(9, 11, 10), levels=4, p_refine=0.5),
                 I.cavity4_kbc("mini")):
        g = lbmr.grid_from_problem(prob, precision=prec)
        g.step(2)
        g.macroscopic(prob.levels - 1)
        g.stats()
        g.close()
    pg = lbmr.PartitionedGrid(I.cavity2("r"), 2, precision=prec)
    pg.step(2)
    pg.macroscopic(1)
    pg.close()
print("sanitize run done")
