"""Short runs for compute-sanitizer (T15): cfg1 cavity (2 levels), a random
2:1 grid with BC leaves, the KBC cavity, every fusion-ablation schedule of
the paper (Fig. 4b-4f: split E / A / O kernels, the atomic scatter
Accumulate) and the in-CTA coalescence gather (CTA_GATHER) on the reduced
tunnel, the warp-cooperative gather kernel on |B| > 4 grids, and 2-slab
partitions with the one-thread wait kernels and with the in-kernel waits,
fp32 and fp64."""
import os
import sys

sys.path.insert(0, os.getcwd())
import lbm_inputs as I  # noqa: E402
from paper_conf_ipps_mahmoudsm24_b200 import lbmr  # noqa: E402

for prec in (lbmr.FP32, lbmr.FP64):
    for prob in (I.cavity2("r"), I.random_balanced(33, n=(9, 11, 10), levels=4, p_refine=0.5),
                 I.cavity4_kbc("mini")):
        g = lbmr.grid_from_problem(prob, precision=prec)
        g.step(2)
        g.macroscopic(prob.levels - 1)
        g.stats()
        g.close()
    prob = I.tunnel4(scale=5)
    for fig, mode in lbmr.FIG4.items():
        g = lbmr.grid_from_problem(prob, precision=prec)
        g.set_schedule(mode)
        g.step(2)
        g.stats()
        g.close()
    os.environ["LBMR_GATHER_WARP"] = "1"
    for prob in (I.random_balanced(33, n=(9, 11, 10), levels=4, p_refine=0.5), I.cavity4_kbc("mini")):
        for mode in (0, lbmr.SCHED_CTA_GATHER):
            g = lbmr.grid_from_problem(prob, precision=prec)
            g.set_schedule(mode)
            g.step(2)
            g.stats()
            g.close()
    os.environ.pop("LBMR_GATHER_WARP", None)
    for spin in ("0", "1"):
        os.environ["LBMR_HALO_SPIN"] = spin
        pg = lbmr.PartitionedGrid(I.cavity2("r"), 2, precision=prec)
        pg.step(2)
        pg.macroscopic(1)
        pg.close()
    os.environ.pop("LBMR_HALO_SPIN", None)
print("sanitize run done")
