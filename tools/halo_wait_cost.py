"""Cost of the one-thread halo-wait kernels: the reduced
tunnel on one GPU as one grid and as P in-process slabs, with the wait
kernels (ranks sharing a GPU, the default there) and with the in-kernel waits
forced on (LBMR_HALO_SPIN=1, the distinct-GPU form); wall time per coarse
step over n steps after a warm-up, all streams synchronised.

  python tools/halo_wait_cost.py [P=2] [scale=5] [steps=50]   (under gpurun)
"""
import json
import os
import sys
import time

sys.path.insert(0, os.getcwd())
import lbm_inputs as I  # noqa: E402


def timed(fn_step, sync, n):
    fn_step(3)
    sync()
    t0 = time.perf_counter()
    fn_step(n)
    sync()
    return (time.perf_counter() - t0) / n * 1e6


def main():
    P = int(sys.argv[1]) if len(sys.argv) > 1 else 2
    scale = int(sys.argv[2]) if len(sys.argv) > 2 else 5
    n = int(sys.argv[3]) if len(sys.argv) > 3 else 50
    from paper_conf_ipps_mahmoudsm24_b200 import lbmr
    prob = I.tunnel4(scale=scale)
    res = {"problem": prob.name, "P": P, "steps": n}
    g = lbmr.grid_from_problem(prob, precision=lbmr.FP32)
    res["single_grid_us_per_step"] = timed(g.step, g.synchronize, n)
    res["single_launches_per_step"] = int(g.info().launches_per_step)
    g.close()
    for spin in ("0", "1"):
        os.environ["LBMR_HALO_SPIN"] = spin
        pg = lbmr.PartitionedGrid(prob, P, precision=lbmr.FP32)
        key = "in_kernel_wait" if spin == "1" else "wait_kernels"
        res[key + "_us_per_step"] = timed(pg.step, pg.synchronize, n)
        res[key + "_launches_per_step_per_slab"] = int(pg.grids[0].info().launches_per_step)
        pg.close()
    os.environ.pop("LBMR_HALO_SPIN", None)
    print(json.dumps(res), flush=True)


if __name__ == "__main__":
    main()
