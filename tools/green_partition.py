"""The 8-GPU code path on one GPU (diagnostic; run under gpurun): P x-slabs of
a problem, each slab's stream on its own SM-disjoint green context (CUDA 12.4+
driver API), so a slab's spinning protocol CTAs and its PDL-parked CTAs can
never take the SMs its neighbour needs; with LBMR_TEST_OTHER_GPU=1 the library
treats the neighbours like ranks on other GPUs (in-kernel halo waits in the
level and gather kernels, PDL chain).  Prints the max |diff| against one grid.
  python tools/green_partition.py [P=2] [steps=6] [problem=tunnel4_s5] [timed steps=0] [precision 0/1]
"""
import os
import sys

sys.path.insert(0, os.getcwd())
import numpy as np  # noqa: E402


def green_streams(P):
    from cuda.bindings import driver as d
    (err,) = d.cuInit(0)
    err, dev = d.cuDeviceGet(0)
    err, res = d.cuDeviceGetDevResource(dev, d.CUdevResourceType.CU_DEV_RESOURCE_TYPE_SM)
    total = res.sm.smCount
    err, groups, n, rem = d.cuDevSmResourceSplitByCount(P, res, 0, max(8, (total // P) // 8 * 8))
    assert err == d.CUresult.CUDA_SUCCESS and n >= P, (err, n, total)
    streams, keep = [], []
    for i in range(P):
        err, desc = d.cuDevResourceGenerateDesc([groups[i]], 1)
        assert err == d.CUresult.CUDA_SUCCESS, err
        err, gctx = d.cuGreenCtxCreate(desc, dev, d.CUgreenCtxCreate_flags.CU_GREEN_CTX_DEFAULT_STREAM)
        assert err == d.CUresult.CUDA_SUCCESS, err
        err, st = d.cuGreenCtxStreamCreate(gctx, d.CUstream_flags.CU_STREAM_NON_BLOCKING, 0)
        assert err == d.CUresult.CUDA_SUCCESS, err
        streams.append(int(st))
        keep.append((gctx, st))
    return streams, keep, [groups[i].sm.smCount for i in range(P)], total


def run(P, steps, name, time_steps=0, precision=None):
    import torch
    from tools.parity_growth import PROBLEMS
    import lbm_inputs as I
    from paper_conf_ipps_mahmoudsm24_b200 import lbmr
    torch.cuda.init()
    import time
    prob = {"tunnel4_s5": lambda: I.tunnel4(scale=5), "cavity2": lambda: I.cavity2("r"),
            "kbc_mini": lambda: I.cavity4_kbc("mini"), "tunnel4": lambda: I.tunnel4()}.get(
                name, lambda: PROBLEMS[name]())()
    prec = lbmr.FP64 if precision is None else precision
    g1 = lbmr.grid_from_problem(prob, precision=prec)
    g1.step(steps)
    ref = [g1.macroscopic(L) for L in range(prob.levels)]
    upd = sum(int(g1.info().leaves[L]) << L for L in range(prob.levels))
    t1 = None
    if time_steps:
        g1.synchronize()
        t0 = time.perf_counter()
        g1.step(time_steps)
        g1.synchronize()
        t1 = time.perf_counter() - t0
    g1.close()
    streams, keep, sms, total = green_streams(P)
    grids = [lbmr.grid_from_problem(prob, precision=prec, stream=streams[r], n_ranks=P, rank=r)
             for r in range(P)]
    for r, g in enumerate(grids):
        if lbmr.g_has(g, 0):
            g.halo_connect_local(0, grids[(r - 1) % P])
        if lbmr.g_has(g, 1):
            g.halo_connect_local(1, grids[(r + 1) % P])
    launches = [int(g.info().launches_per_step) for g in grids]
    for _ in range(steps):
        for g in grids:
            g.step(1)
    for g in grids:
        g.synchronize()
    worst = 0.0
    for L in range(prob.levels):
        parts = [g.macroscopic(L) for g in grids]
        r = np.concatenate([p[0] for p in parts], axis=0)
        u = np.concatenate([p[1] for p in parts], axis=0)
        m = ~np.isnan(ref[L][0])
        assert np.array_equal(m, ~np.isnan(r)), "fluid sets differ"
        worst = max(worst, float(np.abs(r[m] - ref[L][0][m]).max(initial=0.0)),
                    float(np.abs(u[m] - ref[L][1][m]).max(initial=0.0)))
    tp = None
    if time_steps:
        t0 = time.perf_counter()
        for _ in range(time_steps):
            for g in grids:
                g.step(1)
        for g in grids:
            g.synchronize()
        tp = time.perf_counter() - t0
        print(f"  timing ({time_steps} steps, wall clock incl. launch): one grid on {total} SMs "
              f"{upd * time_steps / t1 / 1e6:.0f} MLUPS; {P} slabs on {sum(sms)} SMs {upd * time_steps / tp / 1e6:.0f} MLUPS")
    for g in grids:
        g.close()
    from cuda.bindings import driver as d
    for gctx, st in keep:
        d.cuStreamDestroy(st)
        d.cuGreenCtxDestroy(gctx)
    print(f"P={P} {name} steps={steps}: SMs per slab {sms} of {total}, launches/step {launches}, "
          f"max |(rho, u) - one grid| = {worst:.3e}")
    return worst


if __name__ == "__main__":
    os.environ["LBMR_TEST_OTHER_GPU"] = "1"
    P = int(sys.argv[1]) if len(sys.argv) > 1 else 2
    steps = int(sys.argv[2]) if len(sys.argv) > 2 else 6
    name = sys.argv[3] if len(sys.argv) > 3 else "tunnel4_s5"
    tsteps = int(sys.argv[4]) if len(sys.argv) > 4 else 0
    prec = int(sys.argv[5]) if len(sys.argv) > 5 else None
    run(P, steps, name, tsteps, prec)
