"""Helpers for GPU-vs-oracle parity (SURVEY §8(c.5) error definitions)."""
from __future__ import annotations

import numpy as np

import oracle

TOL = {0: 1e-5, 1: 1e-12}  # fp32 / fp64 (north_star: ≤1e-5 fp32, ≤1e-12 fp64)


def oracle_run(prob, steps):
    o = oracle.Oracle(prob)
    o.step(steps)
    return [o.macroscopic(L) for L in range(prob.levels)]


def gpu_run(prob, steps, precision, chunks=None):
    from paper_conf_ipps_mahmoudsm24_b200 import lbmr
    g = lbmr.grid_from_problem(prob, precision=precision)
    if chunks:
        for c in chunks:
            g.step(c)
    else:
        g.step(steps)
    out = [g.macroscopic(L) for L in range(prob.levels)]
    g.close()
    return out


def errors(gpu, ora):
    """(err_rho, err_u) normalised by the field maxima over all levels; also
    checks the fluid-leaf sets agree."""
    dr = du = 0.0
    mr = mu = 0.0
    for (rg, ug), (ro, uo) in zip(gpu, ora):
        mo = ~np.isnan(ro)
        mg = ~np.isnan(rg)
        assert np.array_equal(mo, mg), "fluid-leaf sets differ"
        if not mo.any():
            continue
        dr = max(dr, np.abs(rg[mo] - ro[mo]).max())
        du = max(du, np.abs(ug[mo] - uo[mo]).max())
        mr = max(mr, np.abs(ro[mo]).max())
        mu = max(mu, np.abs(uo[mo]).max())
    return dr / mr, (du / mu if mu > 0 else du)
