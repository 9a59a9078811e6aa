"""Helpers for GPU-vs-oracle parity (SURVEY §8(c.5) error definitions)."""
from __future__ import annotations

import json
import os
import time

import numpy as np

import oracle

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
# every GPU parity check appends its measured errors here (gpurun merges
# gpurun_out/ back; tools/parity_table.py turns it into
# profiles/r02_parity_errors.json)
PARITY_LOG = os.environ.get("LBMR_PARITY_LOG", os.path.join(ROOT, "gpurun_out", "parity_errors.jsonl"))


def record(test: str, config: str, steps: int, precision: int, err_rho: float, err_u: float, bar=None, **extra):
    """Append one measured (err_rho, err_u) to the parity log (best effort)."""
    try:
        os.makedirs(os.path.dirname(PARITY_LOG), exist_ok=True)
        line = {"test": test, "config": config, "steps": int(steps), "precision": "fp64" if precision else "fp32",
                "err_rho": float(err_rho), "err_u": float(err_u), "bar": float(bar if bar is not None else TOL[precision]),
                "time": time.time(), **extra}
        with open(PARITY_LOG, "a") as f:
            f.write(json.dumps(line) + "\n")
    except OSError:
        pass

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


def errors(gpu, ora, prec=None, steps=None, config=None):
    """(err_rho, err_u) normalised by the field maxima over all levels; also
    checks the fluid-leaf sets agree.  With prec given, the result is also
    appended to the parity log (record)."""
    er, eu = _errors(gpu, ora)
    if prec is not None:
        test = os.environ.get("PYTEST_CURRENT_TEST", "?").split(" ")[0]
        record(test, str(config), int(steps or 0), prec, er, eu)
    return er, eu


def _errors(gpu, ora):
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


def rounding_drift(prob, steps, eps=4e-16, seed=7):
    """The problem's own sensitivity to rounding (reading R-B4): the
    (err_rho, err_u) between the oracle run on `prob` and the oracle run on
    the same problem whose initial density carries a relative perturbation of
    `eps` (2 ulps of 1.0 in fp64), after `steps` coarse steps.  Two fp64
    implementations of the same rules cannot be expected to agree more
    closely than this."""
    import dataclasses
    rng = np.random.default_rng(seed)
    p = dataclasses.replace(prob)
    p.init_rho, p.init_u = [], []
    for L in range(prob.levels):
        r, u = prob.init_fields(L)
        p.init_rho.append(r * (1 + eps * rng.uniform(-1, 1, r.shape)))
        p.init_u.append(u)
    return _errors(oracle_run(p, steps), oracle_run(prob, steps))


def fp32_rounding_floor(name, steps, got):
    """fp32 rounding floor (reading R-B5): the CUDA fp32 result `got`
    of problem `name` (tools/parity_growth.PROBLEMS) against the same step
    computed by the diagnostic build liblbmr_alt.so, whose BGK step is the
    same formula in another association (g - ω (g - g^eq) instead of
    (1 - ω) g + ω g^eq).  Two equally valid fp32 evaluations differing by X
    bound how close any fp32 implementation can stay to the exact (fp64)
    trajectory.  Returns (err_rho, err_u) between the two."""
    import subprocess
    import sys
    import tempfile
    lib = os.path.join(ROOT, "paper_conf_ipps_mahmoudsm24_b200", "_lib", "liblbmr_alt.so")
    if not os.path.exists(lib):
        from paper_conf_ipps_mahmoudsm24_b200 import _build
        _build.build_alt()
    out = os.path.join(tempfile.mkdtemp(), "alt.npz")
    subprocess.check_call([sys.executable, os.path.join(ROOT, "tools", "fp32_floor.py"), "--child", name, str(steps),
                           out], env=dict(os.environ, LBMR_LIB=lib), cwd=ROOT)
    z = np.load(out)
    alt = [(z[f"{steps}_{L}_r"], z[f"{steps}_{L}_u"]) for L in range(len(got))]
    return _errors(got, alt)
