"""Conditioning of the KBC step (reading R-A9) over many coarse steps: how far
two exact-arithmetic-equivalent fp64 runs drift apart when their inputs
differ by rounding only.

The oracle is run on the problem and on the same problem whose initial
density and velocity fields carry a relative perturbation of `eps` (a few
ulps); the drift between the two oracle runs (SURVEY §8(c.5) error measure)
is the problem's own sensitivity to rounding.  The CUDA path in fp64 is
compared with the unperturbed oracle at the same step counts.  A CUDA error of
the size of the oracle's own perturbation drift is rounding, not a rule
difference.

  python tools/kbc_conditioning.py [problem=cavity4_kbc_mini] [eps=4e-16]
"""
import json
import os
import sys

sys.path.insert(0, os.getcwd())
import numpy as np  # noqa: E402

import lbm_inputs as I  # noqa: E402
import oracle  # noqa: E402
from tests._parity import errors  # noqa: E402

PROBLEMS = {
    "cavity4_kbc_mini": lambda: I.cavity4_kbc("mini"),
    "cavity4_bgk_mini": lambda: I.cavity4_kbc("mini", collision="bgk"),
    "tunnel4_s5": lambda: I.tunnel4(scale=5),
    "tunnel4_s5_nu0.04": lambda: I.tunnel4(scale=5, nu3=0.04),
}
CHECK = [10, 25, 50, 75, 100]


def perturbed(prob, eps, seed=7):
    rng = np.random.default_rng(seed)
    p = PROBLEMS[NAME]()
    p.init_rho, p.init_u = [], []
    for L in range(prob.levels):
        r, u = prob.init_fields(L)
        p.init_rho.append(r * (1 + eps * rng.uniform(-1, 1, r.shape)))
        p.init_u.append(u + eps * np.abs(u).max() * rng.uniform(-1, 1, u.shape) if np.abs(u).max() > 0
                        else u + eps * 1e-2 * rng.uniform(-1, 1, u.shape))
    return p


def main():
    global NAME
    NAME = sys.argv[1] if len(sys.argv) > 1 else "cavity4_kbc_mini"
    eps = float(sys.argv[2]) if len(sys.argv) > 2 else 4e-16
    prob = PROBLEMS[NAME]()
    o = oracle.Oracle(prob)
    op = oracle.Oracle(perturbed(prob, eps))
    from paper_conf_ipps_mahmoudsm24_b200 import lbmr
    g = lbmr.grid_from_problem(prob, precision=lbmr.FP64)
    done = 0
    for n in CHECK:
        o.step(n - done)
        op.step(n - done)
        g.step(n - done)
        done = n
        ref = [o.macroscopic(L) for L in range(prob.levels)]
        dp = errors([op.macroscopic(L) for L in range(prob.levels)], ref)
        dg = errors([g.macroscopic(L) for L in range(prob.levels)], ref)
        print(json.dumps({"problem": NAME, "steps": n, "eps": eps, "oracle_vs_perturbed_oracle": {"err_rho": dp[0],
                          "err_u": dp[1]}, "gpu_fp64_vs_oracle": {"err_rho": dg[0], "err_u": dg[1]}}), flush=True)
    g.close()


if __name__ == "__main__":
    main()
