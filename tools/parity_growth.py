"""Growth of the GPU-vs-oracle parity error with the number of coarse steps
(diagnostic for the 100-step bars): for each problem, the oracle and the CUDA
path (fp64 and fp32) are stepped side by side and compared after every
checkpoint; the location (level, cell) of the largest u error is reported.

  python tools/parity_growth.py [problem ...]    (under gpurun; prints JSON lines)
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
    "tunnel4_s5": lambda: I.tunnel4(scale=5),
    "tunnel4_s5_nu0.04": lambda: I.tunnel4(scale=5, nu3=0.04),
    "cavity4_kbc_mini": lambda: I.cavity4_kbc("mini"),
    "cavity2": lambda: I.cavity2(),
    "sphere3_s4_re370": lambda: I.sphere3(scale=4, re=370.0),
}
CHECK = [1, 5, 10, 25, 50, 75, 100]


def worst(gpu, ora):
    best = (0.0, None)
    for L, ((rg, ug), (ro, uo)) in enumerate(zip(gpu, ora)):
        m = ~np.isnan(ro)
        if not m.any():
            continue
        d = np.abs(ug - uo).max(axis=-1)
        d[~m] = 0
        i = np.unravel_index(np.argmax(d), d.shape)
        if d[i] > best[0]:
            best = (float(d[i]), (L, [int(v) for v in i], [float(v) for v in uo[i]]))
    return best


def main(names):
    from paper_conf_ipps_mahmoudsm24_b200 import lbmr
    for name in names:
        prob = PROBLEMS[name]()
        o = oracle.Oracle(prob)
        gs = {p: lbmr.grid_from_problem(prob, precision=p) for p in (lbmr.FP64, lbmr.FP32)}
        done = 0
        for n in CHECK:
            o.step(n - done)
            for g in gs.values():
                g.step(n - done)
            done = n
            ora = [o.macroscopic(L) for L in range(prob.levels)]
            row = {"problem": name, "steps": n}
            for p, g in gs.items():
                got = [g.macroscopic(L) for L in range(prob.levels)]
                er, eu = errors(got, ora)
                w = worst(got, ora)
                row["fp64" if p else "fp32"] = {"err_rho": er, "err_u": eu, "worst_abs_u": w[0], "where": w[1]}
            print(json.dumps(row), flush=True)
        for g in gs.values():
            g.close()


if __name__ == "__main__":
    main(sys.argv[1:] or ["tunnel4_s5", "cavity4_kbc_mini"])
