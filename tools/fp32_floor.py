"""fp32 rounding floor of a problem: the CUDA path built twice with two
equally valid associations of the BGK step ((1-ω) g + ω g^eq, the product, and
g - ω (g - g^eq), LBMR_BGK_ALT_FORM=1 in paper_conf_ipps_mahmoudsm24_b200/
_lib/liblbmr_alt.so), both in fp32, compared with each other and with the fp64
oracle after n coarse steps.  Two correct fp32 evaluations that differ by X
bound how close any fp32 implementation can be expected to stay to the exact
(fp64) trajectory.

  python tools/fp32_floor.py [problem=tunnel4_s5] [steps...]   (run under gpurun; builds nothing)
"""
import json
import os
import subprocess
import sys

sys.path.insert(0, os.getcwd())
import numpy as np  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
ALT = os.path.join(ROOT, "paper_conf_ipps_mahmoudsm24_b200", "_lib", "liblbmr_alt.so")


def child(name, steps, out):
    import lbm_inputs as I  # noqa: F401
    from tools.parity_growth import PROBLEMS
    from paper_conf_ipps_mahmoudsm24_b200 import lbmr
    prob = PROBLEMS[name]()
    g = lbmr.grid_from_problem(prob, precision=lbmr.FP32)
    res = {}
    done = 0
    for n in steps:
        g.step(n - done)
        done = n
        for L in range(prob.levels):
            r, u = g.macroscopic(L)
            res[f"{n}_{L}_r"], res[f"{n}_{L}_u"] = r, u
    np.savez(out, **res)


def main():
    a = sys.argv[1:]
    if a and a[0] == "--child":
        child(a[1], [int(v) for v in a[2].split(",")], a[3])
        return
    name = a[0] if a else "tunnel4_s5"
    steps = [int(v) for v in a[1:]] or [25, 50, 100]
    from tests._parity import errors
    from tools.parity_growth import PROBLEMS
    import oracle
    outs = {}
    for tag, lib in (("product", None), ("alt", ALT)):
        env = dict(os.environ)
        if lib:
            env["LBMR_LIB"] = lib
        out = f"/tmp/fp32_floor_{tag}.npz"
        subprocess.check_call([sys.executable, __file__, "--child", name, ",".join(map(str, steps)), out], env=env,
                              cwd=ROOT)
        outs[tag] = np.load(out)
    prob = PROBLEMS[name]()
    o = oracle.Oracle(prob)
    done = 0
    for n in steps:
        o.step(n - done)
        done = n
        ref = [o.macroscopic(L) for L in range(prob.levels)]
        f = {t: [(outs[t][f"{n}_{L}_r"], outs[t][f"{n}_{L}_u"]) for L in range(prob.levels)] for t in outs}
        print(json.dumps({"problem": name, "steps": n,
                          "product_fp32_vs_oracle": errors(f["product"], ref),
                          "alt_fp32_vs_oracle": errors(f["alt"], ref),
                          "product_fp32_vs_alt_fp32": errors(f["product"], f["alt"])}), flush=True)


if __name__ == "__main__":
    main()
