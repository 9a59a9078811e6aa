#!/usr/bin/env python
"""Mutation check of the oracle pins.

Each mutation is a plausible mistake in oracle/lbm_oracle.cpp (a dropped term,
a wrong sign, index or divisor, the other reading of an ambiguous passage).
The mutated source is compiled to a temporary liboracle.so, and the CPU pin
suites run against it through ORACLE_LIB.  A mutation is "caught" when at
least one pin fails; the report also says whether a pin other than T11 (the
numpy brute force, which restates the rules) catches it.

  python tools/mutation_test.py [--out profiles/r02_mutation.txt]
"""
from __future__ import annotations

import argparse
import os
import re
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = os.path.join(ROOT, "oracle", "lbm_oracle.cpp")
SUITES = ["tests/test_oracle_pins.py", "tests/test_oracle_bc_kbc_pins.py"]

# (name, what it models, exact text, replacement)
MUTATIONS = [
    ("kbc_gamma_sign", "KBC: sign slip in the (2 - 1/beta) term of gamma",
     "1.0 / beta - (2.0 - 1.0 / beta) * sh / hh", "1.0 / beta + (2.0 - 1.0 / beta) * sh / hh"),
    ("kbc_gamma_weight", "KBC: entropic inner product weighted by 1/w_i instead of 1/f^eq_i",
     "sh += ds[i] * dh[i] / feq[i];\n    hh += dh[i] * dh[i] / feq[i];",
     "sh += ds[i] * dh[i] / lat.w[i];\n    hh += dh[i] * dh[i] / lat.w[i];"),
    ("kbc_gamma_const", "KBC: gamma fixed at 1/beta (entropic correction dropped)",
     "1.0 / beta - (2.0 - 1.0 / beta) * sh / hh", "1.0 / beta"),
    ("kbc_ds_edge", "KBC: edge shear part with 1/2 instead of 1/4",
     "if (ez == 0) s = ex * ey * P[0][1] / 4.0;", "if (ez == 0) s = ex * ey * P[0][1] / 2.0;"),
    ("outflow_as_bounceback", "OUTFLOW treated as halfway bounce-back",
     "if (kind == BC_OUTFLOW) return lat.w[i];\n  double v = V.fs", "double v = V.fs"),
    ("outflow_zero_gradient", "OUTFLOW copies the cell's own post-collision f_i",
     "if (kind == BC_OUTFLOW) return lat.w[i];\n  double v = V.fs",
     "if (kind == BC_OUTFLOW) return V.fs[k * lat.Q + i];\n  double v = V.fs"),
    ("outflow_zero", "OUTFLOW assigns 0 instead of w_i",
     "if (kind == BC_OUTFLOW) return lat.w[i];\n  double v = V.fs",
     "if (kind == BC_OUTFLOW) return 0.0;\n  double v = V.fs"),
    ("inlet_sign", "VELOCITY: moving-wall term subtracted",
     "v += 6.0 * lat.w[i] * 1.0 * eu;\n  }\n  return v;\n}\n\n// Face-BC",
     "v -= 6.0 * lat.w[i] * 1.0 * eu;\n  }\n  return v;\n}\n\n// Face-BC"),
    ("inlet_factor", "VELOCITY: 2 w_i e.u instead of 2 w_i e.u / c_s^2",
     "v += 6.0 * lat.w[i] * 1.0 * eu;\n  }\n  return v;\n}\n\n// Face-BC",
     "v += 2.0 * lat.w[i] * 1.0 * eu;\n  }\n  return v;\n}\n\n// Face-BC"),
    ("bounce_same_direction", "bounce-back returns f*_i instead of f*_opp(i)",
     "double v = V.fs[k * lat.Q + lat.opp[i]];", "double v = V.fs[k * lat.Q + i];"),
    ("face_priority", "edge priority NOSLIP below OUTFLOW",
     "int pr = kind == BC_VELOCITY ? 3 : kind == BC_NOSLIP ? 2 : 1;",
     "int pr = kind == BC_VELOCITY ? 3 : kind == BC_NOSLIP ? 1 : 2;"),
    ("coal_divisor_8", "Coalescence divisor n = 8 (volume ratio) instead of 2|B|",
     "val = acc / (2.0 * nb);", "val = acc / 8.0;"),
    ("coal_one_substep", "Coalescence averages the second fine substep twice",
     "for (int m = 0; m < nb; ++m) acc += F.p1[blist[m] * Q + i];",
     "for (int m = 0; m < nb; ++m) acc += F.fs[blist[m] * Q + i];"),
    ("coal_parent_children", "Coalescence over p's own children (the rejected reading of R-A2)",
     "int64_t b[3] = {2 * p[0] - lat.e[i][0] + cx, 2 * p[1] - lat.e[i][1] + cy,\n"
     "                                2 * p[2] - lat.e[i][2] + cz};",
     "int64_t b[3] = {2 * p[0] + cx, 2 * p[1] + cy,\n"
     "                                2 * p[2] + cz};"),
    ("explosion_from_parent", "Explosion reads p's own parent instead of the leaf containing p - e_i",
     "int64_t Sc = C.idx(s[0] >> 1, s[1] >> 1, s[2] >> 1);\n          int code = C.code[Sc];",
     "int64_t Sc = C.idx(p[0] >> 1, p[1] >> 1, p[2] >> 1);\n          int code = C.code[Sc];"),
    ("omega_not_rescaled", "omega_L = omega_0 on every level (Eq.9 dropped)",
     "return 2.0 * omega0 / (2.0 * p + (1.0 - p) * omega0);", "return omega0 + 0.0 * p;"),
    ("equilibrium_quadratic", "Eq.5 quadratic term (e.u)^2/c_s^4 instead of /(2 c_s^4)",
     "(eu * eu) / (2.0 * cs2 * cs2)", "(eu * eu) / (cs2 * cs2)"),
    ("bgk_sign", "BGK relaxes away from equilibrium",
     "fs[i] = f[i] - omega * (f[i] - feq[i]);", "fs[i] = f[i] + omega * (f[i] - feq[i]);"),
    ("accumulate_dropped", "first fine post-collision state not kept (P1 stale)",
     "g->lv[L + 1].p1 = g->lv[L + 1].fs;", "(void)0;"),
    ("substep_once", "one fine substep per coarse substep (acoustic scaling dropped)",
     "    g->lv[L + 1].p1 = g->lv[L + 1].fs;  // Accumulate: keep the first fine post-collision state\n"
     "    substep(g, L + 1);",
     "    g->lv[L + 1].p1 = g->lv[L + 1].fs;  // Accumulate: keep the first fine post-collision state\n"
     "    (void)0;"),
]


def run_suite(lib: str):
    env = dict(os.environ, ORACLE_LIB=lib)
    cmd = [sys.executable, "-m", "pytest", *SUITES, "-q", "-m", "not gpu", "-p", "no:cacheprovider", "-rf",
           "--timeout", "600"]
    r = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True)
    failed = sorted(set(re.findall(r"^FAILED (\S+)", r.stdout, re.M)))
    errors = sorted(set(re.findall(r"^ERROR (\S+)", r.stdout, re.M)))
    tail = r.stdout.strip().splitlines()[-1] if r.stdout.strip() else r.stderr.strip()[-200:]
    return r.returncode, failed + errors, tail


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "r02_mutation.txt"))
    ap.add_argument("--only", default=None)
    args = ap.parse_args()
    src = open(SRC).read()
    lines = []
    tmp = tempfile.mkdtemp(prefix="oracle_mut_")
    # the unmutated oracle must pass
    base = os.path.join(tmp, "base.so")
    subprocess.check_call(["g++", "-O2", "-std=c++17", "-fopenmp", "-fPIC", "-shared", "-o", base, SRC])
    rc, failed, tail = run_suite(base)
    lines.append(f"baseline (unmutated oracle): rc={rc}  {tail}")
    assert rc == 0, failed
    caught_all = True
    for name, what, old, new in MUTATIONS:
        if args.only and name != args.only:
            continue
        n = src.count(old)
        if n != 1:
            lines.append(f"{name}: MUTATION TEXT FOUND {n} TIMES — not applied")
            caught_all = False
            continue
        msrc = os.path.join(tmp, name + ".cpp")
        open(msrc, "w").write(src.replace(old, new))
        lib = os.path.join(tmp, name + ".so")
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-fopenmp", "-fPIC", "-shared", "-o", lib, msrc])
        rc, failed, tail = run_suite(lib)
        non_brute = [f for f in failed if "test_T11" not in f]
        ok = rc != 0
        caught_all &= ok
        lines.append(f"{name}: {'CAUGHT' if ok else 'MISSED'} ({len(failed)} failing, "
                     f"{len(non_brute)} outside the T11 brute force) — {what}")
        for f in failed:
            lines.append(f"    {f.split('::', 1)[-1]}")
        print(lines[-1 - len(failed)], flush=True)
    lines.append(f"all mutations caught: {caught_all}")
    hdr = ("# Oracle mutation check (tools/mutation_test.py): each line is one deliberate mistake in\n"
           "# oracle/lbm_oracle.cpp, compiled separately and run against the CPU pin suites\n"
           f"# {', '.join(SUITES)} via ORACLE_LIB.\n")
    with open(args.out, "w") as f:
        f.write(hdr + "\n".join(lines) + "\n")
    print("\n".join(lines[-1:]))
    return 0 if caught_all else 1


if __name__ == "__main__":
    sys.exit(main())
