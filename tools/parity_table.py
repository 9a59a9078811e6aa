"""Collect the GPU parity log (gpurun_out/parity_errors.jsonl, written by the
-m gpu tests through tests/_parity.record) into one committed JSON:
the last measurement of every (test, config, steps, precision).

  python tools/parity_table.py [log] [out=profiles/r02_parity_errors.json]
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def main(log, out):
    rows = {}
    for line in open(log):
        d = json.loads(line)
        rows[(d["test"], d["config"], d["steps"], d["precision"])] = d
    res = sorted(rows.values(), key=lambda d: (d["test"], d["precision"]))
    worst = {p: max([d["err_u"] for d in res if d["precision"] == p] + [d["err_rho"] for d in res if d["precision"] == p]
                    or [0.0]) for p in ("fp32", "fp64")}
    summary = {"what": "measured GPU-vs-oracle errors of every -m gpu parity check (max error over all fluid leaves "
                       "of all levels, normalised by the field maximum, SURVEY §8(c.5)); bars: fp32 1e-5, fp64 1e-12",
               "n": len(res), "worst": worst,
               "all_within_bar": all(d["err_rho"] <= d["bar"] and d["err_u"] <= d["bar"] for d in res),
               "rows": [{k: v for k, v in d.items() if k != "time"} for d in res]}
    with open(out, "w") as f:
        json.dump(summary, f, indent=1)
    print(f"{len(res)} rows; worst {worst}; all within bar: {summary['all_within_bar']}")


if __name__ == "__main__":
    a = sys.argv[1:]
    main(a[0] if a else os.path.join(ROOT, "gpurun_out", "parity_errors.jsonl"),
         a[1] if len(a) > 1 else os.path.join(ROOT, "profiles", "r02_parity_errors.json"))
