"""Fig. 9-shaped table of the fusion ablation: MLUPS of every
schedule (bench.py --schedule) per workload, from bench JSON lines named
<prefix>_<config>_<schedule>.json.

  python tools/ablation_table.py gpurun_out/r02_fig9 > profiles/r02_fig9_ablation.txt
"""
import glob
import json
import os
import sys

ORDER = ["fig4b", "fig4c", "fig4d", "fig4e", "fig4f", "unfused", "cta_gather", "fused"]
LABEL = {"fig4b": "4b modified baseline (C, A, S, E, O separate)", "fig4c": "4c CA fused (atomic Accumulate)",
         "fig4d": "4d SE fused", "fig4e": "4e CA, SE, SO fused", "fig4f": "4f CASE + SO fused (atomic A)",
         "unfused": "C | SEO (gather A+A+O)", "cta_gather": "CSEO + A+A+O in one kernel (in-CTA gather)",
         "fused": "product: CSEO fused, gather A+A+O (PDL)"}


def main(prefix):
    rows = {}
    for f in sorted(glob.glob(prefix + "_*.json")):
        base = os.path.basename(f)[len(os.path.basename(prefix)) + 1:-5]
        sched = next((s for s in ORDER if base.endswith("_" + s)), None)
        if sched is None:
            continue
        cfg = base[: -len(sched) - 1]
        try:
            d = json.loads(open(f).read().strip().splitlines()[-1])
        except Exception:  # noqa: BLE001
            continue
        rows.setdefault(cfg, {})[sched] = d
    cfgs = sorted(rows)
    print("# Fusion ablation (bench.py --schedule, 1 B200, MLUPS fine-equivalent, CUDA-event timed graph replays)")
    print("# speedup = MLUPS / MLUPS of the 4b modified baseline of the same workload; paper (A100, Tab. I): 4f/4b = 2.20 / 1.40 / 1.30 at s1/s2/s3")
    hdr = f"{'schedule':48s}" + "".join(f"{c:>26s}" for c in cfgs)
    print(hdr)
    for s in ORDER:
        line = f"{LABEL[s]:48s}"
        for c in cfgs:
            d = rows[c].get(s)
            b = rows[c].get("fig4b")
            if d is None:
                line += f"{'-':>26s}"
                continue
            sp = d["value"] / b["value"] if b else float("nan")
            line += f"{d['value']:>12.0f} ({sp:4.2f}x) {d['dtype']:>4s}  "
        print(line)
    for c in cfgs:
        any_d = next(iter(rows[c].values()))
        print(f"# {c}: {any_d['config']['workload']}; launches/step " +
              ", ".join(f"{s}={rows[c][s]['gpu_launches'] // rows[c][s]['steps']}" for s in ORDER if s in rows[c]))


if __name__ == "__main__":
    main(sys.argv[1])
