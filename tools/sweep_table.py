"""Table of bench lines (config, precision, schedule, MLUPS, dominant-level frac, per-level GB/s)."""
import json, sys
rows = []
for f in sorted(sys.argv[1:]):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception:
        print(f"{f}: no bench line")
        continue
    c = d["config"]
    rows.append((c["workload"].split(":")[0], c.get("precision"),
                 c.get("schedule", "fused") + ("/vol" if c.get("variant") == "volumetric" else ""), d["value"],
                 d["roofline"]["frac"], [round(p["GBs"]) for p in d["per_level"]], d.get("vs_baseline"),
                 d["clocks"].get("sm_mhz")))
for r in rows:
    vb = f" vs_paper {r[6]:.2f}x" if r[6] else ""
    print(f"{r[0]:28s} {r[1]:5s} {r[2]:16s} {r[3]:9.0f} MLUPS  frac {r[4]:.3f}  GB/s/level {r[5]}  sm {r[7]}{vb}")
