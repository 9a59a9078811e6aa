"""Summarise an ncu launch list (gpu__time_duration per launch): per kernel and
grid size, count and mean time; the share of one coarse step is taken over the
level_step / coalesce / vavg launches (cold-cache, serialised by ncu: compare shares only)."""
import csv, sys, collections
lines = [l for l in open(sys.argv[1]) if l.startswith('"')]
rows = [r for r in csv.DictReader(lines) if r.get("Metric Name") == "gpu__time_duration.sum"]
agg = collections.OrderedDict()
for r in rows:
    k = (r["Kernel Name"].split("(")[0], r["Grid Size"])
    agg.setdefault(k, []).append(float(r["Metric Value"].replace(",", "")))
STEP = ("level_step", "coalesce", "vavg")  # kernels of the timed coarse steps
step = sum(sum(v) for (n, g), v in agg.items() if any(k in n for k in STEP))
print(f"{'kernel':40s} {'grid':>16s} {'n':>4s} {'mean_us':>9s} {'share_of_step_kernels':>22s}")
for (n, g), v in agg.items():
    share = sum(v) / step if any(k in n for k in STEP) else float("nan")
    print(f"{n[:40]:40s} {g:>16s} {len(v):4d} {sum(v)/len(v)/1e3:9.1f} {share:22.3f}")
