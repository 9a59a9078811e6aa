"""Write profiles/ncu_traffic.json: DRAM bytes per launch (dram__bytes_read.sum +
dram__bytes_write.sum, one `ncu --set full` capture) of each config's dominant
(finest-level) kernel, next to its algorithmic bytes (leaves x 2Q s) — the
`traffic` key of bench.py's roofline object.
usage: python tools/traffic_json.py <tag>   (reads gpurun_out/<tag>_prof*.ncu-rep)"""
import csv, json, os, subprocess, sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
tag = sys.argv[1]


def first_kernel(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    hdr, units, r = rows[0], rows[1], rows[2]

    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9,
             "nsecond": 1e-3, "usecond": 1, "msecond": 1e3, "second": 1e6, "ns": 1e-3, "us": 1, "ms": 1e3, "s": 1e6}

    def val(k):
        i = hdr.index(k)
        return float(r[i].replace(",", "")) * scale.get(units[i], 1)

    return r[hdr.index("Kernel Name")], val("dram__bytes_read.sum") + val("dram__bytes_write.sum"), \
        val("gpu__time_duration.sum")


# config_precision -> (report, Q, bytes per value); finest-level leaves from the sweep's bench line
CASES = {
    "tunnel4_fp32": (f"{tag}_prof", 19, 4),
    "cavity4_kbc_fp32": (f"{tag}_prof_cavity4_kbc_fp32", 27, 4),
    "sphere_tab1_s3_fp64": (f"{tag}_prof_sphere_tab1_s3_fp64", 27, 8),
    "sphere3_fp32": (f"{tag}_prof_sphere3_fp32", 19, 4),
    "uniform512_fp32": (f"{tag}_prof_uniform512_fp32", 19, 4),
}
res = {}
for key, (rep, Q, s) in CASES.items():
    leaves = None
    bj = os.path.join(ROOT, "gpurun_out", f"{tag}sweep_{key}.json")
    if os.path.exists(bj):
        leaves = json.loads(open(bj).read().strip().splitlines()[-1])["config"]["leaves"][-1]
    path = os.path.join(ROOT, "gpurun_out", rep + ".ncu-rep")
    if not os.path.exists(path):
        continue
    name, dram, t = first_kernel(path)
    e = {"kernel": name.split("(")[0].strip() + " (finest level, first launch of a warm-up step)",
         "dram_bytes_per_launch": dram, "duration_us_under_ncu": t,
         "source": f"gpurun_out/{rep}.ncu-rep (ncu --set full --clock-control none, round 1); "
                   "summary in profiles/"}
    if leaves:
        e["algorithmic_bytes_per_launch"] = leaves * 2 * Q * s
        e["traffic_over_algorithmic"] = dram / e["algorithmic_bytes_per_launch"]
    res[key] = e
json.dump(res, open(os.path.join(ROOT, "profiles", "ncu_traffic.json"), "w"), indent=1)
print(json.dumps(res, indent=1))
