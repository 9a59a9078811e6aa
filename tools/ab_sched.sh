# A/B of build / schedule variants (bench.py), alternating, R repetitions per config
# usage (under gpurun): bash tools/ab_sched.sh <tag> <R> "<variants>" [configs...]
#   variant = name:schedule[:lib[:VAR=value]]   (lib = a .so under paper_conf_ipps_mahmoudsm24_b200/_lib,
#             default liblbmr.so; VAR=value an environment setting for that run)
#   config  = config:precision
tag=$1; R=$2; variants=$3; shift 3
cfgs=${@:-"tunnel4:fp32 sphere3:fp32 cavity4_kbc:fp32 sphere_tab1_s3:fp64 tunnel4:fp64"}
libdir=$PWD/paper_conf_ipps_mahmoudsm24_b200/_lib
for cp in $cfgs; do
  c=${cp%%:*}; p=${cp##*:}
  for r in $(seq 1 $R); do
    for v in $variants; do
      IFS=: read -r name sched lib envset <<< "$v"
      env ${envset:-LBMR_AB=1} LBMR_LIB=$libdir/${lib:-liblbmr.so} timeout 300 python bench.py --config $c --precision $p --schedule $sched \
        --steps 30 --no-cpu-baseline --no-secondary --no-ncu-traffic > gpurun_out/${tag}_${c}_${p}_${name}_${r}.json 2>/dev/null
    done
  done
done
python - "$tag" <<'PY'
import glob, json, sys, collections
tag = sys.argv[1]
rows = collections.defaultdict(list)
for f in sorted(glob.glob(f"gpurun_out/{tag}_*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception:
        continue
    key = f[len(f"gpurun_out/{tag}_"):-5].rsplit("_", 1)[0]
    lv = " ".join(f"{x['frac']:.3f}/{x.get('frac_incl_gather', x['frac']):.3f}" for x in d.get("per_level", []))
    rows[key].append((d["value"], d["clocks"]["sm_mhz"], lv))
for k, v in rows.items():
    for val, mhz, lv in v:
        print(f"{k:44s} {val:10.0f} MLUPS  {mhz:6.0f} MHz  per-level {lv}")
    print(f"{k:44s} mean {sum(x[0] for x in v) / len(v):10.0f}")
PY
