run() {  # name lib env...
  name=$1; lib=$2; shift 2
  env "$@" LBMR_LIB=$PWD/paper_conf_ipps_mahmoudsm24_b200/_lib/$lib python bench.py --steps 50 --no-cpu-baseline > gpurun_out/var.json 2>gpurun_out/var.err
  python -c "
import json; d=json.load(open('gpurun_out/var.json'))
print('$name', round(d['value']), 'MLUPS', 'frac', round(d['roofline']['frac'],3), [ (p['level'], round(p['GBs'])) for p in d['per_level']])"
}
run single5 liblbmr.so LBMR_SPLIT=0
run single6 exp/occ6.so LBMR_SPLIT=0
run single4 exp/occ4.so LBMR_SPLIT=0
run split5 liblbmr.so LBMR_SPLIT=1
run split6 exp/occ6.so LBMR_SPLIT=1
python -m pytest tests -m gpu -x -q 2>&1 | tail -2
LBMR_SPLIT=1 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
LBMR_SPLIT=1 ncu --set full --clock-control none -k regex:level_step -s 30 -c 4 -o gpurun_out/prof_split2 python bench.py --steps 2 --warmup 3 --no-cpu-baseline --profile-steps 1 > /dev/null 2>&1
