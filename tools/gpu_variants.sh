run() {  # name lib env...
  name=$1; lib=$2; shift 2
  env "$@" LBMR_LIB=$PWD/paper_conf_ipps_mahmoudsm24_b200/_lib/$lib python bench.py --steps 50 --no-cpu-baseline ${BENCH_ARGS} > gpurun_out/var.json 2>gpurun_out/var.err
  python -c "
import json; d=json.load(open('gpurun_out/var.json'))
print('$name', round(d['value']), 'MLUPS', 'frac', round(d['roofline']['frac'],3), [ (p['level'], round(p['GBs'])) for p in d['per_level']])" || tail -3 gpurun_out/var.err
}
for v in ${VARIANTS:-liblbmr}; do run $v $( [ $v = liblbmr ] && echo liblbmr.so || echo exp/$v.so ); done
