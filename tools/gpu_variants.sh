for v in 0 1; do
  LBMR_VARIANT=$v python bench.py --steps 50 --no-cpu-baseline > gpurun_out/var$v.json 2>gpurun_out/var$v.err
  python -c "
import json; d=json.load(open('gpurun_out/var$v.json'))
print('variant $v', round(d['value']), 'MLUPS', 'frac', round(d['roofline']['frac'],3), [ (p['level'], round(p['GBs'])) for p in d['per_level']])"
done
python -m pytest tests -m gpu -x -q 2>&1 | tail -2
LBMR_VARIANT=1 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
