for cfg in ${CONFIGS:-tunnel4 sphere3 cavity4_kbc uniform512 cavity2}; do
  for prec in ${PRECS:-fp32 fp64}; do
    python bench.py --config $cfg --precision $prec --steps ${STEPS:-20} --no-cpu-baseline > gpurun_out/cfg_${cfg}_${prec}.json 2>gpurun_out/cfg.err
    python -c "
import json; d=json.load(open('gpurun_out/cfg_${cfg}_${prec}.json'))
print('$cfg $prec', round(d['value']), 'MLUPS', 'ms/step', round(d['ms_per_step'],3), 'dom frac', round(d['roofline']['frac'],3), 'step frac', round(d['roofline']['step_frac'],3), [ (p['level'], round(p['GBs']), round(p['share_of_step'],3)) for p in d['per_level']])" || tail -3 gpurun_out/cfg.err
  done
done
