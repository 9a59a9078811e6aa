# persistent (cooperative, one launch per lbm_step) schedule: tests + cfg1 / cfg4 / cfg5 timing
timeout 900 python -m pytest tests/test_gpu_schedule_ckpt.py -m gpu -x -q 2>&1 | tail -3
for c in cavity2 cavity4_kbc tunnel4; do for sch in fused persistent; do
  timeout 300 python bench.py --config $c --schedule $sch --steps 50 --no-cpu-baseline > gpurun_out/r45_${c}_${sch}.json 2>gpurun_out/r45_${c}_${sch}.err
  python -c "import json; d=json.load(open('gpurun_out/r45_${c}_${sch}.json')); print('$c $sch', round(d['value']), 'MLUPS', round(d['ms_per_step']*1e3,1), 'us/step')" || tail -3 gpurun_out/r45_${c}_${sch}.err
done; done
for p in fp64; do timeout 300 python bench.py --config cavity2 --precision $p --schedule persistent --steps 50 --no-cpu-baseline > gpurun_out/r45_cavity2_persistent_$p.json 2>/dev/null; python -c "import json; d=json.load(open('gpurun_out/r45_cavity2_persistent_$p.json')); print('cavity2 $p persistent', round(d['value']))"; done
