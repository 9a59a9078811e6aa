# bench line of every config / precision (+ the fusion-ablation schedules on cfg5)
# usage (under gpurun): bash tools/gpu_sweep.sh <tag>
tag=${1:-sweep}
for c in tunnel4 sphere3 uniform512 cavity4_kbc cavity4_bgk cavity2 sphere_tab1_s1 sphere_tab1_s2 sphere_tab1_s3; do
  for p in fp32 fp64; do
    timeout 300 python bench.py --config $c --precision $p --steps 50 --no-cpu-baseline > gpurun_out/${tag}_${c}_${p}.json 2>/dev/null
  done
done
for s in unfused nograph unfused_nograph; do
  timeout 300 python bench.py --config tunnel4 --schedule $s --steps 50 --no-cpu-baseline > gpurun_out/${tag}_tunnel4_fp32_$s.json 2>/dev/null
  timeout 300 python bench.py --config sphere_tab1_s3 --schedule $s --steps 20 --no-cpu-baseline > gpurun_out/${tag}_sphere_tab1_s3_fp64_$s.json 2>/dev/null
done
python tools/sweep_table.py gpurun_out/${tag}_*.json
