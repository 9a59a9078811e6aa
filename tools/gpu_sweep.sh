# bench line of every config / precision (+ the volumetric variant), round-2 build
# usage (under gpurun): bash tools/gpu_sweep.sh <tag>
tag=${1:-sweep}
for c in tunnel4 sphere3 uniform512 cavity4_kbc cavity4_bgk cavity2 sphere_tab1_s1 sphere_tab1_s2 sphere_tab1_s3; do
  for p in fp32 fp64; do
    timeout 300 python bench.py --config $c --precision $p --steps 30 --no-cpu-baseline --no-secondary --no-ncu-traffic > gpurun_out/${tag}_${c}_${p}.json 2>/dev/null
  done
done
for c in tunnel4 sphere3 cavity4_kbc; do
  timeout 300 python bench.py --config $c --variant volumetric --steps 30 --no-cpu-baseline --no-secondary --no-ncu-traffic > gpurun_out/${tag}_${c}_fp32_vol.json 2>/dev/null
done
timeout 300 python bench.py --config sphere_tab1_s3 --variant volumetric --steps 10 --no-cpu-baseline --no-secondary --no-ncu-traffic > gpurun_out/${tag}_sphere_tab1_s3_fp64_vol.json 2>/dev/null
python tools/sweep_table.py gpurun_out/${tag}_*.json
