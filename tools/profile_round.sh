# Full measurement pass for the current build (run under gpurun from the repo root):
#   bench line (cfg5 default), launch list of every kernel, ncu --set full of the
#   four cfg5 level kernels and of the dominant kernel of the other configs,
#   then the sweep of every config / precision / schedule / variant.
# usage: bash tools/profile_round.sh <tag>
tag=${1:-r01}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem --format=csv > gpurun_out/${tag}_gpu.txt
python bench.py > gpurun_out/${tag}_bench.json 2> gpurun_out/${tag}_bench.err
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/${tag}_launches.csv \
    python bench.py --steps 3 --warmup 3 --no-cpu-baseline --profile-steps 1 > /dev/null 2>&1
# cfg5: F3^1 F2^1 F1^1 F0^1 of the second warm-up step
ncu --set full --clock-control none --import-source on -k regex:level_step -s 15 -c 4 -o gpurun_out/${tag}_prof \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline --profile-steps 1 > gpurun_out/${tag}_ncu.log 2>&1
# dominant (finest-level) kernel of the other configs: first launch of the second warm-up step
ncu --set full --clock-control none --import-source on -k regex:level_step -s 15 -c 1 -o gpurun_out/${tag}_prof_cavity4_kbc_fp32 \
    python bench.py --config cavity4_kbc --precision fp32 --steps 2 --warmup 3 --no-cpu-baseline --profile-steps 1 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:level_step -s 7 -c 1 -o gpurun_out/${tag}_prof_sphere_tab1_s3_fp64 \
    python bench.py --config sphere_tab1_s3 --precision fp64 --steps 2 --warmup 3 --no-cpu-baseline --profile-steps 1 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:level_step -s 7 -c 1 -o gpurun_out/${tag}_prof_sphere3_fp32 \
    python bench.py --config sphere3 --precision fp32 --steps 2 --warmup 3 --no-cpu-baseline --profile-steps 1 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:level_step -s 2 -c 1 -o gpurun_out/${tag}_prof_uniform512_fp32 \
    python bench.py --config uniform512 --precision fp32 --steps 2 --warmup 3 --no-cpu-baseline --profile-steps 1 > /dev/null 2>&1
bash tools/gpu_sweep.sh ${tag}sweep > gpurun_out/${tag}_sweep_table.txt 2>&1
for c in tunnel4 sphere3 cavity4_kbc; do
  timeout 300 python bench.py --config $c --variant volumetric --steps 50 --no-cpu-baseline > gpurun_out/${tag}sweep_${c}_fp32_vol.json 2>/dev/null
done
timeout 300 python bench.py --config sphere_tab1_s3 --variant volumetric --steps 20 --no-cpu-baseline > gpurun_out/${tag}sweep_sphere_tab1_s3_fp64_vol.json 2>/dev/null
python tools/sweep_table.py gpurun_out/${tag}sweep_*.json > gpurun_out/${tag}_sweep_table.txt
cat gpurun_out/${tag}_sweep_table.txt
