# Full measurement pass for the current build (run under gpurun from the repo root):
#   bench line (cfg5 default incl. secondary blocks, in-run ncu traffic, cpu baseline), launch list of
#   every kernel of two coarse steps, ncu --set full of the four cfg5 level kernels and of the
#   dominant kernel of the other configs, then the sweep of every config / precision / variant.
# usage: bash tools/profile_round.sh <tag>
tag=${1:-r02}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem --format=csv > gpurun_out/${tag}_gpu.txt
python bench.py > gpurun_out/${tag}_bench.json 2> gpurun_out/${tag}_bench.err
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/${tag}_launches.csv \
    python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-secondary --no-ncu-traffic --profile-steps 1 > /dev/null 2>&1
# cfg5: F3 F2 F1 F0 of the second coarse step (2 steps of 15 level-kernel launches)
ncu --set full --clock-control none --import-source on -k regex:level_step_all -s 15 -c 4 -o gpurun_out/${tag}_prof \
    python bench.py --traffic-child --config tunnel4 > gpurun_out/${tag}_ncu.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:level_step_all -s 15 -c 1 -o gpurun_out/${tag}_prof_cavity4_kbc_fp32 \
    python bench.py --traffic-child --config cavity4_kbc --precision fp32 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:level_step_all -s 7 -c 1 -o gpurun_out/${tag}_prof_sphere_tab1_s3_fp64 \
    python bench.py --traffic-child --config sphere_tab1_s3 --precision fp64 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:level_step_all -s 15 -c 1 -o gpurun_out/${tag}_prof_tunnel4_fp64 \
    python bench.py --traffic-child --config tunnel4 --precision fp64 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:level_step_all -s 1 -c 1 -o gpurun_out/${tag}_prof_uniform512_fp32 \
    python bench.py --traffic-child --config uniform512 --precision fp32 > /dev/null 2>&1
bash tools/gpu_sweep.sh ${tag}sweep > gpurun_out/${tag}_sweep_table.txt 2>&1
cat gpurun_out/${tag}_sweep_table.txt
# summaries on the box (gpurun copies back at most 64 MiB): text summaries of every report, then the reports go
python tools/launch_summary.py gpurun_out/${tag}_launches.csv > gpurun_out/${tag}_launches_summary.txt 2>&1
for r in gpurun_out/${tag}_prof*.ncu-rep; do echo "# $r"; python tools/ncu_summary.py $r; done > gpurun_out/${tag}_ncu_summary.txt 2>&1
ncu -i gpurun_out/${tag}_prof.ncu-rep --page source --csv --print-source sass > gpurun_out/${tag}_ncu_source_cfg5.csv 2>/dev/null
gzip -f gpurun_out/${tag}_ncu_source_cfg5.csv
rm -f gpurun_out/${tag}_prof*.ncu-rep
