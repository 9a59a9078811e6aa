# Full measurement pass for the current build: bench line, launch list, ncu full capture.
# usage (under gpurun): bash tools/profile_round.sh <tag>
tag=${1:-r01}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem --format=csv > gpurun_out/${tag}_gpu.txt
python bench.py > gpurun_out/${tag}_bench.json 2> gpurun_out/${tag}_bench.err
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"level_step|level_collide|macroscopic|init_eq" -c 200 --csv --log-file gpurun_out/${tag}_launches.csv \
    python bench.py --steps 3 --warmup 3 --no-cpu-baseline --profile-steps 1 > /dev/null 2>&1
# dominant kernel (finest level, first launch of step 2) and the next two (L2, L1)
ncu --set full --clock-control none --import-source on -k regex:level_step -s 15 -c 3 -o gpurun_out/${tag}_prof \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline --profile-steps 1 > gpurun_out/${tag}_ncu.log 2>&1
tail -1 gpurun_out/${tag}_ncu.log
