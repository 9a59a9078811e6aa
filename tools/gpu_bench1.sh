set -x
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm --format=csv
python bench.py > gpurun_out/bench1.json 2> gpurun_out/bench1.err
tail -3 gpurun_out/bench1.err
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:lbmr -c 120 --csv --log-file gpurun_out/launches1.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --profile-steps 2 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:level_step_kernel -s 19 -c 3 -o gpurun_out/prof1 python bench.py --steps 2 --warmup 3 --no-cpu-baseline --profile-steps 1 > gpurun_out/ncu1.log 2>&1
tail -3 gpurun_out/ncu1.log
