# KBC deep-dive: ncu full (source counters) of the finest-level kernel of cfg4 KBC fp32 and Tab. I s3 fp64
ncu --set full --clock-control none --import-source on -k regex:level_step -s 15 -c 1 -o gpurun_out/r20_kbc4 \
    python bench.py --config cavity4_kbc --steps 2 --warmup 3 --no-cpu-baseline --profile-steps 1 > gpurun_out/r20_kbc4.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:level_step -s 7 -c 1 -o gpurun_out/r20_tab3 \
    python bench.py --config sphere_tab1_s3 --steps 2 --warmup 3 --no-cpu-baseline --profile-steps 1 > gpurun_out/r20_tab3.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:level_step -s 15 -c 1 -o gpurun_out/r20_bgk4 \
    python bench.py --config cavity4_bgk --steps 2 --warmup 3 --no-cpu-baseline --profile-steps 1 > gpurun_out/r20_bgk4.log 2>&1
tail -2 gpurun_out/r20_*.log
