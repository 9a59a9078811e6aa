# ncu of cfg5 L1 (third launch of the second warm-up step): HEAD~ build vs current
ncu --set full --clock-control none --import-source on -k regex:level_step -s 17 -c 1 -o gpurun_out/r30_L1_new \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline --profile-steps 1 > /dev/null 2>&1
LBMR_LIB=$PWD/paper_conf_ipps_mahmoudsm24_b200/_lib/exp/base.so ncu --set full --clock-control none --import-source on -k regex:level_step -s 17 -c 1 -o gpurun_out/r30_L1_base \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline --profile-steps 1 > /dev/null 2>&1
ls gpurun_out/r30*
