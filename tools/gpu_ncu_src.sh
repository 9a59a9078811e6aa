# usage: bash tools/gpu_ncu_src.sh <tag> <skip> <count> [bench args]: full set + source counters
tag=$1; skip=$2; cnt=$3; shift 3
ncu --set full --import-source on --clock-control none -k regex:level_step -s $skip -c $cnt -o gpurun_out/prof_$tag python bench.py --steps 2 --warmup 3 --no-cpu-baseline --profile-steps 1 "$@" > gpurun_out/ncu_$tag.log 2>&1
tail -1 gpurun_out/ncu_$tag.log
