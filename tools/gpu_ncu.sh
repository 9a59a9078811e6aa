# usage: bash tools/gpu_ncu.sh <tag> [extra bench args]
tag=$1; shift
ncu --set full --clock-control none --import-source on -k regex:level_step -s 15 -c 4 -o gpurun_out/prof_$tag python bench.py --steps 2 --warmup 3 --no-cpu-baseline --profile-steps 1 "$@" > gpurun_out/ncu_$tag.log 2>&1
tail -2 gpurun_out/ncu_$tag.log
