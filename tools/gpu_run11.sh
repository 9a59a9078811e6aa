bash tools/profile_round.sh r01c
bash tools/gpu_sweep.sh r01sweep
