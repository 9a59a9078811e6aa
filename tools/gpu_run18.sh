# Re-verify the restored build: gpu tests, smoke, bench line, launch list, ncu full of level_step.
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem --format=csv
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r18_pytest.log 2>&1; tail -3 gpurun_out/r18_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
bash tools/profile_round.sh r01b
