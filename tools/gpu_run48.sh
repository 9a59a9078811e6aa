# re-entry verification of the restored build: smoke, -m gpu suite, default bench line
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r48_smoke.txt 2>&1; tail -1 gpurun_out/r48_smoke.txt
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r48_pytest_gpu.txt 2>&1; tail -3 gpurun_out/r48_pytest_gpu.txt
python bench.py > gpurun_out/r48_bench.json 2> gpurun_out/r48_bench.err; head -c 400 gpurun_out/r48_bench.json
