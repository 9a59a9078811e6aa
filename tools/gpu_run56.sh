# final verification of the session's last build: full -m gpu suite, smoke, default bench line
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/r56_pytest_gpu.txt 2>&1; tail -1 gpurun_out/r56_pytest_gpu.txt
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
python bench.py > gpurun_out/r56_bench.json 2> gpurun_out/r56_bench.err
python -c "import json; d=json.load(open('gpurun_out/r56_bench.json')); print(round(d['value']), 'e2e', round(d['e2e']['value']), 'frac', round(d['roofline']['frac'],3), d['clocks'])"
