# lbm_set_bc as a by-value kernel update: full -m gpu suite, smoke, IPC stress, bench
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/r57_pytest_gpu.txt 2>&1; tail -1 gpurun_out/r57_pytest_gpu.txt
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 600 python tools/ipc_diag.py 30 0 2>&1 | tail -2
python bench.py > gpurun_out/r57_bench.json 2> gpurun_out/r57_bench.err
python -c "import json; d=json.load(open('gpurun_out/r57_bench.json')); print(round(d['value']), 'e2e', round(d['e2e']['value']), 'frac', round(d['roofline']['frac'],3), d['clocks'])"
