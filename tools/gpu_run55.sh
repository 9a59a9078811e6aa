# probe without the pre-upload stream wait: probe/fullsize tests, then two bench lines (e2e)
timeout 900 python -m pytest tests/test_gpu_fullsize.py tests/test_gpu_schedule_ckpt.py tests/test_gpu_edge.py -m gpu -q 2>&1 | tail -1
for r in 1 2; do python bench.py --no-cpu-baseline > gpurun_out/r55_bench_$r.json 2>/dev/null
python -c "import json; d=json.load(open('gpurun_out/r55_bench_$r.json')); print(round(d['value']), 'e2e', round(d['e2e']['value']), d['clocks']['sm_mhz'])"; done
