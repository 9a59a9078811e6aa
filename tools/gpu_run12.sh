timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
timeout 600 python bench.py > gpurun_out/r01d_bench.json 2> gpurun_out/r01d_bench.err; tail -1 gpurun_out/r01d_bench.json | cut -c1-400
python -c "
import json; d=json.loads(open('gpurun_out/r01d_bench.json').read().strip().splitlines()[-1]); print(d['value'], d['e2e'], d['cpu_baseline'], d['roofline']['frac'], d['gpu_launches'])"
LBMR_BENCH_SHARE_DEVICE=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --steps 5 --warmup 3 > gpurun_out/r01d_bench_n2share.json 2> gpurun_out/r01d_bench_n2share.err; tail -1 gpurun_out/r01d_bench_n2share.json | cut -c1-300
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 | cut -c1-300
