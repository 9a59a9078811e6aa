# quarter-block CTAs for the partitioned (halo-protocol) kernels
for i in 1 2 3; do timeout 900 python -m pytest tests/test_gpu_partition.py tests/test_gpu_schedule_ckpt.py -m gpu -q 2>&1 | tail -1; done
timeout 900 python tools/ipc_stress.py 15 2>&1 | tail -2
LBMR_BENCH_SHARE_DEVICE=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 \
  bench.py --gpus 2 --steps 5 --warmup 3 --config tunnel4 > gpurun_out/r47_bench_2rank_shared.json 2> gpurun_out/r47_bench_2rank.err
python -c "import json; d=json.load(open('gpurun_out/r47_bench_2rank_shared.json')); print('2-rank shared', round(d['value']), d['config']['parallelism'])" || tail -3 gpurun_out/r47_bench_2rank.err
