# N=2 bench path (two ranks sharing the one GPU) after the setup/connect ordering change
LBMR_BENCH_SHARE_DEVICE=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 \
  bench.py --gpus 2 --steps 5 --warmup 3 --config tunnel4 > gpurun_out/r54_bench_2rank_shared.json 2> gpurun_out/r54_bench_2rank.err
python -c "import json; d=json.load(open('gpurun_out/r54_bench_2rank_shared.json')); print('2-rank shared', round(d['value']), d['config']['parallelism'], d.get('scaling'))" || tail -5 gpurun_out/r54_bench_2rank.err
