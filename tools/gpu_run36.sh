# compute-sanitizer on the current build + the N>1 bench path (2 ranks sharing the one GPU)
out=gpurun_out/r36_compute_sanitizer.txt; : > $out
for t in memcheck racecheck synccheck initcheck; do
  echo "== $t" >> $out
  timeout 900 compute-sanitizer --tool $t python tools/sanitize.py >> $out 2>&1
done
grep -E "^==|SUMMARY" $out
LBMR_BENCH_SHARE_DEVICE=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 \
  bench.py --gpus 2 --steps 5 --warmup 3 --config tunnel4 > gpurun_out/r36_bench_2rank_shared.json 2> gpurun_out/r36_bench_2rank.err
tail -c 600 gpurun_out/r36_bench_2rank_shared.json; tail -3 gpurun_out/r36_bench_2rank.err
