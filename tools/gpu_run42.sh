# is the two-process IPC halo test flaky in sequence with the other partition tests?
for i in 1 2 3 4; do timeout 900 python -m pytest tests/test_gpu_partition.py -m gpu -q 2>&1 | tail -1; done
for i in 1 2; do timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_partition.py -m gpu -q 2>&1 | tail -1; done
