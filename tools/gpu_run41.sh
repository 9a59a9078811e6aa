# two-process CUDA IPC halo test: current build x3, HEAD build (base.so = c84ebf1-era? no: 7910dbb) x2
for i in 1 2 3; do timeout 600 python -m pytest tests/test_gpu_partition.py -m gpu -q -k two_processes 2>&1 | tail -1; done
for i in 1 2; do LBMR_LIB=$PWD/paper_conf_ipps_mahmoudsm24_b200/_lib/exp/base.so timeout 600 python -m pytest tests/test_gpu_partition.py -m gpu -q -k two_processes 2>&1 | tail -1; done
