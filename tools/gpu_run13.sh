timeout 1500 python -m pytest tests/test_gpu_volumetric.py -m gpu -q -x 2>&1 | grep -E "assert|Error|passed|failed|error" | head -20
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_schedule_ckpt.py tests/test_gpu_partition.py -m gpu -q -x 2>&1 | tail -2
