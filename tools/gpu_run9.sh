timeout 1500 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -k "cavity4 or tunnel4 or uniform or probe" 2>&1 | grep -E "assert|Error|passed|failed" | head -20
