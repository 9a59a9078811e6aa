# after moving every setup upload onto the grid's stream
timeout 600 python tools/ipc_diag.py 60 0 2>&1 | tail -4
(timeout 700 python bench.py --config uniform512 --steps 8000 --warmup 3 --no-cpu-baseline > /dev/null 2>&1 &)
sleep 15
timeout 600 python tools/ipc_diag.py 40 0 2>&1 | tail -4
sleep 5
timeout 900 python -m pytest tests -m gpu -q 2>&1 | tail -2
