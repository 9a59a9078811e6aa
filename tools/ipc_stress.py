"""Stress the multi-process CUDA-IPC halo path (tests/test_gpu_partition.py
test_processes_cuda_ipc_halo): run `world` processes on one GPU `n` times and
report where results differ from one grid when they do.

  python tools/ipc_stress.py [n=20] [world=2] [problem=cavity2|tunnel4_s5] [steps=4]
"""
import os
import socket
import sys

sys.path.insert(0, os.getcwd())
import numpy as np  # noqa: E402

from tests.test_gpu_partition import IPC_PROBLEMS, _ipc_worker, _single  # noqa: E402
from paper_conf_ipps_mahmoudsm24_b200.lbmr import FP64  # noqa: E402


def main(n, world, pname, steps):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    prob = IPC_PROBLEMS[pname]()
    ref = _single(prob, steps, FP64)
    bad = 0
    for it in range(n):
        q = ctx.Queue()
        s = socket.socket()
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
        s.close()
        procs = [ctx.Process(target=_ipc_worker, args=(r, world, port, steps, q, pname)) for r in range(world)]
        for p in procs:
            p.start()
        res = dict(q.get(timeout=900) for _ in range(world))
        for p in procs:
            p.join(timeout=120)
        errs = [k for k in range(world) if isinstance(res[k], str)]
        if errs:
            bad += 1
            print(f"iter {it}: rank error {res[errs[0]]}", flush=True)
            continue
        msg = []
        for L in range(prob.levels):
            r = np.concatenate([res[k][L][0] for k in range(world)], axis=0)
            d = np.abs(np.nan_to_num(r) - np.nan_to_num(ref[L][0]))
            if d.max() > 0:
                idx = np.argwhere(d > 0)
                msg.append(f"L{L}: {len(idx)} cells differ (max {d.max():.3e}); x range {idx[:, 0].min()}..{idx[:, 0].max()}")
        if msg:
            bad += 1
            print(f"iter {it}: MISMATCH", "; ".join(msg), flush=True)
    print(f"{pname} world={world} steps={steps}: {bad} of {n} runs differ", flush=True)


if __name__ == "__main__":
    a = sys.argv[1:]
    main(int(a[0]) if len(a) > 0 else 20, int(a[1]) if len(a) > 1 else 2, a[2] if len(a) > 2 else "cavity2",
         int(a[3]) if len(a) > 3 else 4)
