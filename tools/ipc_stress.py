"""Stress the two-process CUDA-IPC halo path (tests/test_gpu_partition.py
test_two_processes_cuda_ipc_halo) and report where results differ when they do."""
import os, socket, sys
sys.path.insert(0, os.getcwd())
import numpy as np
import lbm_inputs as I
from tests.test_gpu_partition import _ipc_worker, _single
from paper_conf_ipps_mahmoudsm24_b200.lbmr import FP64


def main(n):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    prob = I.cavity2("r")
    steps = 4
    ref = _single(prob, steps, FP64)
    bad = 0
    for it in range(n):
        q = ctx.Queue()
        s = socket.socket(); s.bind(("127.0.0.1", 0)); port = s.getsockname()[1]; s.close()
        procs = [ctx.Process(target=_ipc_worker, args=(r, 2, port, steps, q)) for r in range(2)]
        for p in procs: p.start()
        res = dict(q.get(timeout=600) for _ in range(2))
        for p in procs: p.join(timeout=120)
        msg = []
        for L in range(prob.levels):
            r = np.concatenate([res[0][L][0], res[1][L][0]], axis=0)
            d = np.abs(np.nan_to_num(r) - np.nan_to_num(ref[L][0]))
            if d.max() > 0:
                idx = np.argwhere(d > 0)
                msg.append(f"L{L}: {len(idx)} cells differ (max {d.max():.3e}); x range {idx[:,0].min()}..{idx[:,0].max()}, "
                           f"rank-0 x extent {res[0][L][0].shape[0]}")
        if msg:
            bad += 1
            print(f"iter {it}: MISMATCH", "; ".join(msg), flush=True)
    print(f"{bad} of {n} runs differ", flush=True)


if __name__ == "__main__":
    main(int(sys.argv[1]) if len(sys.argv) > 1 else 20)
