"""Diagnose rare two-process CUDA-IPC mismatches: per-step snapshots of both ranks,
first differing step, and the (x, y, z) extent of the differing cells."""
import os, socket, sys
sys.path.insert(0, os.getcwd())
import numpy as np
import lbm_inputs as I
from paper_conf_ipps_mahmoudsm24_b200.lbmr import FP64


def worker(rank, world, port, steps, q, per_step):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    import torch
    import torch.distributed as dist
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_ipps_mahmoudsm24_b200 import lbmr
    torch.cuda.set_device(0)
    prob = I.cavity2("r")
    s = torch.cuda.Stream()
    g = lbmr.grid_from_problem(prob, FP64, stream=s.cuda_stream, n_ranks=world, rank=rank)
    blobs = {side: (g.halo_export(side) if lbmr.g_has(g, side) else None) for side in (0, 1)}
    allb = [None] * world
    dist.all_gather_object(allb, blobs)
    for side in (0, 1):
        if lbmr.g_has(g, side):
            g.halo_connect(side, allb[(rank + (1 if side else -1)) % world][1 - side])
    dist.barrier()
    snaps = []
    if per_step:
        for _ in range(steps):
            g.step(1)
            snaps.append([g.macroscopic(L)[0] for L in range(prob.levels)])
    else:
        g.step(steps)
        g.synchronize()
        snaps.append([g.macroscopic(L)[0] for L in range(prob.levels)])
    q.put((rank, snaps))
    dist.barrier()
    g.close()
    dist.destroy_process_group()


def main(n, per_step):
    import torch.multiprocessing as mp
    from paper_conf_ipps_mahmoudsm24_b200 import lbmr
    ctx = mp.get_context("spawn")
    prob = I.cavity2("r")
    steps = 4
    ref = []
    g = lbmr.grid_from_problem(prob, precision=FP64)
    for _ in range(steps):
        g.step(1)
        ref.append([g.macroscopic(L)[0] for L in range(prob.levels)])
    g.close()
    bad = 0
    for it in range(n):
        q = ctx.Queue()
        s = socket.socket(); s.bind(("127.0.0.1", 0)); port = s.getsockname()[1]; s.close()
        procs = [ctx.Process(target=worker, args=(r, 2, port, steps, q, per_step)) for r in range(2)]
        for p in procs: p.start()
        res = dict(q.get(timeout=600) for _ in range(2))
        for p in procs: p.join(timeout=120)
        msgs = []
        for si in range(len(res[0])):
            st = si if per_step else steps - 1
            for L in range(prob.levels):
                r = np.concatenate([res[0][si][L], res[1][si][L]], axis=0)
                d = np.abs(np.nan_to_num(r) - np.nan_to_num(ref[st][L]))
                if d.max() > 0:
                    idx = np.argwhere(d > 0)
                    lo, hi = idx.min(0), idx.max(0)
                    per_x = np.bincount(idx[:, 0], minlength=r.shape[0])
                    stale = [k for k in range(steps) if k != st and np.array_equal(
                        np.nan_to_num(r)[d > 0], np.nan_to_num(ref[k][L])[d > 0])]
                    msgs.append(f"step {st+1} L{L}: {len(idx)} cells (max {d.max():.3e}) box {lo.tolist()}..{hi.tolist()} "
                                f"per-x {dict((int(i), int(c)) for i, c in enumerate(per_x) if c)} equal-to-ref-steps {[k+1 for k in stale]}")
            if msgs:
                break
        if msgs:
            bad += 1
            print(f"iter {it}:", " | ".join(msgs), flush=True)
    print(f"{bad} of {n} runs differ (per_step={per_step})", flush=True)


if __name__ == "__main__":
    main(int(sys.argv[1]), int(sys.argv[2]))
