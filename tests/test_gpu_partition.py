"""Multi-GPU x-slab path on one device (T13): P partitions == one grid, bitwise
in fp64 (the gather coalescence is deterministic and a halo cell is a copy).

* in one process: P slab grids on P streams, halos connected directly
  (`lbm_halo_connect_local`), the device-side flag protocol orders them;
* in two processes sharing the GPU: halos connected through CUDA IPC
  (`lbm_halo_export` / `lbm_halo_connect`), exactly the multi-GPU transport.
"""
import os
import socket

import numpy as np
import pytest

import lbm_inputs as I

pytestmark = pytest.mark.gpu

FP32, FP64 = 0, 1


def _single(prob, steps, prec):
    from paper_conf_ipps_mahmoudsm24_b200 import lbmr
    g = lbmr.grid_from_problem(prob, precision=prec)
    g.step(steps)
    out = [g.macroscopic(L) for L in range(prob.levels)]
    g.close()
    return out


CASES = [
    ("tunnel4_s5", lambda: I.tunnel4(scale=5), 3, 4),
    ("tunnel4_s5", lambda: I.tunnel4(scale=5), 2, 4),
    ("cavity2", lambda: I.cavity2("r"), 2, 10),
    ("cavity2", lambda: I.cavity2("r"), 4, 6),
    ("slab_periodic", lambda: I.planar_slab(levels=3, n=(16, 8, 8)), 2, 6),
    ("slab_periodic", lambda: I.planar_slab(levels=3, n=(16, 8, 8)), 3, 6),
    ("random_px", lambda: I.random_balanced(41, n=(12, 6, 6), levels=3, p_refine=0.6, periodic=(1, 0, 1)), 3, 5),
    ("kbc_mini", lambda: I.cavity4_kbc("mini"), 2, 3),
]


@pytest.mark.parametrize("name,mk,P,steps", CASES, ids=[f"{c[0]}-P{c[2]}" for c in CASES])
def test_partitioned_equals_single_grid(name, mk, P, steps):
    from paper_conf_ipps_mahmoudsm24_b200 import lbmr
    prob = mk()
    ref = _single(prob, steps, FP64)
    pg = lbmr.PartitionedGrid(prob, P, precision=FP64)
    pg.step(steps)
    for L in range(prob.levels):
        r, u = pg.macroscopic(L)
        assert np.array_equal(np.isnan(r), np.isnan(ref[L][0])), (name, L)
        m = ~np.isnan(r)
        assert np.array_equal(r[m], ref[L][0][m]), (name, L, np.abs(r[m] - ref[L][0][m]).max())
        assert np.array_equal(u[m], ref[L][1][m]), (name, L)
    pg.close()


def test_partitioned_fp32_and_chunked_steps():
    from paper_conf_ipps_mahmoudsm24_b200 import lbmr
    prob = I.tunnel4(scale=5)
    ref = _single(prob, 5, FP32)
    pg = lbmr.PartitionedGrid(prob, 3, precision=FP32)
    for n in (1, 3, 1):
        pg.step(n)
    for L in range(prob.levels):
        r, u = pg.macroscopic(L)
        m = ~np.isnan(r)
        assert np.array_equal(r[m], ref[L][0][m]) and np.array_equal(u[m], ref[L][1][m])
    pg.close()


def _ipc_worker(rank, world, port, steps, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    import torch
    import torch.distributed as dist
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_ipps_mahmoudsm24_b200 import lbmr
        torch.cuda.set_device(0)
        prob = I.cavity2("r")
        s = torch.cuda.Stream()
        g = lbmr.grid_from_problem(prob, FP64, stream=s.cuda_stream, n_ranks=world, rank=rank)
        blobs = {}
        for side in (0, 1):
            blobs[side] = g.halo_export(side) if lbmr.g_has(g, side) else None
        allb = [None] * world
        dist.all_gather_object(allb, blobs)
        for side in (0, 1):
            if lbmr.g_has(g, side):
                nb = (rank + (1 if side else -1)) % world
                g.halo_connect(side, allb[nb][1 - side])
        dist.barrier()
        g.step(steps)
        g.synchronize()
        out = [g.macroscopic(L) for L in range(prob.levels)]
        q.put((rank, out))
        dist.barrier()
        g.close()
    except Exception as e:  # pragma: no cover
        q.put((rank, repr(e)))
    finally:
        dist.destroy_process_group()


def test_two_processes_cuda_ipc_halo():
    """Two processes on the same GPU, halos written into the neighbour's
    buffers through CUDA IPC + the device flag protocol (the 8xB200 path)."""
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    steps = 4
    procs = [ctx.Process(target=_ipc_worker, args=(r, 2, port, steps, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=600) for _ in range(2))
    for p in procs:
        p.join(timeout=120)
    for r in range(2):
        assert not isinstance(res[r], str), res[r]
    prob = I.cavity2("r")
    ref = _single(prob, steps, FP64)
    for L in range(prob.levels):
        r = np.concatenate([res[0][L][0], res[1][L][0]], axis=0)
        m = ~np.isnan(r)
        assert np.array_equal(m, ~np.isnan(ref[L][0]))
        assert np.array_equal(r[m], ref[L][0][m])
