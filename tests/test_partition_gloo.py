"""Host-side logic of the multi-GPU x-slab partition, run as real multi-process
groups (torch.distributed, gloo backend, CPU only): every rank builds its own
slab from the same masks; the ranks exchange their halo plans and check that
what one rank sends across a cut is exactly what its neighbour expects in its
halo, cell by cell and in the same order, and that the owned slabs tile the
domain (leaves add up to the single-rank counts)."""
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

import lbm_inputs as I
from paper_conf_ipps_mahmoudsm24_b200 import lbmr

PROBLEMS = {
    "tunnel4_s5": lambda: I.tunnel4(scale=5),
    "cavity2": lambda: I.cavity2(),
    "slab_periodic": lambda: I.planar_slab(levels=3, n=(16, 8, 8)),
    "random": lambda: I.random_balanced(41, n=(12, 6, 6), levels=3, p_refine=0.6, periodic=(1, 0, 1)),
}


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, name, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        prob = PROBLEMS[name]()
        cuts = lbmr.partition_cuts(prob, world)
        allcuts = [None] * world
        dist.all_gather_object(allcuts, cuts)
        assert all(c == cuts for c in allcuts), "ranks disagree on the cuts"
        gi = lbmr.analyze(prob.nx, prob.ny, prob.nz, prob.masks, n_ranks=world, rank=rank,
                          **lbmr._problem_kw(prob))
        leaves = [int(gi.leaves[L]) for L in range(prob.levels)]
        plans = {}
        for side in (0, 1):
            for L in range(prob.levels):
                try:
                    send, halo = lbmr.halo_plan(prob, world, rank, side, L)
                except lbmr.LBMError:
                    send = halo = None  # no neighbour on this side
                plans[(side, L)] = (send, halo)
        gathered = [None] * world
        dist.all_gather_object(gathered, (leaves, plans))
        if rank == 0:
            per = prob.periodic[0]
            for r in range(world):
                for side in (0, 1):
                    nb = r + (1 if side == 1 else -1)
                    if not per and (nb < 0 or nb >= world):
                        for L in range(prob.levels):  # a domain face: nothing crosses it
                            send, halo = gathered[r][1][(side, L)]
                            assert send is None or (len(send) == 0 and len(halo) == 0)
                        continue
                    nb %= world
                    for L in range(prob.levels):
                        send, halo = gathered[r][1][(side, L)]
                        nsend, nhalo = gathered[nb][1][(1 - side, L)]
                        assert np.array_equal(send, nhalo), (r, side, L)
                        assert np.array_equal(halo, nsend), (r, side, L)
                        # the sent layer is the first owned layer at the cut
                        x_cut = cuts[r + 1] if side == 1 else cuts[r]
                        if len(send):
                            want = ((x_cut << L) - (1 if side == 1 else 0)) % (prob.nx << L)
                            assert np.all(send[:, 0] == want)
            total = np.sum([g[0] for g in gathered], axis=0)
            single = lbmr.analyze_problem(prob)
            assert list(total) == [int(single.leaves[L]) for L in range(prob.levels)]
        q.put((rank, "ok"))
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put((rank, repr(e)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("name,world", [("tunnel4_s5", 2), ("tunnel4_s5", 3), ("cavity2", 2),
                                        ("slab_periodic", 2), ("slab_periodic", 3), ("random", 2)])
def test_partition_plans_agree_across_ranks(name, world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, name, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    assert all(v == "ok" for v in res.values()), res
