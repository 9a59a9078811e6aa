"""Fusion ablation schedules (lbm_set_schedule) and checkpoint / resume
(lbm_checkpoint_*), SURVEY §8(f) rows 2 and 4.

The unfused schedule (stream-only S_L^k, then in-place collision) and the
graph-free launch path run the same arithmetic as the fused F_L^k graph, so
they must agree BITWISE with it; a resumed run must agree bitwise with an
uninterrupted one.  Each is also checked against the fp64 oracle once."""
import numpy as np
import pytest

import lbm_inputs as I
from tests._parity import TOL, errors, oracle_run

pytestmark = pytest.mark.gpu

FP32, FP64 = 0, 1


def _lbmr():
    from paper_conf_ipps_mahmoudsm24_b200 import lbmr
    return lbmr


def _fields(g, levels):
    return [g.macroscopic(L) for L in range(levels)]


def _same(a, b):
    for (ra, ua), (rb, ub) in zip(a, b):
        assert np.array_equal(np.isnan(ra), np.isnan(rb))
        m = ~np.isnan(ra)
        assert np.array_equal(ra[m], rb[m]) and np.array_equal(ua[m], ub[m])


PROBLEMS = {
    "cavity2r": lambda: I.cavity2("r"),
    "random4": lambda: I.random_balanced(33, n=(9, 11, 10), levels=4, p_refine=0.5),
    "kbc_mini": lambda: I.cavity4_kbc("mini"),
    "tunnel_s5": lambda: I.tunnel4(scale=5),
}


def _run(prob, prec, steps, mode):
    lbmr = _lbmr()
    g = lbmr.grid_from_problem(prob, precision=prec)
    g.set_schedule(mode)
    g.step(steps)
    out = _fields(g, prob.levels)
    g.close()
    return out


@pytest.mark.parametrize("prec", [FP64, FP32])
@pytest.mark.parametrize("name", list(PROBLEMS))
def test_schedules_bitwise_equal(name, prec):
    lbmr = _lbmr()
    prob = PROBLEMS[name]()
    steps = 3
    ref = _run(prob, prec, steps, lbmr.SCHED_FUSED)
    for mode in (lbmr.SCHED_UNFUSED, lbmr.SCHED_NO_GRAPH, lbmr.SCHED_UNFUSED | lbmr.SCHED_NO_GRAPH):
        _same(ref, _run(prob, prec, steps, mode))


def test_unfused_matches_oracle():
    lbmr = _lbmr()
    prob = I.cavity2("r")
    ora = oracle_run(prob, 10)
    for prec in (FP64, FP32):
        er, eu = errors(_run(prob, prec, 10, lbmr.SCHED_UNFUSED), ora, prec, 10, "cavity2r/unfused")
        assert er <= TOL[prec] and eu <= TOL[prec], (prec, er, eu)


def test_schedule_switch_mid_run():
    """Switching the schedule between lbm_step calls keeps the trajectory."""
    lbmr = _lbmr()
    prob = I.tunnel4(scale=5)
    ref = _run(prob, FP64, 4, lbmr.SCHED_FUSED)
    g = lbmr.grid_from_problem(prob, precision=FP64)
    for mode in (lbmr.SCHED_UNFUSED, lbmr.SCHED_FUSED, lbmr.SCHED_NO_GRAPH, lbmr.SCHED_UNFUSED):
        g.set_schedule(mode)
        g.step(1)
    _same(ref, _fields(g, prob.levels))
    g.close()


def test_bad_schedule_mode():
    lbmr = _lbmr()
    g = lbmr.grid_from_problem(I.cavity2(), precision=FP32)
    for bad in (128, -1, lbmr.SCHED_SPLIT_A | lbmr.SCHED_ATOMIC_A):
        with pytest.raises(lbmr.LBMError):
            g.set_schedule(bad)
    g.close()


@pytest.mark.parametrize("prec", [FP64, FP32])
@pytest.mark.parametrize("name", list(PROBLEMS))
@pytest.mark.parametrize("at", [0, 1, 2])
def test_checkpoint_resume_bitwise(name, prec, at):
    """save after `at` coarse steps (0: before the prologue ran), restore into
    a FRESH grid (its other buffers zero), continue: == uninterrupted run."""
    lbmr = _lbmr()
    prob = PROBLEMS[name]()
    total = 5
    ref = _run(prob, prec, total, lbmr.SCHED_FUSED)
    g = lbmr.grid_from_problem(prob, precision=prec)
    g.step(at)
    ck = g.save_checkpoint()
    assert ck.nbytes == g.checkpoint_size()
    g.close()
    h = lbmr.grid_from_problem(prob, precision=prec, init=False)
    h.load_checkpoint(ck)
    assert h.info().steps_done == at
    h.step(total - at)
    _same(ref, _fields(h, prob.levels))
    h.close()


def test_checkpoint_rejects_other_grid():
    lbmr = _lbmr()
    g = lbmr.grid_from_problem(I.cavity2(), precision=FP32)
    g.step(1)
    ck = g.save_checkpoint()
    g.close()
    for other in (lambda: lbmr.grid_from_problem(I.cavity2(), precision=FP64),
                  lambda: lbmr.grid_from_problem(I.tunnel4(scale=5), precision=FP32)):
        h = other()
        with pytest.raises(lbmr.LBMError):
            h.load_checkpoint(ck)
        h.close()
    h = lbmr.grid_from_problem(I.cavity2(), precision=FP32)
    with pytest.raises(lbmr.LBMError):
        h.load_checkpoint(ck[:-4])  # truncated
    bad = ck.copy()
    bad[:4] = 0
    with pytest.raises(lbmr.LBMError):
        h.load_checkpoint(bad)
    h.close()


def test_checkpoint_partitioned_bitwise():
    """Each slab of a 2-slab partition checkpoints its own state; resuming
    both into fresh slabs == uninterrupted single grid."""
    lbmr = _lbmr()
    prob = I.tunnel4(scale=5)
    ref = _run(prob, FP64, 4, lbmr.SCHED_FUSED)
    pg = lbmr.PartitionedGrid(prob, 2, precision=FP64)
    pg.step(2)
    pg.synchronize()
    cks = [g.save_checkpoint() for g in pg.grids]
    pg.close()
    pg2 = lbmr.PartitionedGrid(prob, 2, precision=FP64)
    for g, ck in zip(pg2.grids, cks):
        g.load_checkpoint(ck)
    pg2.step(2)
    got = [pg2.macroscopic(L) for L in range(prob.levels)]
    pg2.close()
    _same(ref, got)


def test_checkpoint_partitioned_without_global_sync():
    """lbm_checkpoint_save on one slab must itself wait for the
    neighbour's final halo stores into its buffers (no caller-side global
    synchronisation before saving).  Slabs are saved right after the steps
    are issued, slab 0 first (its neighbour's kernels may still be running)."""
    lbmr = _lbmr()
    prob = I.tunnel4(scale=5)
    ref = _run(prob, FP64, 6, lbmr.SCHED_FUSED)
    for P in (2, 4):
        pg = lbmr.PartitionedGrid(prob, P, precision=FP64)
        pg.step(3)
        cks = [g.save_checkpoint() for g in pg.grids]
        pg.close()
        pg2 = lbmr.PartitionedGrid(prob, P, precision=FP64)
        for g, ck in zip(pg2.grids, cks):
            g.load_checkpoint(ck)
        pg2.step(3)
        got = [pg2.macroscopic(L) for L in range(prob.levels)]
        pg2.close()
        _same(ref, got)


def test_device_bytes_and_launch_count_match_analyze():
    """lbm_grid_analyze predicts exactly the device bytes lbm_grid_create
    allocates and the kernels one coarse step launches."""
    lbmr = _lbmr()
    for prob in (I.tunnel4(scale=5), I.cavity4_kbc("mini"), I.cavity2()):
        for prec in (FP32, FP64):
            a = lbmr.analyze_problem(prob, precision=prec)
            g = lbmr.grid_from_problem(prob, precision=prec, init=False)
            i = g.info()
            assert i.device_bytes == a.device_bytes, (prob.name, prec, i.device_bytes, a.device_bytes)
            assert i.launches_per_step == a.launches_per_step
            g.close()
    prob = I.tunnel4(scale=5)
    pg = lbmr.PartitionedGrid(prob, 2, precision=FP32)
    for r, g in enumerate(pg.grids):
        a = lbmr.analyze(prob.nx, prob.ny, prob.nz, prob.masks, n_ranks=2, rank=r, **lbmr._problem_kw(prob, FP32))
        i = g.info()
        assert i.device_bytes >= a.device_bytes  # + the peer cell lists uploaded at connect
        # one halo wait per level kernel and per coalescence gather
        assert i.launches_per_step == a.launches_per_step
        assert i.launches_per_step > i.kernels_per_step * 2
    pg.close()


@pytest.mark.parametrize("prec", [0, 1])
def test_set_bc_mid_run_applies_from_next_step(prec):
    """lbm_set_bc is enqueued on the grid's stream (include/lbmr.h): a lid
    change after 2 coarse steps acts on steps 3.. only, i.e. equals a grid
    built with the new lid that resumes from the 2-step checkpoint."""
    import dataclasses
    lbmr = _lbmr()
    prob = I.cavity2("r")
    u2 = (0.03, 0.0, 0.01)
    prob2 = dataclasses.replace(prob, bc={**prob.bc, I.CLS_LID: (I.BC_VELOCITY, u2)})
    g = lbmr.grid_from_problem(prob, precision=prec)
    g.step(2)
    g.set_bc(I.CLS_LID, lbmr.BC_VELOCITY, u2)
    g.step(3)
    changed = _fields(g, prob.levels)
    g.close()
    h = lbmr.grid_from_problem(prob, precision=prec)
    h.step(2)
    ck = h.save_checkpoint()
    h.step(3)
    unchanged = _fields(h, prob.levels)
    h.close()
    k = lbmr.grid_from_problem(prob2, precision=prec, init=False)
    k.load_checkpoint(ck)
    k.step(3)
    _same(changed, _fields(k, prob.levels))
    k.close()
    assert not np.array_equal(np.nan_to_num(changed[0][1]), np.nan_to_num(unchanged[0][1]))


@pytest.mark.parametrize("env", [{"LBMR_NO_PDL": "1"}, {"LBMR_PREFETCH": "0"}, {"LBMR_PREFETCH": "200"},
                                 {"LBMR_NO_BLOCK_ALIGN": "1"}, {"LBMR_BLOCK_ORDER": "hilbert"}],
                         ids=["no_pdl", "no_prefetch", "far_prefetch", "no_align", "hilbert"])
def test_performance_switches_do_not_change_results(env, monkeypatch):
    """The programmatic-dependent-launch chain, the L2 prefetch distance, the
    block-grid alignment and the block order are performance choices only:
    bitwise the same fields (fp64 and fp32) with each switched."""
    for prec in (FP64, FP32):
        for name in ("tunnel_s5", "kbc_mini"):
            prob = PROBLEMS[name]()
            ref = _run(prob, prec, 3, _lbmr().SCHED_FUSED)
            with monkeypatch.context() as m:
                for k, v in env.items():
                    m.setenv(k, v)
                got = _run(prob, prec, 3, _lbmr().SCHED_FUSED)
            _same(ref, got)
