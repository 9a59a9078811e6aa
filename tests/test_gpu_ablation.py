"""Fusion-ablation schedules of the paper (§IV, Fig. 4 and Fig. 9, P:L208-222,
P:L282-284) on the GPU: every combination of the C/A/S/E/O splits
(lbm_set_schedule bits) computes the same step as the fused product schedule.

* schedules without the atomic Accumulate are BITWISE equal to the product
  (the split gather kernels add in the oracle's order);
* the atomic (CA-fused) schedules differ by summation order only: within the
  parity bars of the fp64 oracle (fp64 ≤ 1e-12, fp32 ≤ 1e-5);
* every paper configuration 4b-4f is checked against the oracle directly;
* switching schedules at a coarse-step boundary keeps the trajectory
  (pending accumulations are rebuilt), and checkpoints resume under them.
"""
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


def _run(prob, prec, steps, mode):
    lbmr = _lbmr()
    g = lbmr.grid_from_problem(prob, precision=prec)
    g.set_schedule(mode)
    g.step(steps)
    out = _fields(g, prob.levels)
    g.close()
    return out


PROBLEMS = {
    "cavity2r": lambda: I.cavity2("r"),
    "random4": lambda: I.random_balanced(33, n=(9, 11, 10), levels=4, p_refine=0.5),
    "kbc_mini": lambda: I.cavity4_kbc("mini"),
    "tunnel_s5": lambda: I.tunnel4(scale=5),
}


def _all_modes(lbmr):
    bits = [lbmr.SCHED_UNFUSED, lbmr.SCHED_SPLIT_E, lbmr.SCHED_SPLIT_A, lbmr.SCHED_ATOMIC_A, lbmr.SCHED_SPLIT_O]
    modes = []
    for m in range(1 << len(bits)):
        mode = sum(b for i, b in enumerate(bits) if m >> i & 1)
        if (mode & lbmr.SCHED_SPLIT_A) and (mode & lbmr.SCHED_ATOMIC_A):
            continue
        modes.append(mode)
    return modes


@pytest.mark.parametrize("prec", [FP64, FP32])
@pytest.mark.parametrize("name", list(PROBLEMS))
def test_every_schedule_matches_the_product(name, prec):
    lbmr = _lbmr()
    prob = PROBLEMS[name]()
    steps = 4
    ref = _run(prob, prec, steps, lbmr.SCHED_FUSED)
    for mode in _all_modes(lbmr):
        got = _run(prob, prec, steps, mode)
        if mode & lbmr.SCHED_ATOMIC_A:
            er, eu = errors(got, ref)
            assert er <= TOL[prec] and eu <= TOL[prec], (mode, er, eu)
        else:
            _same(ref, got)


@pytest.mark.parametrize("prec", [FP64, FP32])
@pytest.mark.parametrize("fig", ["4b", "4c", "4d", "4e", "4f"])
def test_fig4_schedules_match_the_oracle(fig, prec):
    lbmr = _lbmr()
    for name in ("tunnel_s5", "kbc_mini"):
        prob = PROBLEMS[name]()
        steps = 10
        ora = oracle_run(prob, steps)
        er, eu = errors(_run(prob, prec, steps, lbmr.FIG4[fig]), ora, prec, steps, f"{name}/fig{fig}")
        assert er <= TOL[prec] and eu <= TOL[prec], (fig, name, er, eu)


def test_atomic_accumulate_is_a_scatter_of_the_same_sums():
    """The atomic form adds the same terms in another order: fp64 results
    agree with the gather form to rounding after several steps."""
    lbmr = _lbmr()
    prob = I.tunnel4(scale=5)
    a = _run(prob, FP64, 6, lbmr.SCHED_FUSED)
    b = _run(prob, FP64, 6, lbmr.SCHED_ATOMIC_A)
    er, eu = errors(b, a)
    assert er < 1e-14 and eu < 1e-13


def test_schedule_switch_mid_run_rebuilds_accumulations():
    lbmr = _lbmr()
    prob = I.tunnel4(scale=5)
    ref = _run(prob, FP64, 7, lbmr.SCHED_FUSED)
    g = lbmr.grid_from_problem(prob, precision=FP64)
    seq = [lbmr.FIG4["4b"], lbmr.SCHED_FUSED, lbmr.SCHED_SPLIT_A, lbmr.FIG4["4d"], lbmr.SCHED_SPLIT_O,
           lbmr.FIG4["4b"], lbmr.SCHED_FUSED]
    for mode in seq:
        g.set_schedule(mode)
        g.step(1)
    _same(ref, _fields(g, prob.levels))  # no atomics in the sequence: bitwise
    g.close()
    g = lbmr.grid_from_problem(prob, precision=FP64)
    for mode in (lbmr.FIG4["4f"], lbmr.SCHED_SPLIT_A, lbmr.FIG4["4c"], lbmr.SCHED_FUSED, lbmr.FIG4["4e"],
                 lbmr.SCHED_ATOMIC_A | lbmr.SCHED_SPLIT_O, lbmr.FIG4["4b"]):
        g.set_schedule(mode)
        g.step(1)
    er, eu = errors(_fields(g, prob.levels), ref)
    assert er < 1e-14 and eu < 1e-13, (er, eu)
    g.close()


@pytest.mark.parametrize("fig", ["4b", "4f"])
def test_checkpoint_resume_under_ablation_schedules(fig):
    """At a coarse-step boundary the accumulations in flight live in the
    coarse ghost slots of the current buffers, which the checkpoint holds."""
    lbmr = _lbmr()
    prob = I.tunnel4(scale=5)
    mode = lbmr.FIG4[fig]
    ref = _run(prob, FP64, 5, mode)
    g = lbmr.grid_from_problem(prob, precision=FP64)
    g.set_schedule(mode)
    g.step(2)
    ck = g.save_checkpoint()
    g.close()
    h = lbmr.grid_from_problem(prob, precision=FP64, init=False)
    h.set_schedule(mode)
    h.load_checkpoint(ck)
    h.step(3)
    got = _fields(h, prob.levels)
    h.close()
    if mode & lbmr.SCHED_ATOMIC_A:
        er, eu = errors(got, ref)
        assert er < 1e-14 and eu < 1e-13
    else:
        _same(ref, got)


def test_ablation_rejected_where_unsupported():
    lbmr = _lbmr()
    prob = I.tunnel4(scale=5)
    pg = lbmr.PartitionedGrid(prob, 2, precision=FP32)
    with pytest.raises(lbmr.LBMError):
        pg.grids[0].set_schedule(lbmr.SCHED_ATOMIC_A)
    pg.close()
    g = lbmr.grid_from_problem(prob, precision=FP32, variant=lbmr.VARIANT_VOLUMETRIC)
    with pytest.raises(lbmr.LBMError):
        g.set_schedule(lbmr.SCHED_SPLIT_E)
    g.set_schedule(lbmr.SCHED_UNFUSED)  # the C/S split is supported there
    g.close()
