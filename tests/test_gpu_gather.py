"""The coalescence gather (Eq.11, readings R-A2/R-A3: A + A + O of the
two fine substeps) in its three forms, all adding the same terms in the
oracle's order and therefore BITWISE equal:

* the product: a gather kernel before F_L^k, one thread per (ghost, q)
  entry, F_L^k its programmatic dependent;
* a warp-cooperative gather kernel (LBMR_GATHER_WARP=1: four lanes per 4-slot
  unit, the values added by warp shuffles; |B| > 4 links span two units);
* LBM_SCHED_CTA_GATHER: inside F_L^k, each CTA gathers its own cells' links
  (no gather kernel).

Checked on problems with |B| > 4 links (concave interface edges), D3Q27 KBC,
fp32 and fp64, periodic wraps and partitioned grids (cut-plane cells gather
L+1 halo cells); the product also against the fp64 oracle directly.
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


def _same(a, b):
    for (ra, ua), (rb, ub) in zip(a, b):
        assert np.array_equal(np.isnan(ra), np.isnan(rb))
        m = ~np.isnan(ra)
        assert np.array_equal(ra[m], rb[m]) and np.array_equal(ua[m], ub[m])


def _run(prob, prec, steps, mode=0):
    lbmr = _lbmr()
    g = lbmr.grid_from_problem(prob, precision=prec)
    g.set_schedule(mode)
    g.step(steps)
    out = [g.macroscopic(L) for L in range(prob.levels)]
    info = g.info()
    g.close()
    return out, info


PROBLEMS = {
    "cavity2r": lambda: I.cavity2("r"),
    # random refinement: |B| > 4 links on 2 levels (coal_wide > 0)
    "random4": lambda: I.random_balanced(33, n=(9, 11, 10), levels=4, p_refine=0.5),
    "random_px": lambda: I.random_balanced(41, n=(12, 6, 6), levels=3, p_refine=0.6, periodic=(1, 0, 1)),
    "random_b": lambda: I.random_balanced(7, n=(10, 10, 10), levels=3, p_refine=0.5),
    # D3Q27 KBC with thin refined wall shells: wide links on every coarse level
    "kbc_mini": lambda: I.cavity4_kbc("mini"),
    "tunnel_s5": lambda: I.tunnel4(scale=5),
    "tab1_s1": lambda: I.sphere_tab1(1),
}


@pytest.mark.parametrize("prec", [FP64, FP32])
@pytest.mark.parametrize("name", list(PROBLEMS))
def test_gather_forms_bitwise_equal(name, prec, monkeypatch):
    lbmr = _lbmr()
    prob = PROBLEMS[name]()
    steps = 3 if name == "tab1_s1" else 6
    got, gi = _run(prob, prec, steps)  # product: thread-per-entry gather kernel
    cta, ci = _run(prob, prec, steps, lbmr.SCHED_CTA_GATHER)
    _same(got, cta)
    monkeypatch.setenv("LBMR_GATHER_WARP", "1")
    warp, _ = _run(prob, prec, steps)
    _same(got, warp)
    # CTA_GATHER launches no gather kernel
    ncoal = sum(1 << L for L in range(prob.levels) if gi.coal_links[L] > 0)
    assert gi.launches_per_step - ci.launches_per_step == ncoal
    assert ci.launches_per_step == (1 << prob.levels) - 1


def test_wide_links_are_exercised():
    lbmr = _lbmr()
    for name in ("random4", "random_px", "kbc_mini"):
        info = lbmr.analyze_problem(PROBLEMS[name]())
        assert sum(info.coal_wide) > 0, name


@pytest.mark.parametrize("prec", [FP64, FP32])
@pytest.mark.parametrize("name", ["random4", "kbc_mini"])
def test_product_gather_equals_oracle(name, prec):
    prob = PROBLEMS[name]()
    steps = 10
    got, _ = _run(prob, prec, steps)
    ref = oracle_run(prob, steps)
    er, eu = errors(got, ref)
    assert er <= TOL[prec] and eu <= TOL[prec], (er, eu)


@pytest.mark.parametrize("P", [2, 3])
@pytest.mark.parametrize("name", ["random_px", "kbc_mini", "tunnel_s5"])
def test_partitioned_warp_gather_equals_thread_gather(name, P, monkeypatch):
    lbmr = _lbmr()
    prob = PROBLEMS[name]()
    steps = 5

    def run():
        pg = lbmr.PartitionedGrid(prob, P, precision=FP64)
        pg.step(steps)
        out = [pg.macroscopic(L) for L in range(prob.levels)]
        pg.close()
        return out

    a = run()
    monkeypatch.setenv("LBMR_GATHER_WARP", "1")
    _same(a, run())


@pytest.mark.parametrize("name", ["cavity2r", "random4", "tunnel_s5"])
def test_multi_step_graphs_bitwise(name, monkeypatch):
    """lbm_step(n) replays graphs of several coarse steps when n allows
    (LBMR_GRAPH_STEPS, default 4) and single-step graphs for the rest: any
    chunking equals one-step graphs bitwise."""
    lbmr = _lbmr()
    prob = PROBLEMS[name]()
    monkeypatch.setenv("LBMR_GRAPH_STEPS", "1")
    ref, _ = _run(prob, FP64, 11)
    for gs, chunks in (("4", (11,)), ("4", (3, 5, 1, 2)), ("3", (7, 4)), ("2", (1, 10))):
        monkeypatch.setenv("LBMR_GRAPH_STEPS", gs)
        g = lbmr.grid_from_problem(prob, precision=FP64)
        for c in chunks:
            g.step(c)
        got = [g.macroscopic(L) for L in range(prob.levels)]
        g.close()
        _same(got, ref)
