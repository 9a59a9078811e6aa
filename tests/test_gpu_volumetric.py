"""CUDA path of the VOLUMETRIC variant
vs the oracle's volumetric mode, element by element; and the property the
variant exists for — exact mass on interface edges and corners — on the GPU.
Bars as everywhere: fp64 <= 1e-12, fp32 <= 1e-5."""
import numpy as np
import pytest

import lbm_inputs as I
import oracle
from tests._parity import TOL, errors
from tests.test_oracle_volumetric import CORNERS, _randomise, _walled_box

pytestmark = pytest.mark.gpu

FP32, FP64 = 0, 1


def _lbmr():
    from paper_conf_ipps_mahmoudsm24_b200 import lbmr
    return lbmr


def _oracle_vol(prob, steps):
    o = oracle.Oracle(prob)
    o.set_variant("volumetric")
    o.step(steps)
    return [o.macroscopic(L) for L in range(prob.levels)]


def _gpu_vol(prob, prec, steps, schedule=0):
    lbmr = _lbmr()
    g = lbmr.grid_from_problem(prob, precision=prec, variant=lbmr.VARIANT_VOLUMETRIC)
    g.set_schedule(schedule)
    g.step(steps)
    out = [g.macroscopic(L) for L in range(prob.levels)]
    g.close()
    return out


def _walled(case):
    p = _walled_box(None if case == "coarse_interface_wall" else case)
    if case == "coarse_interface_wall":
        p.masks[0][1, 3, 3] = 2
    return p


PROBS = {f"corner{k}": (lambda k=k: _randomise(CORNERS[k](), 2 + k)) for k in range(len(CORNERS))}
PROBS.update({c: (lambda c=c: _randomise(_walled(c), 5)) for c in
              ("coarse_bc_leaf", "fine_bc_leaf_inside", "fine_bc_leaf_at_interface", "x_walls",
               "coarse_interface_wall")})
PROBS.update({"cavity2r": lambda: I.cavity2("r"), "sphere3_s4": lambda: I.sphere3(scale=4),
              "tunnel4_s5": lambda: I.tunnel4(scale=5)})
STEPS = {"tunnel4_s5": 2, "sphere3_s4": 3}

_cache = {}


@pytest.mark.parametrize("prec", [FP64, FP32])
@pytest.mark.parametrize("name", list(PROBS))
def test_volumetric_matches_oracle(name, prec):
    prob = PROBS[name]()
    steps = STEPS.get(name, 5)
    if name not in _cache:
        _cache[name] = _oracle_vol(prob, steps)
    er, eu = errors(_gpu_vol(prob, prec, steps), _cache[name], prec, steps, name + "/volumetric")
    assert er <= TOL[prec] and eu <= TOL[prec], (name, prec, er, eu)


@pytest.mark.parametrize("k", [0, 1, 3])
def test_volumetric_gpu_mass_exact_on_corners(k):
    lbmr = _lbmr()
    p = _randomise(CORNERS[k](), 20 + k)
    g = lbmr.grid_from_problem(p, precision=FP64, variant=lbmr.VARIANT_VOLUMETRIC)
    _, m0 = g.stats()
    g.step(20)
    _, m1 = g.stats()
    g.close()
    assert abs(m1 - m0) / m0 < 1e-13


def test_volumetric_schedules_and_resume_bitwise():
    lbmr = _lbmr()
    p = _randomise(CORNERS[3](), 8)
    ref = _gpu_vol(p, FP64, 4)
    for mode in (lbmr.SCHED_UNFUSED, lbmr.SCHED_NO_GRAPH):
        got = _gpu_vol(p, FP64, 4, schedule=mode)
        for (ra, ua), (rb, ub) in zip(ref, got):
            m = ~np.isnan(ra)
            assert np.array_equal(ra[m], rb[m]) and np.array_equal(ua[m], ub[m])
    g = lbmr.grid_from_problem(p, precision=FP64, variant=lbmr.VARIANT_VOLUMETRIC)
    g.step(1)
    ck = g.save_checkpoint()
    g.close()
    h = lbmr.grid_from_problem(p, precision=FP64, init=False, variant=lbmr.VARIANT_VOLUMETRIC)
    h.load_checkpoint(ck)
    h.step(3)
    got = [h.macroscopic(L) for L in range(p.levels)]
    h.close()
    for (ra, ua), (rb, ub) in zip(ref, got):
        m = ~np.isnan(ra)
        assert np.array_equal(ra[m], rb[m]) and np.array_equal(ua[m], ub[m])


def test_volumetric_rejects_partitions():
    lbmr = _lbmr()
    with pytest.raises(lbmr.LBMError):
        lbmr.grid_from_problem(I.cavity2(), n_ranks=2, rank=0, variant=lbmr.VARIANT_VOLUMETRIC)
