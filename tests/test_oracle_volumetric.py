"""Pins of the oracle's VOLUMETRIC variant (the baseline
algorithm's fine-ghost advection, exact mass conservation on any interface;
DESIGN.md §16).  CPU only; none of these call the CUDA path.

V1 pure-transport worked examples (tests/golden/transport_volumetric.json):
   diagonal packets are translated exactly (they differ from the paper
   variant's T6 table);
V2 exact mass (and, periodic without walls, momentum) conservation on grids
   with interface edges and corners, 2-4 levels, D3Q19/D3Q27, BGK/KBC, with
   no-slip BC leaves — where the paper variant drifts (T8b);
V3 uniform-equilibrium invariance in any geometry;
V4 reductions: one level == the paper variant (no interface); all-refined
   2-level == textbook uniform fine LBM at omega_1 (T5)."""
import json
import os

import numpy as np
import pytest

import lbm_inputs as I
import oracle
from tests.test_oracle_pins import textbook_lbm

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _vol(p, **kw):
    o = oracle.Oracle(p, **kw)
    o.set_variant("volumetric")
    return o


def _totals(o, p):
    mass, mom = 0.0, np.zeros(3)
    for L in range(p.levels):
        r, u = o.macroscopic(L)
        m = ~np.isnan(r)
        V = 8.0 ** -L
        mass += r[m].sum() * V
        mom += (r[m][:, None] * u[m]).sum(0) * V
    return mass, mom


def _randomise(p, seed):
    rng = np.random.default_rng(seed)
    p.init_rho = [1 + 0.01 * rng.uniform(-1, 1, p.level_shape(L)) for L in range(p.levels)]
    p.init_u = [0.03 * rng.uniform(-1, 1, p.level_shape(L) + (3,)) for L in range(p.levels)]
    return p


def test_V1_pure_transport_worked_examples():
    spec = json.load(open(os.path.join(GOLDEN, "transport_volumetric.json")))
    e, w, _ = oracle.lattice(19)
    for case in spec["cases"]:
        n = tuple(spec["coarse"])
        masks = [np.ones(n, dtype=np.uint8), np.zeros((2 * n[0], 2 * n[1], 2 * n[2]), dtype=np.uint8)]
        x0, x1 = spec["refined_coarse_x"]
        masks[0][x0:x1] = 0
        masks[1][2 * x0:2 * x1] = 1
        p = I.Problem(name="v1", nx=n[0], ny=n[1], nz=n[2], masks=masks, periodic=(1, 1, 1), Q=19, omega0=0.0)
        o = _vol(p, init=False)
        i = next(k for k in range(19) if list(e[k]) == case["direction"])
        for L in range(2):
            f = np.zeros(p.level_shape(L) + (19,)) + w
            for c in case["start"].get(str(L), []):
                f[tuple(c) + (i,)] += 1.0
            o.set_f(L, f)
        o.step(1)
        for L in range(2):
            f = o.get_f(L) - w
            fluid = ~np.isnan(f[..., 0])
            got = np.where(fluid[..., None], f, 0.0)
            want = np.zeros_like(got)
            for c, v in case["after"].get(str(L), []):
                want[tuple(c) + (i,)] = v
            assert np.abs(got - want).max() < 1e-14, (case["name"], L)


CORNERS = [
    lambda: I.refined_box(levels=2, n=(8, 8, 8)),
    lambda: I.refined_box(levels=3, n=(8, 8, 8)),
    lambda: I.refined_box(levels=3, n=(8, 8, 8), Q=27, collision="kbc"),
    lambda: I.random_balanced(31, n=(6, 6, 6), levels=3, p_refine=0.6, p_bc=0.0, periodic=(1, 1, 1)),
    lambda: I.random_balanced(12, n=(6, 5, 4), levels=4, p_refine=0.6, p_bc=0.0, periodic=(1, 1, 1), Q=27),
]


@pytest.mark.parametrize("k", range(len(CORNERS)))
def test_V2_exact_mass_and_momentum_on_corner_grids(k):
    p = _randomise(CORNERS[k](), 2 + k)
    o = _vol(p)
    m0, j0 = _totals(o, p)
    o.step(10)
    m1, j1 = _totals(o, p)
    assert abs(m1 - m0) / m0 < 1e-13
    assert np.abs(j1 - j0).max() / m0 < 1e-13
    # the paper variant drifts on the same grid (R-A18): the pin has teeth
    q = oracle.Oracle(p)
    n0, _ = _totals(q, p)
    q.step(10)
    n1, _ = _totals(q, p)
    assert abs(n1 - n0) / n0 > 1e-9


def _walled_box(case):
    p = I.refined_box(levels=2, n=(8, 8, 8))
    p.bc = {2: (I.BC_NOSLIP, (0.0, 0.0, 0.0))}
    if case == "coarse_bc_leaf":
        p.masks[0][0, 0, 0] = 2
    elif case == "fine_bc_leaf_inside":
        p.masks[1][8, 8, 8] = 2
    elif case == "fine_bc_leaf_at_interface":
        p.masks[1][4, 6, 6] = 2
    elif case == "x_walls":
        p.periodic, p.face_bc = (0, 1, 1), (2, 2, 2, 2, 2, 2)
    return p


@pytest.mark.parametrize("case", ["coarse_bc_leaf", "fine_bc_leaf_inside", "fine_bc_leaf_at_interface", "x_walls"])
def test_V2_exact_mass_with_walls_off_the_coarse_interface(case):
    """Halfway bounce-back conserves mass at either resolution.  Exact as long
    as no wall touches the COARSE side of an interface (reading R-V4: there the
    coarse-resolution and fine-resolution bounce-back of diagonal links move a
    packet to different cells, so no single-resolution rule is conservative;
    test_V2_walls_on_the_coarse_interface_report_drift)."""
    p = _randomise(_walled_box(case), 5)
    o = _vol(p)
    m0, _ = _totals(o, p)
    o.step(10)
    m1, _ = _totals(o, p)
    assert abs(m1 - m0) / m0 < 1e-13


def test_V2_walls_on_the_coarse_interface_report_drift():
    p = _walled_box(None)
    p.masks[0][1, 3, 3] = 2  # coarse BC leaf next to the refined box
    _randomise(p, 5)
    o = _vol(p)
    m0, _ = _totals(o, p)
    o.step(10)
    m1, _ = _totals(o, p)
    assert 0 < abs(m1 - m0) / m0 < 1e-4


@pytest.mark.parametrize("k", range(len(CORNERS)))
def test_V3_uniform_equilibrium_invariance(k):
    p = CORNERS[k]()
    p.init_rho = p.init_u = None
    p.uniform_rho, p.uniform_u = 1.02, (0.031, -0.017, 0.022)
    o = _vol(p)
    o.step(6)
    for L in range(p.levels):
        r, u = o.macroscopic(L)
        m = ~np.isnan(r)
        if m.any():
            assert np.abs(r[m] - 1.02).max() < 1e-14
            assert np.abs(u[m] - np.array(p.uniform_u)).max() < 1e-14


def test_V4_single_level_equals_paper_variant():
    p = _randomise(I.random_balanced(7, n=(6, 5, 4), levels=1, p_bc=0.1), 7)
    a, b = oracle.Oracle(p), _vol(p)
    a.step(5)
    b.step(5)
    assert np.array_equal(a.get_f(0), b.get_f(0), equal_nan=True)


def test_V4_all_refined_equals_uniform_fine():
    n = (3, 2, 4)
    masks = [np.zeros(n, dtype=np.uint8), np.ones((6, 4, 8), dtype=np.uint8)]
    p = I.Problem(name="allref", nx=3, ny=2, nz=4, masks=masks, periodic=(1, 1, 1), Q=19, omega0=1.1)
    rng = np.random.default_rng(9)
    p.init_rho = [None, 1 + 0.01 * rng.uniform(-1, 1, (6, 4, 8))]
    p.init_u = [None, 0.03 * rng.uniform(-1, 1, (6, 4, 8, 3))]
    o = _vol(p)
    e, w, _ = oracle.lattice(19)
    f0 = o.get_f(1)
    o.step(5)
    ref = textbook_lbm(f0.copy(), e, w, 2 * 1.1 / (4 - 1.1), 10)
    assert np.abs(o.get_f(1) - ref).max() < 1e-15
