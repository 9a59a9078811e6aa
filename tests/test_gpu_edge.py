"""Edge and degenerate cases of the CUDA path against the fp64 oracle
(SURVEY §8(c.5) error definitions, tolerances of tests/_parity.py):

* zero coarse steps (lbm_step(0)) leaves the initial equilibrium;
* a level whose leaves are all boundary cells (no fluid leaf to update on it);
* a domain with no fluid leaf at all (every cell a wall leaf);
* domains smaller than one 8^3 block, periodic and walled, 1-3 levels;
* a refined level thinner than a block (1 coarse cell = 2 fine cells).
"""
import numpy as np
import pytest

import lbm_inputs as I
from tests._parity import TOL, errors, gpu_run, oracle_run

pytestmark = pytest.mark.gpu


def _lbmr():
    from paper_conf_ipps_mahmoudsm24_b200 import lbmr
    return lbmr


def _random_state(p, seed):
    rng = np.random.default_rng(seed)
    p.init_rho, p.init_u = [], []
    for L in range(p.levels):
        s = p.level_shape(L)
        p.init_rho.append(1 + 0.01 * rng.uniform(-1, 1, s))
        p.init_u.append(0.03 * rng.uniform(-1, 1, s + (3,)))
    return p


@pytest.mark.parametrize("prec", [0, 1])
def test_zero_steps_is_the_initial_state(prec):
    p = _random_state(I.cavity2(), 21)
    lbmr = _lbmr()
    g = lbmr.grid_from_problem(p, precision=prec)
    g.step(0)
    for L in range(p.levels):
        r, u = g.macroscopic(L)
        m = p.masks[L] == 1
        assert np.array_equal(~np.isnan(r), m)
        rho0, u0 = p.init_fields(L)
        tol = 1e-6 if prec == 0 else 1e-14
        assert np.abs(r[m] - rho0[m]).max() < tol
        assert np.abs(u[m] - u0[m]).max() < tol
    g.close()


def _two_level(n, refined, fine_code=1, periodic=(1, 1, 1), Q=19, collision="bgk"):
    """Level-0 mask n with the coarse cells `refined` (a slice tuple) refined;
    the level-1 leaves there get code fine_code."""
    m0 = np.ones(n, dtype=np.uint8)
    m0[refined] = 0
    m1 = np.zeros(tuple(2 * a for a in n), dtype=np.uint8)
    fine = tuple(slice(2 * s.start, 2 * s.stop) for s in refined)
    m1[fine] = fine_code
    return I.Problem(name="edge", nx=n[0], ny=n[1], nz=n[2], masks=[m0, m1], periodic=periodic, Q=Q,
                     collision=collision, omega0=1.6, bc={2: (0, (0.0, 0.0, 0.0))})


@pytest.mark.parametrize("prec", [0, 1])
def test_level_without_fluid_leaves(prec):
    """The refined level holds only wall leaves (a solid block at the fine
    resolution): level 1 has nothing to update, level 0 bounces off it."""
    p = _random_state(_two_level((6, 5, 4), (slice(2, 4), slice(1, 3), slice(1, 3)), fine_code=2), 22)
    o = oracle_run(p, 6)
    er, eu = errors(gpu_run(p, 6, prec), o, prec, 6, p.name)
    assert er <= TOL[prec] and eu <= TOL[prec], (er, eu)


@pytest.mark.parametrize("prec", [0, 1])
def test_domain_without_fluid(prec):
    """Every cell a wall leaf: the step runs, every output is NaN, no mass."""
    m = np.full((5, 3, 4), 2, dtype=np.uint8)
    p = I.Problem(name="solid", nx=5, ny=3, nz=4, masks=[m], periodic=(0, 0, 0), face_bc=(2,) * 6, Q=19,
                  omega0=1.2, bc={2: (0, (0.0, 0.0, 0.0))})
    lbmr = _lbmr()
    g = lbmr.grid_from_problem(p, precision=prec)
    g.step(3)
    r, u = g.macroscopic(0)
    assert np.isnan(r).all() and np.isnan(u).all()
    leaves, mass = g.stats()
    assert int(leaves[0]) == 0 and mass == 0.0
    g.close()


def tiny_problem(n, levels, periodic):
    """Domains smaller than one 8^3 block: one level all fluid, or coarse
    cell x = 0 refined (and, for 3 levels, its lower corner refined again)."""
    shapes = [tuple(a << L for a in n) for L in range(levels)]
    masks = [np.zeros(s, dtype=np.uint8) for s in shapes]
    if levels == 1:
        masks[0][...] = 1
    else:
        masks[0][...] = 1
        masks[0][0] = 0
        masks[1][0:2] = 1
        if levels == 3:
            masks[1][0, 0, 0] = 0
            masks[2][0:2, 0:2, 0:2] = 1
    p = I.Problem(name="tiny", nx=n[0], ny=n[1], nz=n[2], masks=masks, periodic=periodic, Q=19, omega0=1.4,
                  face_bc=(2, 2, 3, 2, 2, 2), bc={2: (0, (0.0, 0.0, 0.0)), 3: (1, (0.02, 0.0, 0.01))})
    return _random_state(p, 23)


TINY = [((1, 1, 1), 1, (1, 1, 1)), ((2, 3, 1), 1, (1, 0, 1)), ((3, 2, 2), 2, (1, 1, 1)),
        ((4, 4, 4), 3, (0, 0, 0))]


@pytest.mark.parametrize("n,levels,periodic", TINY)
@pytest.mark.parametrize("prec", [0, 1])
def test_domains_smaller_than_a_block(n, levels, periodic, prec):
    p = tiny_problem(n, levels, periodic)
    o = oracle_run(p, 5)
    er, eu = errors(gpu_run(p, 5, prec), o, prec, 5, p.name)
    assert er <= TOL[prec] and eu <= TOL[prec], (er, eu)


@pytest.mark.parametrize("Q,coll", [(19, "bgk"), (27, "kbc")])
@pytest.mark.parametrize("prec", [0, 1])
def test_refined_slab_thinner_than_a_block(Q, coll, prec):
    """One coarse cell refined across a periodic domain: the fine level is 2
    cells thick, so its explosion ghosts, coalescence candidates and fluid
    cells share blocks on both sides."""
    p = _random_state(_two_level((9, 4, 5), (slice(4, 5), slice(0, 4), slice(0, 5)), Q=Q, collision=coll), 24)
    o = oracle_run(p, 8)
    er, eu = errors(gpu_run(p, 8, prec), o, prec, 8, p.name)
    assert er <= TOL[prec] and eu <= TOL[prec], (er, eu)
