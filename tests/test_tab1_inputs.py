"""Tab. I sphere sweep inputs: the synthetic
recipe reproduces the paper's printed leaf distribution, tiles the domain,
is strongly 2:1 balanced (library validation), and sets Re = u R / nu = 4000
(Fig. 8 caption) at the finest level."""
import numpy as np
import pytest

import lbm_inputs as I


@pytest.mark.parametrize("size", [1, 2])
def test_leaf_distribution_matches_table1(size):
    p = I.sphere_tab1(size)
    leaves = p.fluid_leaves()[::-1]  # finest first, as Tab. I prints them
    for got, ref in zip(leaves, I.TAB1[size]["leaves_M"]):
        assert abs(got / 1e6 - ref) / ref < 0.02, (got, ref)
    # Tab. I consistency: the rows scale as size^3 (the voxelised sphere only
    # approximately, so the finest level within 0.5 %)
    if size == 2:
        one = I.sphere_tab1(1).fluid_leaves()
        assert [8 * v for v in one[:2]] == p.fluid_leaves()[:2]
        assert abs(8 * one[2] - p.fluid_leaves()[2]) / p.fluid_leaves()[2] < 5e-3


def test_domain_and_reynolds():
    p = I.sphere_tab1(1)
    assert (p.nx * 4, p.ny * 4, p.nz * 4) == (272, 192, 272)
    assert p.Q == 27 and p.collision == "kbc" and p.levels == 3
    nu0 = (1.0 / p.omega0 - 0.5) / 3.0
    nu2 = 4.0 * nu0  # nu constant in physical units: nu_L = 2^L nu_0
    R = 16.0
    assert abs(0.05 * R / nu2 - 4000.0) < 1e-6
    # the sphere is inside the finest region and made of no-slip BC leaves
    f = p.masks[2]
    assert np.count_nonzero(f == I.CLS_WALL) == pytest.approx(4.0 / 3.0 * np.pi * R ** 3, rel=0.02)


def test_library_accepts_tiling():
    from paper_conf_ipps_mahmoudsm24_b200 import lbmr
    p = I.sphere_tab1(1)
    gi = lbmr.analyze_problem(p, precision=lbmr.FP64)
    assert [gi.leaves[L] for L in range(3)] == p.fluid_leaves()
    assert gi.kernels_per_step == 7
    assert gi.launches_per_step == 7 + 1 + 2  # coalescence gathers before F_0 and the two F_1
