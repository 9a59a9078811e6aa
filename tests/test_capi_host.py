"""Host-side checks of the C-ABI library (no GPU): exports, lattice tables,
Eq.9, the pipelined level schedule, and the grid builder's validation and
block statistics (T14)."""
import ctypes
import math
import os
import re

import numpy as np
import pytest

import lbm_inputs as I
from paper_conf_ipps_mahmoudsm24_b200 import lbmr

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_functions():
    names = set()
    for fn in os.listdir(os.path.join(ROOT, "include")):
        if fn.endswith(".h"):
            txt = open(os.path.join(ROOT, "include", fn)).read()
            txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
            names |= set(re.findall(r"\b(lbm_[a-z_]+)\s*\(", txt))
    return names


def test_library_exports_every_declared_symbol():
    lib = lbmr.load_library()
    declared = header_functions()
    assert len(declared) >= 17
    for name in declared:
        assert hasattr(lib, name), name
    assert lib.lbm_version().startswith(b"lbmr")


@pytest.mark.parametrize("Q", [19, 27])
def test_product_lattice_isotropy(Q):
    e, w = lbmr.lattice_table(Q)
    assert len({tuple(v) for v in e}) == Q
    d = np.eye(3)
    assert abs(w.sum() - 1) < 1e-15
    assert np.abs(w @ e).max() < 1e-15
    assert np.abs(np.einsum("q,qa,qb->ab", w, e, e) - d / 3).max() < 1e-15
    m4 = np.einsum("q,qa,qb,qc,qd->abcd", w, e, e, e, e)
    iso = (np.einsum("ab,cd->abcd", d, d) + np.einsum("ac,bd->abcd", d, d) + np.einsum("ad,bc->abcd", d, d)) / 9
    assert np.abs(m4 - iso).max() < 1e-15
    # opposite pairs (q, q+1) for odd q, as the kernels assume
    for q in range(1, Q, 2):
        assert np.all(e[q] == -e[q + 1])
    if Q == 27:
        e19, _ = lbmr.lattice_table(19)
        assert np.array_equal(e[:19], e19)


def test_omega_level_eq9_and_tau_relation():
    for om0 in [0.7, 1.0, 1.824818, 1.994018]:
        for L in range(5):
            tau = 2 ** L / om0 + 0.5 * (1 - 2 ** L)
            assert abs(lbmr.omega_level(om0, L) * tau - 1) < 1e-13


@pytest.mark.parametrize("levels", [1, 2, 3, 4, 5, 6])
def test_pipelined_schedule_reads_what_algorithm1_reads(levels):
    """Symbolic data flow of the pipelined order with two buffers per level.
    Every F_L^k must find, at the moment it runs: C_L^k in buf[L][k%2], the
    coarse post-collision C_{L-1}^{ceil(k/2)} (Explosion, both fine substeps
    read the same coarse value) and the two fine post-collision states
    C_{L+1}^{2k-1}, C_{L+1}^{2k} (Accumulate/Coalescence) -- exactly the
    values the recursion of Algorithm 1 uses."""
    buf = [[0, 1] for _ in range(levels)]  # version held: f^0 in buf 0, C^1 in buf 1 (prologue)
    done = [0] * levels
    for n in range(4):
        order = lbmr.schedule(levels, n)
        assert len(order) == 2 ** levels - 1
        for L, k in order:
            assert k == done[L] + 1, "substeps of a level run in order"
            assert buf[L][k % 2] == k
            if L > 0:
                kc = (k + 1) // 2
                assert buf[L - 1][kc % 2] == kc
            if L < levels - 1:
                assert buf[L + 1][1] == 2 * k - 1 and buf[L + 1][0] == 2 * k
            buf[L][(k + 1) % 2] = k + 1
            done[L] = k
        for L in range(levels):
            assert done[L] == (n + 1) * 2 ** L  # acoustic scaling


# ---------------------------------------------------------------- T14 validation
def _analyze(masks, n, **kw):
    kw.setdefault("face_bc", (2,) * 6)
    return lbmr.analyze(*n, masks, **kw)


def test_valid_two_level_grid_counts():
    p = I.cavity2()
    gi = lbmr.analyze_problem(p)
    assert list(gi.leaves[:2]) == [28672, 32768]
    assert gi.kernels_per_step == 3


def test_rejects_uncovered_cell():
    m0 = np.zeros((4, 4, 4), np.uint8)
    m1 = np.ones((8, 8, 8), np.uint8)
    m1[3, 4, 5] = 0
    with pytest.raises(lbmr.LBMError) as ei:
        _analyze([m0, m1], (4, 4, 4))
    assert ei.value.status == 2 and "level 1 cell (3,4,5)" in str(ei.value)


def test_rejects_overlap():
    m0 = np.ones((4, 4, 4), np.uint8)
    m1 = np.zeros((8, 8, 8), np.uint8)
    m1[0, 0, 0] = 1
    with pytest.raises(lbmr.LBMError) as ei:
        _analyze([m0, m1], (4, 4, 4))
    assert ei.value.status == 2


def test_rejects_two_level_jump():
    # level-0 leaves touching level-2 leaves (diagonal contact counts)
    n = (4, 4, 4)
    m0 = np.ones(n, np.uint8)
    m0[2:, 2:, 2:] = 0
    m1 = np.zeros((8, 8, 8), np.uint8)
    m1[4:, 4:, 4:] = 1
    m1[4:6, 4:6, 4:6] = 0
    m2 = np.zeros((16, 16, 16), np.uint8)
    m2[8:12, 8:12, 8:12] = 1
    with pytest.raises(lbmr.LBMError) as ei:
        _analyze([m0, m1, m2], n)
    assert ei.value.status == 3
    # the same with a one-cell buffer is fine
    m0b = np.ones((6, 6, 6), np.uint8)
    m0b[2:, 2:, 2:] = 0
    m1b = np.zeros((12, 12, 12), np.uint8)
    m1b[4:, 4:, 4:] = 1
    m1b[6:10, 6:10, 6:10] = 0
    m2b = np.zeros((24, 24, 24), np.uint8)
    m2b[12:20, 12:20, 12:20] = 1
    gi = _analyze([m0b, m1b, m2b], (6, 6, 6))
    assert gi.leaves[2] == 512


def test_rejects_bad_arguments():
    m = [np.ones((4, 4, 4), np.uint8)]
    with pytest.raises(lbmr.LBMError) as ei:
        _analyze(m, (4, 4, 4), lattice=19, collision=lbmr.KBC)
    assert ei.value.status == 8
    with pytest.raises(lbmr.LBMError) as ei:
        _analyze(m, (4, 4, 4), face_bc=(2, 2, 0, 2, 2, 2))
    assert ei.value.status == 1
    with pytest.raises(lbmr.LBMError) as ei:
        _analyze(m, (4, 4, 4), omega0=2.0)
    assert ei.value.status == 1
    bad = np.ones((4, 4, 4), np.uint8)
    bad[1, 1, 1] = 255
    with pytest.raises(lbmr.LBMError) as ei:
        _analyze([bad], (4, 4, 4))
    assert ei.value.status == 1
    # periodic faces need no face BC
    gi = _analyze(m, (4, 4, 4), face_bc=(0,) * 6, periodic=(1, 1, 1))
    assert gi.leaves[0] == 64


def test_builder_statistics_of_the_baseline_configs():
    """Interface structure of cfg3/cfg5 (6.4/5.2/3.1 % and
    9.0/6.5/6.3/3.0 % of the leaves have a link that is not a same-level
    fluid pull).  With explosion and coalescence ghosts those interface links
    become plain pulls, so only wall / BC-body links stay on the slow path:
    cfg5 level 2 (no wall, no body) has none at all."""
    gi = lbmr.analyze_problem(I.sphere3())
    assert list(gi.leaves[:3]) == [3375104, 5373952, 9299808]
    sc = [gi.special_cells[L] / gi.leaves[L] for L in range(3)]
    assert sc[0] < 0.064 and sc[1] < 0.052 and sc[2] < 0.031 * 0.2
    assert gi.special_cells[1] == 0  # level 1 touches neither walls nor the sphere
    gi = lbmr.analyze_problem(I.tunnel4())
    assert list(gi.leaves[:4]) == [1413300, 4670400, 8940544, 33155968]
    assert gi.kernels_per_step == 15
    sc = [gi.special_cells[L] / gi.leaves[L] for L in range(4)]
    assert sc[0] < 0.090 and sc[1] < 0.065 and sc[3] < 0.01
    assert gi.special_cells[2] == 0


# ---------------------------------------------------------------- block-grid alignment
def _offset_problem():
    """2 levels, the refined box starting at coarse x = 3 (level-1 x = 6, 6 mod 8 = 6):
    the builder should shift level 1's block grid by 2 in x."""
    n = (16, 12, 10)
    masks = I._box_masks(n, [((3, 11), (2, 8), (0, 10))])
    return I.Problem(name="offset", nx=n[0], ny=n[1], nz=n[2], masks=masks, face_bc=(2,) * 6, Q=19,
                     omega0=1.2, bc={2: (I.BC_NOSLIP, (0.0, 0.0, 0.0))})


def test_block_grid_offsets_align_level_faces(monkeypatch):
    p = _offset_problem()
    a = lbmr.analyze_problem(p)
    off = [[a.block_offset[L][k] for k in range(3)] for L in range(p.levels)]
    # level 1 fluid region x in [6, 22): faces at 6 and 22 (both 6 mod 8) -> offset 2;
    # y in [4, 16): faces 4 and 16 (4 and 0 mod 8) and the domain faces 0 and 24 -> 0 wins
    assert off[1][0] == 2, off
    assert off[0] == [0, 0, 0], off
    monkeypatch.setenv("LBMR_NO_BLOCK_ALIGN", "1")
    b = lbmr.analyze_problem(p)
    assert [[b.block_offset[L][k] for k in range(3)] for L in range(2)] == [[0, 0, 0], [0, 0, 0]]
    # same leaves and work (the aligned grid stores its explosion ghosts in ghost-only blocks
    # outside the fluid region's rows, so it may hold more population blocks)
    assert list(a.leaves[:2]) == list(b.leaves[:2])


def test_block_grid_offsets_zero_on_periodic_axes():
    p = I.random_balanced(31, n=(12, 10, 9), levels=3, p_refine=0.6, periodic=(1, 1, 1), p_bc=0.0)
    a = lbmr.analyze_problem(p)
    assert all(a.block_offset[L][k] == 0 for L in range(3) for k in range(3))
