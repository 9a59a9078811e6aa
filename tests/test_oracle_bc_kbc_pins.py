"""Pins of the two oracle parts the round-1 pins left open:

T12  KBC's entropic stabiliser γ (reading R-A9; ref [18] P:L338).
     In Karlin et al.'s construction γ is the stationary point of the
     quadratic entropy H = Σ_i (f*_i − f^eq_i)^2 / f^eq_i along Δh.  The
     oracle's post-collision state must therefore make dH/dt vanish on the
     line through it and the γ = 2 (BGK) state, whatever Δs is (Δs itself is
     pinned by T2's deviatoric-relaxation test).  f^eq is Eq.5 written out
     here, independently of the oracle.
T13  Outflow ("the missing directions of the distribution function
     f_i at the boundary are simply assigned the corresponding lattice
     weights w_i"), per link, after one step from a random state.
T14  Velocity inlet / moving wall ("prescribed using the same
     bounce-back technique"), per link: f_i = f*_ī + 6 w_i ρ_w e_i·u_w, ρ_w = 1
     (reading R-A11), with f* the cell's own post-collision state.
T15  Edge priority (R-A11): a link whose source leaves the domain through an
     outflow face AND a no-slip face bounces back; through an inlet face and a
     no-slip face takes the inlet rule.
T16  A fluid at rest is invariant for 100 coarse steps on a 2-level grid whose
     faces are outflow, inlet (u = 0) and no-slip.
None of these call the CUDA path.
"""
import numpy as np
import pytest

import lbm_inputs as I
import oracle


def _feq_eq5(e, w, rho, u):
    """Eq.(5) P:L61-64 with c_s^2 = 1/3, written out here."""
    eu = e @ u
    return w * rho * (1.0 + 3.0 * eu + 4.5 * eu * eu - 1.5 * (u @ u))


def _random_state(Q, rng, amp):
    e, w, _ = oracle.lattice(Q)
    u = rng.uniform(-0.06, 0.06, 3)
    rho = 1.0 + rng.uniform(-0.03, 0.03)
    f = _feq_eq5(e.astype(float), w, rho, u)
    return f * (1.0 + amp * rng.uniform(-1, 1, Q))


# ---------------------------------------------------------------- T12 KBC γ
@pytest.mark.parametrize("amp", [0.02, 0.1, 0.3])
def test_T12_kbc_gamma_is_quadratic_entropy_stationary(amp):
    Q = 27
    e, w, _ = oracle.lattice(Q)
    e = e.astype(float)
    rng = np.random.default_rng(1200 + int(amp * 100))
    worst = 0.0
    for _ in range(30):
        f = _random_state(Q, rng, amp)
        om = rng.uniform(0.8, 1.999)
        rho = f.sum()
        feq = _feq_eq5(e, w, rho, (f @ e) / rho)
        fk = oracle.collide_cell(Q, "kbc", om, f)
        fb = oracle.collide_cell(Q, "kbc", om, f, force_gamma2=True)
        d = fk - fb  # = -β (γ - 2) Δh: the line of all γ
        if np.abs(d).max() < 1e-13 * np.abs(f).max():
            continue  # γ == 2 to rounding: the line is degenerate
        # H(t) = Σ (fb + t d - feq)^2 / feq ;  dH/dt(1) = 2 Σ (fk - feq) d / feq
        dH = np.sum((fk - feq) * d / feq)
        # scale of the terms of that sum
        scale = np.sum(np.abs((fk - feq) * d / feq))
        worst = max(worst, abs(dH) / scale)
        # t = 1 is the minimum of the convex quadratic H(t)
        H = lambda t: np.sum((fb + t * d - feq) ** 2 / feq)
        assert H(1.0) <= H(0.9) and H(1.0) <= H(1.1)
    assert worst < 1e-10, worst


# ---------------------------------------------------------------- T13-T15 BCs
def _face_problem(Q, levels, face_bc, periodic, bc, rng, omega0=1.3, collision="bgk"):
    n = (4, 5, 6)
    masks = [np.ones(n, dtype=np.uint8)]
    if levels == 2:  # refined slab touching the -x face (fine cells at the boundary)
        masks = [np.ones(n, dtype=np.uint8), np.zeros((8, 10, 12), dtype=np.uint8)]
        masks[0][:2] = 0
        masks[1][:4] = 1
    p = I.Problem(name="faces", nx=n[0], ny=n[1], nz=n[2], masks=masks, periodic=periodic, face_bc=face_bc,
                  Q=Q, collision=collision, omega0=omega0, bc=bc)
    p.init_rho = [1 + 0.02 * rng.uniform(-1, 1, p.level_shape(L)) for L in range(levels)]
    p.init_u = [0.04 * rng.uniform(-1, 1, p.level_shape(L) + (3,)) for L in range(levels)]
    return p


def _one_step_links(p):
    """(f before, f after one coarse step, post-collision of the initial state)
    per level, dense [x,y,z,Q], in the oracle's direction order."""
    o = oracle.Oracle(p)
    f0 = [o.get_f(L) for L in range(p.levels)]
    o.step(1)
    f1 = [o.get_f(L) for L in range(p.levels)]
    return o, f0, f1


CLS_OUT, CLS_IN, CLS_WALL = 7, 8, 9
U_IN = (0.041, -0.013, 0.027)


@pytest.mark.parametrize("Q,coll", [(19, "bgk"), (27, "bgk"), (27, "kbc")])
def test_T13_T14_outflow_and_inlet_per_link(Q, coll):
    """Single level, x faces only (y, z periodic): -x OUTFLOW, +x VELOCITY.
    Every link entering through -x carries exactly w_i; every link entering
    through +x carries f*_ī + 6 w_i e_i·u_in, f* = collide(initial f) of the
    same cell."""
    rng = np.random.default_rng(1300 + Q)
    bc = {CLS_OUT: (I.BC_OUTFLOW, (0.0, 0.0, 0.0)), CLS_IN: (I.BC_VELOCITY, U_IN)}
    p = _face_problem(Q, 1, (CLS_OUT, CLS_IN, 0, 0, 0, 0), (0, 1, 1), bc, rng, collision=coll)
    e, w, opp = oracle.lattice(Q)
    o, f0, f1 = _one_step_links(p)
    nx = p.level_shape(0)[0]
    n_out = n_in = 0
    for y in range(p.ny):
        for z in range(p.nz):
            for i in range(Q):
                if e[i][0] == 1:  # source x = -1: outside the -x face
                    assert f1[0][0, y, z, i] == w[i]
                    n_out += 1
                if e[i][0] == -1:  # source x = nx: outside the +x face
                    fs = oracle.collide_cell(Q, coll, p.omega0, f0[0][nx - 1, y, z])
                    eu = e[i][0] * U_IN[0] + e[i][1] * U_IN[1] + e[i][2] * U_IN[2]
                    want = fs[opp[i]] + 6.0 * w[i] * 1.0 * eu
                    assert abs(f1[0][nx - 1, y, z, i] - want) <= 2e-16, (i, y, z)
                    n_in += 1
    assert n_out == n_in == p.ny * p.nz * (5 if Q == 19 else 9)
    del o


def test_T13_outflow_on_a_refined_face():
    """2 levels, the fine slab touches the -x OUTFLOW face: the fine boundary
    cells get w_i on every entering link (both substeps; the value after the
    coarse step is the second substep's)."""
    rng = np.random.default_rng(1310)
    bc = {CLS_OUT: (I.BC_OUTFLOW, (0.0, 0.0, 0.0)), CLS_IN: (I.BC_VELOCITY, U_IN)}
    p = _face_problem(19, 2, (CLS_OUT, CLS_IN, 0, 0, 0, 0), (0, 1, 1), bc, rng)
    e, w, _ = oracle.lattice(19)
    _, _, f1 = _one_step_links(p)
    fine = f1[1]
    cnt = 0
    for i in range(19):
        if e[i][0] == 1:
            assert np.all(fine[0, :, :, i] == w[i])
            cnt += 1
    assert cnt == 5
    # the coarse level never touches -x (ABSENT there): no outflow value leaks in
    assert np.all(np.isnan(f1[0][0]))


@pytest.mark.parametrize("Q", [19, 27])
def test_T15_edge_priority_per_link(Q):
    """y walls (NOSLIP) meet the x faces: at the (x=0, y=0) edge a link whose
    source is outside both -x (OUTFLOW) and -y (NOSLIP) bounces back (NOSLIP >
    OUTFLOW); at (x=nx-1, y=0) a link outside +x (VELOCITY) and -y (NOSLIP) takes
    the inlet rule (VELOCITY > NOSLIP), R-A11."""
    rng = np.random.default_rng(1500 + Q)
    bc = {CLS_OUT: (I.BC_OUTFLOW, (0.0, 0.0, 0.0)), CLS_IN: (I.BC_VELOCITY, U_IN),
          CLS_WALL: (I.BC_NOSLIP, (0.0, 0.0, 0.0))}
    p = _face_problem(Q, 1, (CLS_OUT, CLS_IN, CLS_WALL, CLS_WALL, 0, 0), (0, 0, 1), bc, rng)
    e, w, opp = oracle.lattice(Q)
    _, f0, f1 = _one_step_links(p)
    nx = p.level_shape(0)[0]
    checked = 0
    for z in range(p.nz):
        fs0 = oracle.collide_cell(Q, "bgk", p.omega0, f0[0][0, 0, z])
        fs1 = oracle.collide_cell(Q, "bgk", p.omega0, f0[0][nx - 1, 0, z])
        for i in range(Q):
            if e[i][0] == 1 and e[i][1] == 1:  # outside -x and -y: NOSLIP wins
                assert f1[0][0, 0, z, i] == fs0[opp[i]]
                checked += 1
            if e[i][0] == 1 and e[i][1] == 0:  # outside -x only: OUTFLOW
                assert f1[0][0, 0, z, i] == w[i]
            if e[i][0] == -1 and e[i][1] == 1:  # outside +x and -y: VELOCITY wins
                eu = e[i][0] * U_IN[0] + e[i][1] * U_IN[1] + e[i][2] * U_IN[2]
                assert abs(f1[0][nx - 1, 0, z, i] - (fs1[opp[i]] + 6.0 * w[i] * 1.0 * eu)) <= 2e-16
                checked += 1
            if e[i][0] == 0 and e[i][1] == 1:  # outside -y only: NOSLIP
                assert f1[0][0, 0, z, i] == fs0[opp[i]]
    assert checked == p.nz * (2 if Q == 19 else 6)


def test_T16_rest_state_invariant_with_open_faces():
    """ρ = 1, u = 0 (f = w) is a fixed point of collision, streaming, explosion,
    coalescence, no-slip, a u = 0 inlet and the outflow rule f_i = w_i: 100
    coarse steps on a 2-level grid with all three face kinds."""
    n = (8, 6, 6)
    masks = [np.ones(n, dtype=np.uint8), np.zeros((16, 12, 12), dtype=np.uint8)]
    masks[0][2:6, 2:4, 1:5] = 0
    masks[1][4:12, 4:8, 2:10] = 1
    bc = {CLS_OUT: (I.BC_OUTFLOW, (0.0, 0.0, 0.0)), CLS_IN: (I.BC_VELOCITY, (0.0, 0.0, 0.0)),
          CLS_WALL: (I.BC_NOSLIP, (0.0, 0.0, 0.0))}
    p = I.Problem(name="rest", nx=n[0], ny=n[1], nz=n[2], masks=masks, periodic=(0, 0, 0),
                  face_bc=(CLS_IN, CLS_OUT, CLS_WALL, CLS_WALL, CLS_OUT, CLS_WALL), Q=19, omega0=1.7, bc=bc)
    o = oracle.Oracle(p)
    o.step(100)
    _, w, _ = oracle.lattice(19)
    for L in range(2):
        f = o.get_f(L)
        m = ~np.isnan(f[..., 0])
        assert np.abs(f[m] - w).max() < 1e-15
