"""Parity at BASELINE.json's FULL sizes, in the launch configuration bench.py
times (the fused kernels replayed from the CUDA graph), on sampled outputs.

Dense per-level arrays do not fit at these sizes (cfg5's finest level alone
has 1.13 G cells), so both sides are read through probes (lbm_probe /
Oracle.probe) at seeded random fluid leaves of every level, after FIVE coarse
steps (so interface, wall, inlet and outflow cells have left the uniform
initial state).  Half of every level's samples are drawn from its *special*
leaves — fluid leaves with a 26-neighbour that is not a same-level fluid leaf
(refinement interface, BC leaf, domain face) — where all the non-trivial
rules act; the other half uniformly from all fluid leaves.  cfg3 / cfg4 / cfg5 compare with the fp64 oracle run on the same full
grid; cfg2 (512^3 periodic, too large for the oracle's dense maps) compares
with the one-step result the oracle's own collision and equilibrium compute
cell by cell.  Bars as everywhere: fp32 <= 1e-5, fp64 <= 1e-12 relative to
the sample's field maxima."""
import gc

import numpy as np
import pytest

import lbm_inputs as I
import oracle
from tests._parity import TOL

pytestmark = pytest.mark.gpu

FP32, FP64 = 0, 1
N_SAMPLE = 100_000  # per level
N_STEPS = 5


def _special(prob, L):
    """Fluid leaves of level L with a 26-neighbour that is not a same-level
    fluid leaf (outside the domain counts on non-periodic axes)."""
    fluid = prob.masks[L] == 1
    d = ~fluid
    for ax in range(3):
        a = d.copy()
        if prob.periodic[ax]:
            a |= np.roll(d, 1, ax)
            a |= np.roll(d, -1, ax)
        else:
            lo = [slice(None)] * 3
            hi = [slice(None)] * 3
            lo[ax], hi[ax] = slice(1, None), slice(None, -1)
            a[tuple(lo)] |= d[tuple(hi)]
            a[tuple(hi)] |= d[tuple(lo)]
            e0 = [slice(None)] * 3
            e1 = [slice(None)] * 3
            e0[ax], e1[ax] = 0, -1
            a[tuple(e0)] = True
            a[tuple(e1)] = True
        d = a
    return fluid & d


def _sample_mixed(prob, L, n, seed):
    """n/2 special leaves and n/2 uniform fluid leaves of level L (fewer if the
    level has fewer)."""
    m = prob.masks[L]
    rng = np.random.default_rng(seed + 100 * L)
    spec = np.flatnonzero(_special(prob, L))
    flat = np.flatnonzero(m == 1)
    a = rng.choice(spec, size=min(n // 2, spec.size), replace=False) if spec.size else np.zeros(0, np.int64)
    b = rng.choice(flat, size=min(n - a.size, flat.size), replace=False)
    pick = np.concatenate([a, b])
    return np.stack(np.unravel_index(pick, m.shape), axis=1).astype(np.int64), a.size


def _sample(prob, L, n, seed):
    m = prob.masks[L]
    flat = np.flatnonzero(m == 1)
    rng = np.random.default_rng(seed + L)
    pick = rng.choice(flat, size=min(n, flat.size), replace=False)
    return np.stack(np.unravel_index(pick, m.shape), axis=1).astype(np.int64)


def _rel_err(gpu, ref):
    """Max errors over all levels normalised by the field maxima over all
    levels (as tests/_parity.errors)."""
    dr = du = mr = mu = 0.0
    for (rg, ug), (ro, uo) in zip(gpu, ref):
        assert not np.isnan(rg).any() and not np.isnan(ro).any()
        dr, du = max(dr, np.abs(rg - ro).max()), max(du, np.abs(ug - uo).max())
        mr, mu = max(mr, np.abs(ro).max()), max(mu, np.abs(uo).max())
    return dr / mr, du / max(mu, 1e-300)


def _gpu_probe(prob, prec, samples, steps=N_STEPS):
    from paper_conf_ipps_mahmoudsm24_b200 import lbmr
    g = lbmr.grid_from_problem(prob, precision=prec)
    g.step(steps)
    out = [g.probe(L, xyz) for L, xyz in enumerate(samples)]
    g.close()
    return out


FULL = {
    "cfg3_sphere3": lambda: I.sphere3(),
    "cfg4_cavity4_kbc": lambda: I.cavity4_kbc(),
    "cfg5_tunnel4": lambda: I.tunnel4(),
}


@pytest.mark.parametrize("name", list(FULL))
def test_full_size_sampled_parity(name):
    from tests._parity import record
    prob = FULL[name]()
    mixed = [_sample_mixed(prob, L, N_SAMPLE, 17) for L in range(prob.levels)]
    samples = [m[0] for m in mixed]
    n_special = [m[1] for m in mixed]
    # half of every level's sample is special (all of its special leaves when it has fewer)
    for L in range(prob.levels):
        assert n_special[L] == min(N_SAMPLE // 2, int(_special(prob, L).sum())), (L, n_special[L])
    o = oracle.Oracle(prob)
    o.step(N_STEPS)
    ref = [o.probe(L, xyz) for L, xyz in enumerate(samples)]
    del o
    gc.collect()
    for prec in (FP64, FP32):
        got = _gpu_probe(prob, prec, samples)
        er, eu = _rel_err(got, ref)
        record("test_full_size_sampled_parity", name, N_STEPS, prec, er, eu,
               samples=[len(s) for s in samples], special_samples=n_special)
        assert er <= TOL[prec] and eu <= TOL[prec], (name, prec, er, eu)


def test_full_size_uniform512_one_step():
    """cfg2: 512^3 periodic Taylor-Green at omega = 1.  The oracle's own
    collision (ora_collide_cell) and equilibrium give the one-step value at
    every sampled cell from its Q upwind neighbours' initial equilibria."""
    prob = I.uniform(512)
    n = 512
    xyz = _sample(prob, 0, 20_000, 5)
    e, _, _ = oracle.lattice(19)
    rho0, u0 = prob.init_fields(0)
    ref_r = np.empty(len(xyz))
    ref_u = np.empty((len(xyz), 3))
    for k, p in enumerate(xyz):
        f = np.empty(19)
        for i in range(19):
            s = (p - e[i]) % n
            feq = oracle.equilibrium(19, rho0[tuple(s)], u0[tuple(s)])
            f[i] = oracle.collide_cell(19, "bgk", prob.omega0, feq)[i]
        ref_r[k] = f.sum()
        ref_u[k] = (e * f[:, None]).sum(axis=0) / ref_r[k]
    for prec in (FP64, FP32):
        got = _gpu_probe(prob, prec, [xyz], steps=1)[0]
        er, eu = _rel_err([got], [(ref_r, ref_u)])
        assert er <= TOL[prec] and eu <= TOL[prec], (prec, er, eu)


def test_probe_matches_macroscopic():
    """lbm_probe == the dense lbm_macroscopic at the same cells (small grid),
    NaN off fluid leaves and outside the domain."""
    from paper_conf_ipps_mahmoudsm24_b200 import lbmr
    prob = I.tunnel4(scale=5)
    g = lbmr.grid_from_problem(prob, precision=FP64)
    g.step(2)
    for L in range(prob.levels):
        r, u = g.macroscopic(L)
        sh = prob.level_shape(L)
        rng = np.random.default_rng(L)
        xyz = np.stack([rng.integers(-1, s + 1, 3000) for s in sh], axis=1)
        pr, pu = g.probe(L, xyz)
        inside = np.all((xyz >= 0) & (xyz < np.array(sh)), axis=1)
        assert np.isnan(pr[~inside]).all()
        c = tuple(xyz[inside].T)
        np.testing.assert_array_equal(pr[inside], r[c])
        np.testing.assert_array_equal(pu[inside], u[c])
    g.close()
