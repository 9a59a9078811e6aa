"""Brute-force per-link definition of one coarse step (TEST INFRASTRUCTURE).

An independent second reading of the method for tiny grids, written from the
paper without the structured oracle's classification code:

* every link is resolved by POINT LOCATION in the multi-level tiling: the leaf
  containing the point y = x_p - e_i h (x_p the centre of leaf p, h = 2^-L);
* same level -> Streaming, Eq.(2); one level coarser -> Explosion,
  Eq.(10); y inside a refined cell -> Coalescence, Eq.(11) P:L110 over
  the fine fluid leaves beta whose point x_beta + e_i h/2 lies inside p;
  BC leaf / outside -> bounce-back / moving wall / outflow;
* the fine-to-coarse sum is formed as the paper's Accumulate: after
  every fine Collision the post-collision values are added into a per-leaf
  accumulator, the coarse side divides by n = 2|B| and resets it;
* the recursion is Algorithm 1 line by line.

Its lattice, equilibrium and collisions are its own numpy code.  Used only on
grids of a few thousand cells (pure-Python link loop).
"""
from __future__ import annotations

import itertools

import numpy as np

NOSLIP, VELOCITY, OUTFLOW = 0, 1, 2


def lattice(Q):
    dirs = [d for d in itertools.product((0, 1, -1), repeat=3) if Q == 27 or sum(abs(c) for c in d) <= 2]
    e = np.array(dirs, dtype=np.int64)
    n2 = (e * e).sum(1)
    if Q == 19:
        w = np.choose(n2, [1 / 3, 1 / 18, 1 / 36, 0.0])
    else:
        w = np.choose(n2, [8 / 27, 2 / 27, 1 / 54, 1 / 216])
    opp = np.array([dirs.index(tuple(-c for c in d)) for d in dirs])
    return e, w.astype(np.float64), opp


def feq_of(e, w, rho, u):
    eu = u @ e.T
    uu = (u * u).sum(-1, keepdims=True)
    return w * rho[:, None] * (1 + 3 * eu + 4.5 * eu * eu - 1.5 * uu)


def collide(e, w, f, omega, kind):
    rho = f.sum(1)
    u = (f @ e) / rho[:, None]
    feq = feq_of(e, w, rho, u)
    fneq = f - feq
    if kind == "bgk":
        return f - omega * fneq
    # KBC [18] (reading R-A9), vectorised over cells
    P = np.einsum("qa,qb,cq->cab", e, e, fneq)
    Nxz = P[:, 0, 0] - P[:, 2, 2]
    Nyz = P[:, 1, 1] - P[:, 2, 2]
    ds = np.zeros_like(f)
    n2 = (e * e).sum(1)
    for i in range(e.shape[0]):
        ex, ey, ez = e[i]
        if n2[i] == 1:
            if ex:
                ds[:, i] = (2 * Nxz - Nyz) / 6
            elif ey:
                ds[:, i] = (-Nxz + 2 * Nyz) / 6
            else:
                ds[:, i] = (-Nxz - Nyz) / 6
        elif n2[i] == 2:
            if ez == 0:
                ds[:, i] = ex * ey * P[:, 0, 1] / 4
            elif ey == 0:
                ds[:, i] = ex * ez * P[:, 0, 2] / 4
            else:
                ds[:, i] = ey * ez * P[:, 1, 2] / 4
    dh = fneq - ds
    sh = (ds * dh / feq).sum(1)
    hh = (dh * dh / feq).sum(1)
    beta = omega / 2
    with np.errstate(divide="ignore", invalid="ignore"):
        gamma = np.where(hh < 1e-30, 2.0, 1 / beta - (2 - 1 / beta) * sh / np.where(hh < 1e-30, 1.0, hh))
    return f - beta * (2 * ds + gamma[:, None] * dh)


class Brute:
    def __init__(self, prob):
        self.p = prob
        self.Q = prob.Q
        self.e, self.w, self.opp = lattice(prob.Q)
        self.Lmax = prob.levels
        self.masks = [np.asarray(m) for m in prob.masks]
        self.shape = [prob.level_shape(L) for L in range(self.Lmax)]
        self.kind, self.uw = prob.bc_arrays()
        # omega per level from the tau relation of P:L96 (not Eq.9's closed form)
        t0 = 1.0 / prob.omega0
        self.omega = [1.0 / (2 ** L * t0 + 0.5 * (1 - 2 ** L)) for L in range(self.Lmax)]
        self.f, self.fs, self.acc = [], [], []
        self.fluid = []
        for L in range(self.Lmax):
            fl = np.argwhere(self.masks[L] == 1)
            self.fluid.append(fl)
            rho, u = prob.init_fields(L)
            r = rho[tuple(fl.T)]
            uu = u[tuple(fl.T)]
            self.f.append(feq_of(self.e, self.w, r, uu))
            self.fs.append(np.zeros_like(self.f[-1]))
            self.acc.append(np.zeros_like(self.f[-1]))
        self.index = []
        for L in range(self.Lmax):
            idx = -np.ones(self.shape[L], dtype=np.int64)
            idx[tuple(self.fluid[L].T)] = np.arange(len(self.fluid[L]))
            self.index.append(idx)

    # ---- point location in the multi-level tiling -------------------------
    def locate(self, y):
        """y in coarse units -> ('out', faces) or (level, cell, code)."""
        y = np.array(y, dtype=np.float64)
        out = [0, 0, 0]
        n0 = (self.p.nx, self.p.ny, self.p.nz)
        for a in range(3):
            if y[a] < 0 or y[a] >= n0[a]:
                if self.p.periodic[a]:
                    y[a] = y[a] % n0[a]
                else:
                    out[a] = -1 if y[a] < 0 else 1
        if any(out):
            return ("out", out)
        for L in range(self.Lmax):
            c = tuple(int(np.floor(y[a] * 2 ** L)) for a in range(3))
            code = int(self.masks[L][c])
            if code:
                return (L, c, code)
        raise AssertionError("point not covered by a leaf")

    def bc(self, L, k, i, cls):
        kind = self.kind[cls]
        if kind == OUTFLOW:
            return self.w[i]
        v = self.fs[L][k, self.opp[i]]
        if kind == VELOCITY:
            v += 6 * self.w[i] * float(self.e[i] @ self.uw[cls])
        return v

    def face_class(self, out):
        best, bp = None, -1
        for a in range(3):
            if out[a]:
                cls = self.p.face_bc[2 * a + (1 if out[a] > 0 else 0)]
                pr = {VELOCITY: 3, NOSLIP: 2, OUTFLOW: 1}[int(self.kind[cls])]
                if pr > bp:
                    best, bp = cls, pr
        return best

    def stream(self, L):
        h = 0.5 ** L
        newf = np.empty_like(self.f[L])
        for k, p in enumerate(self.fluid[L]):
            xp = (p + 0.5) * h
            for i in range(self.Q):
                y = xp - self.e[i] * h
                loc = self.locate(y)
                if loc[0] == "out":
                    newf[k, i] = self.bc(L, k, i, self.face_class(loc[1]))
                    continue
                M, c, code = loc
                if M == L or M == L - 1:
                    if code == 1:
                        newf[k, i] = self.fs[M][self.index[M][c], i]  # Eq.(2) / Eq.(10)
                    else:
                        newf[k, i] = self.bc(L, k, i, code)
                    continue
                # y lies in a level-L cell that is refined (the leaf holding
                # the point itself may be finer than L+1 away from p)
                assert M > L, "2:1 balance violated"
                newf[k, i] = self.coalesce(L, k, p, i)
        self.f[L] = newf

    def coalesce(self, L, k, p, i):
        F = L + 1
        shp = np.array(self.shape[F])
        h = 0.5 ** L
        pts = (self.fluid_and_bc(F) + 0.5 + self.e[i]) * (h / 2)
        n0 = np.array((self.p.nx, self.p.ny, self.p.nz), dtype=np.float64)
        for a in range(3):
            if self.p.periodic[a]:
                pts[:, a] = pts[:, a] % n0[a]
        inside = np.all(np.floor(pts / h).astype(np.int64) == p[None, :], axis=1)
        cells = self.fluid_and_bc(F)[inside]
        codes = self.masks[F][tuple(cells.T)]
        fl = cells[codes == 1]
        if len(fl):
            ids = self.index[F][tuple(fl.T)]
            # Accumulate holds the sum over both fine substeps
            return self.acc[F][ids, i].sum() / (2 * len(fl))
        # every candidate is a BC leaf: first one by offset c = beta - (2p - e_i)
        base = 2 * p - self.e[i]
        offs = (cells - base[None, :]) % shp[None, :]
        order = np.lexsort((offs[:, 2], offs[:, 1], offs[:, 0]))
        return self.bc(L, k, i, int(codes[order[0]]))

    def fluid_and_bc(self, L):
        if not hasattr(self, "_fb"):
            self._fb = {}
        if L not in self._fb:
            self._fb[L] = np.argwhere(self.masks[L] != 0)
        return self._fb[L]

    def collision(self, L):
        self.fs[L] = collide(self.e, self.w, self.f[L], self.omega[L], self.p.collision)
        if L > 0:
            self.acc[L] += self.fs[L]  # Accumulate after every fine Collision

    def nonuniform_time_step(self, L):
        """Algorithm 1."""
        self.collision(L)
        if L != self.Lmax - 1:
            self.nonuniform_time_step(L + 1)
        self.stream(L)  # Explosion(L,L-1) + Streaming(L) + Coalescence(L,L+1)
        if L != self.Lmax - 1:
            self.acc[L + 1][:] = 0.0  # Coalescence resets the accumulator
        if L == 0:
            return
        self.collision(L)
        if L != self.Lmax - 1:
            self.nonuniform_time_step(L + 1)
        self.stream(L)
        if L != self.Lmax - 1:
            self.acc[L + 1][:] = 0.0

    def step(self, n=1):
        for _ in range(n):
            self.nonuniform_time_step(0)

    def macroscopic(self, L):
        rho = np.full(self.shape[L], np.nan)
        u = np.full(self.shape[L] + (3,), np.nan)
        f = self.f[L]
        r = f.sum(1)
        rho[tuple(self.fluid[L].T)] = r
        u[tuple(self.fluid[L].T)] = (f @ self.e) / r[:, None]
        return rho, u
