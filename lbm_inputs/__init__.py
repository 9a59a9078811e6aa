"""Seeded synthetic inputs shared by the oracle and the CUDA path.

This module holds NO arithmetic of the method (no equilibrium, collision,
streaming or refinement rule).  It only produces problem descriptions: per-level
uint8 leaf masks, boundary-condition class tables, relaxation parameter ω0 and
initial macroscopic fields.  Both ``oracle/`` and the product binding consume
these descriptions; neither imports the other.

Mask convention (include/lbmr.h): ``masks[L]`` is C-order of shape
``(nx<<L, ny<<L, nz<<L)``; 0 = not a leaf at this level, 1 = fluid leaf,
2..255 = boundary-condition leaf of that class id.

The five BASELINE.json configurations are built exactly as SURVEY.md §8(d)
states them (recipes restated in DESIGN.md §4).
"""
from __future__ import annotations

import dataclasses
from typing import Dict, List, Optional, Sequence, Tuple

import numpy as np

BC_NOSLIP = 0
BC_VELOCITY = 1
BC_OUTFLOW = 2

# conventional class ids used by the configs
CLS_WALL = 2
CLS_LID = 3      # moving wall / velocity inlet
CLS_OUT = 4


@dataclasses.dataclass
class Problem:
    name: str
    nx: int
    ny: int
    nz: int
    masks: List[np.ndarray]
    periodic: Tuple[int, int, int] = (0, 0, 0)
    face_bc: Tuple[int, int, int, int, int, int] = (0, 0, 0, 0, 0, 0)
    Q: int = 19
    collision: str = "bgk"           # "bgk" | "kbc"
    omega0: float = 1.0
    bc: Dict[int, Tuple[int, Tuple[float, float, float]]] = dataclasses.field(default_factory=dict)
    # initial state: per-level dense (rho, u) arrays, or a uniform (rho0, u0)
    init_rho: Optional[List[Optional[np.ndarray]]] = None
    init_u: Optional[List[Optional[np.ndarray]]] = None
    uniform_rho: float = 1.0
    uniform_u: Tuple[float, float, float] = (0.0, 0.0, 0.0)

    @property
    def levels(self) -> int:
        return len(self.masks)

    def level_shape(self, L: int) -> Tuple[int, int, int]:
        return (self.nx << L, self.ny << L, self.nz << L)

    def bc_arrays(self):
        """(kind[256] int32, u[256,3] float64) class table."""
        kind = np.zeros(256, dtype=np.int32)
        u = np.zeros((256, 3), dtype=np.float64)
        for c, (k, uw) in self.bc.items():
            kind[c] = k
            u[c] = uw
        return kind, u

    def fluid_leaves(self) -> List[int]:
        return [int(np.count_nonzero(m == 1)) for m in self.masks]

    def init_fields(self, L: int):
        """Dense (rho, u) initial fields of level L (u interleaved [...,3])."""
        shape = self.level_shape(L)
        if self.init_rho is not None and self.init_rho[L] is not None:
            rho = self.init_rho[L]
        else:
            rho = np.full(shape, self.uniform_rho)
        if self.init_u is not None and self.init_u[L] is not None:
            u = self.init_u[L]
        else:
            u = np.empty(shape + (3,))
            u[...] = np.asarray(self.uniform_u)
        return np.ascontiguousarray(rho, dtype=np.float64), np.ascontiguousarray(u, dtype=np.float64)


# ---------------------------------------------------------------------------
# helpers: masks from a per-level "leaf level" description
# ---------------------------------------------------------------------------

def _box_masks(n: Tuple[int, int, int], boxes: Sequence[Tuple[Tuple[int, int], ...]]) -> List[np.ndarray]:
    """Nested refinement boxes (coarse units).  boxes[k] is the region refined
    to level >= k+1.  Returns per-level masks with 1 on leaves."""
    levels = len(boxes) + 1
    masks = []
    for L in range(levels):
        shape = (n[0] << L, n[1] << L, n[2] << L)
        m = np.zeros(shape, dtype=np.uint8)
        # region covered at level >= L
        if L == 0:
            m[...] = 1
        else:
            (x0, x1), (y0, y1), (z0, z1) = boxes[L - 1]
            m[x0 << L:x1 << L, y0 << L:y1 << L, z0 << L:z1 << L] = 1
        if L < levels - 1:
            (x0, x1), (y0, y1), (z0, z1) = boxes[L]
            m[x0 << L:x1 << L, y0 << L:y1 << L, z0 << L:z1 << L] = 0
        masks.append(m)
    return masks


def _shell_masks(n: int, bounds: Sequence[Tuple[float, float]]) -> List[np.ndarray]:
    """Wall-distance refinement of a cube of n coarse cells: level >= k+1
    outside the cube bounds[k] = (lo, hi) (coarse units, may be half-integer
    multiples of the finer spacing)."""
    levels = len(bounds) + 1
    masks = []
    for L in range(levels):
        N = n << L
        c = (np.arange(N) + 0.5) / (1 << L)  # cell centres, coarse units

        def inside(k):
            lo, hi = bounds[k]
            a = (c > lo) & (c < hi)
            return a[:, None, None] & a[None, :, None] & a[None, None, :]

        if L == 0:
            covered = np.ones((N, N, N), dtype=bool)
        else:
            covered = ~inside(L - 1)
        if L < levels - 1:
            covered &= inside(L)
        masks.append(covered.astype(np.uint8))
    return masks


# ---------------------------------------------------------------------------
# BASELINE.json configurations
# ---------------------------------------------------------------------------

def cavity2(variant: str = "", n: int = 32) -> Problem:
    """cfg1: D3Q19 BGK lid-driven cavity, 32^3 coarse, 2 levels, refined core
    [8,24)^3, +y lid u=(0.05,0,0), other faces no-slip.  Re=100 on 32 coarse
    cells: nu0 = 0.05*32/100 = 0.016, omega0 = 1/(3*nu0 + 1/2) (Eq.4).
    variant "r": rho = 1 + 0.01 xi, u = 0.02 xi_vec, xi ~ U(-1,1), seed 1."""
    q = n // 4
    masks = _box_masks((n, n, n), [((q, 3 * q), (q, 3 * q), (q, 3 * q))])
    p = Problem(
        name="cavity2" + variant, nx=n, ny=n, nz=n, masks=masks,
        periodic=(0, 0, 0),
        face_bc=(CLS_WALL, CLS_WALL, CLS_WALL, CLS_LID, CLS_WALL, CLS_WALL),
        Q=19, collision="bgk", omega0=1.0 / (3 * 0.05 * n / 100.0 + 0.5),
        bc={CLS_WALL: (BC_NOSLIP, (0.0, 0.0, 0.0)), CLS_LID: (BC_VELOCITY, (0.05, 0.0, 0.0))},
    )
    if variant == "r":
        rng = np.random.default_rng(1)
        p.init_rho, p.init_u = [], []
        for L in range(p.levels):
            shape = p.level_shape(L)
            p.init_rho.append(1.0 + 0.01 * rng.uniform(-1, 1, size=shape))
            p.init_u.append(0.02 * rng.uniform(-1, 1, size=shape + (3,)))
    return p


def uniform(n: int = 512, omega: float = 1.0, Q: int = 19, taylor_green: bool = True) -> Problem:
    """cfg2: single-level periodic n^3 box, omega = 1, Taylor-Green initial
    velocity u = 0.05 (sin x cos y cos z, -cos x sin y cos z, 0), rho = 1."""
    masks = [np.ones((n, n, n), dtype=np.uint8)]
    p = Problem(name=f"uniform{n}", nx=n, ny=n, nz=n, masks=masks, periodic=(1, 1, 1),
                Q=Q, collision="bgk", omega0=omega)
    if taylor_green:
        x = 2 * np.pi * (np.arange(n) + 0.5) / n
        sx, cx = np.sin(x), np.cos(x)
        u = np.empty((n, n, n, 3))
        u[..., 0] = 0.05 * sx[:, None, None] * cx[None, :, None] * cx[None, None, :]
        u[..., 1] = -0.05 * cx[:, None, None] * sx[None, :, None] * cx[None, None, :]
        u[..., 2] = 0.0
        p.init_u = [u]
    return p


def sphere3(scale: int = 1, re: float = 3700.0) -> Problem:
    """cfg3: D3Q19 BGK flow past a sphere, coarse 256x128x128 / scale, 3 levels.
    L1 box x[32,160) y,z[24,104); L2 box x[48,112) y,z[40,88) (coarse units,
    divided by scale).  Sphere centre (64,64,64)/scale coarse, R = 32/scale
    finest cells; cells whose centre is inside are no-slip BC leaves.
    -x velocity inlet (0.05,0,0), +x outflow, +-y,+-z no-slip.
    Re = u D / nu_2 => nu_0 = nu_2 / 4, omega0 = 1/(3 nu_0 + 1/2) (Eq.4)."""
    s = scale
    n = (256 // s, 128 // s, 128 // s)
    b1 = ((32 // s, 160 // s), (24 // s, 104 // s), (24 // s, 104 // s))
    b2 = ((48 // s, 112 // s), (40 // s, 88 // s), (40 // s, 88 // s))
    masks = _box_masks(n, [b1, b2])
    f = masks[2]
    R = 32 // s
    cc = (64 // s) * 4
    (x0, x1), (y0, y1), (z0, z1) = [(a * 4, b * 4) for a, b in b2]
    xs = np.arange(x0, x1) + 0.5 - cc
    ys = np.arange(y0, y1) + 0.5 - cc
    zs = np.arange(z0, z1) + 0.5 - cc
    inside = (xs[:, None, None] ** 2 + ys[None, :, None] ** 2 + zs[None, None, :] ** 2) < R * R
    sub = f[x0:x1, y0:y1, z0:z1]
    sub[inside] = CLS_WALL
    D = 2 * R
    nu2 = 0.05 * D / re
    nu0 = nu2 / 4.0
    return Problem(
        name=f"sphere3" + (f"_s{s}" if s != 1 else ""), nx=n[0], ny=n[1], nz=n[2], masks=masks,
        face_bc=(CLS_LID, CLS_OUT, CLS_WALL, CLS_WALL, CLS_WALL, CLS_WALL),
        Q=19, collision="bgk", omega0=1.0 / (3 * nu0 + 0.5),
        bc={CLS_WALL: (BC_NOSLIP, (0.0, 0.0, 0.0)), CLS_LID: (BC_VELOCITY, (0.05, 0.0, 0.0)),
            CLS_OUT: (BC_OUTFLOW, (0.0, 0.0, 0.0))},
        uniform_u=(0.05, 0.0, 0.0),
    )


def cavity4_kbc(size: str = "full", collision: str = "kbc") -> Problem:
    """cfg4: D3Q27 KBC lid-driven cavity, coarse 48^3 (384^3 effective), 4 levels
    by wall distance: level>=1 outside [8,40)^3, >=2 outside [4,44)^3, 3 outside
    [2,46)^3 (coarse units).  +y lid (0.05,0,0), other faces no-slip.
    Re = 1000 on 384 finest cells: nu_3 = 0.0192, nu_0 = nu_3/8.
    size "half": coarse 24^3, bounds [4,20),[2,22),[1,23);
    size "mini": coarse 16^3, bounds [3,13),[2,14),[1,15)."""
    if size == "full":
        n, bounds = 48, [(8, 40), (4, 44), (2, 46)]
    elif size == "half":
        n, bounds = 24, [(4, 20), (2, 22), (1, 23)]
    elif size == "mini":
        n, bounds = 16, [(3, 13), (2, 14), (1, 15)]
    else:
        raise ValueError(size)
    masks = _shell_masks(n, bounds)
    eff = n * 8
    nu3 = 0.05 * eff / 1000.0
    nu0 = nu3 / 8.0
    return Problem(
        name=f"cavity4_{collision}" + ("" if size == "full" else "_" + size), nx=n, ny=n, nz=n,
        masks=masks, face_bc=(CLS_WALL, CLS_WALL, CLS_WALL, CLS_LID, CLS_WALL, CLS_WALL),
        Q=27, collision=collision, omega0=1.0 / (3 * nu0 + 0.5),
        bc={CLS_WALL: (BC_NOSLIP, (0.0, 0.0, 0.0)), CLS_LID: (BC_VELOCITY, (0.05, 0.0, 0.0))},
    )


def tunnel4(scale: int = 1, nu3: float = 0.004) -> Problem:
    """cfg5: D3Q19 BGK airplane-like virtual wind tunnel, coarse 200x105x105
    (1600x840x840 effective; reading R-A20), 4 levels.  Body in finest units:
    fuselage cylinder r=32, axis x in [400,880), centre (y,z)=(420,420); wing
    box x[560,640) y[416,424) z[220,620); no-slip BC leaves.  Refinement boxes
    (coarse units): L1 x[22,138) y[20,85) z[0,105); L2 x[38,122) y[36,69)
    z[15,90); L3 x[46,114) y[44,61) z[23,82).  Inlet/outflow/walls as cfg3;
    nu_3 = 0.004 => nu_0 = nu_3/8.  scale=s divides every length by s (s in
    {1, 5}: s=5 gives a 40x21x21 coarse grid for parity tests); nu3 != 0.004
    gives the same geometry at another viscosity (a lower-Re parity case)."""
    s = scale

    def d(v):
        assert v % s == 0, (v, s)
        return v // s

    n = (d(200), d(105), d(105))
    # boxes in coarse units; for s != 1 round outward (2:1 spacing is preserved)
    def box(x0, x1, y0, y1, z0, z1):
        return ((x0 // s, -(-x1 // s)), (y0 // s, -(-y1 // s)), (z0 // s, -(-z1 // s)))
    b1 = box(22, 138, 20, 85, 0, 105)
    b2 = box(38, 122, 36, 69, 15, 90)
    b3 = box(46, 114, 44, 61, 23, 82)
    masks = _box_masks(n, [b1, b2, b3])
    f = masks[3]
    (x0, x1), (y0, y1), (z0, z1) = [(a * 8, b * 8) for a, b in b3]
    xs = np.arange(x0, x1) + 0.5
    ys = np.arange(y0, y1) + 0.5
    zs = np.arange(z0, z1) + 0.5
    r = 32.0 / s
    cy = cz = 420.0 / s
    disc = ((ys[:, None] - cy) ** 2 + (zs[None, :] - cz) ** 2) < r * r
    fx = (xs >= 400.0 / s) & (xs < 880.0 / s)
    sub = f[x0:x1, y0:y1, z0:z1]
    body = fx[:, None, None] & disc[None, :, :]
    wx = (xs >= 560.0 / s) & (xs < 640.0 / s)
    wy = (ys >= 416.0 / s) & (ys < 424.0 / s)
    wz = (zs >= 220.0 / s) & (zs < 620.0 / s)
    body |= wx[:, None, None] & wy[None, :, None] & wz[None, None, :]
    sub[body] = CLS_WALL
    nu0 = nu3 / 8.0
    return Problem(
        name="tunnel4" + (f"_s{s}" if s != 1 else "") + (f"_nu{nu3:g}" if nu3 != 0.004 else ""),
        nx=n[0], ny=n[1], nz=n[2], masks=masks,
        face_bc=(CLS_LID, CLS_OUT, CLS_WALL, CLS_WALL, CLS_WALL, CLS_WALL),
        Q=19, collision="bgk", omega0=1.0 / (3 * nu0 + 0.5),
        bc={CLS_WALL: (BC_NOSLIP, (0.0, 0.0, 0.0)), CLS_LID: (BC_VELOCITY, (0.05, 0.0, 0.0)),
            CLS_OUT: (BC_OUTFLOW, (0.0, 0.0, 0.0))},
        uniform_u=(0.05, 0.0, 0.0),
    )


def sphere_tab1(size: int = 1, re: float = 4000.0, collision: str = "kbc", Q: int = 27) -> Problem:
    """the paper's Tab. I flow over a sphere (P:L292-300,
    Fig. 8): D3Q27 KBC, 3 levels, virtual wind tunnel of (272, 192, 272) * size
    finest cells (size = 1, 2, 3 are the three rows of Tab. I), i.e. a coarse
    grid of (68, 48, 68) * size.  The paper prints the leaf distribution only
    (finest, middle, coarse = 0.602, 0.296, 0.175 M at size 1, x size^3), not the
    refinement regions; this recipe uses two nested boxes
    (coarse units, x size):  L1 x[4,48) y[8,40) z[17,50);  L2 x[13,40) y[14,33)
    z[24,43), giving 0.607 / 0.294 / 0.175 M leaves at size 1 (+0.8 / -0.8 /
    +0.3 %).  Sphere of radius R = 16 * size finest cells centred at
    (80, 94, 134) * size finest units (cells whose centre is inside are
    no-slip BC leaves).  -x velocity inlet (0.05, 0, 0), +x outflow, +-y, +-z
    no-slip.  Re = u_in R / nu_finest = 4000 (Fig. 8 caption) =>
    nu_0 = nu_2 / 4, omega0 = 1 / (3 nu_0 + 1/2) (Eq.4)."""
    s = int(size)
    if s < 1:
        raise ValueError("size >= 1")
    n = (68 * s, 48 * s, 68 * s)
    b1 = ((4 * s, 48 * s), (8 * s, 40 * s), (17 * s, 50 * s))
    b2 = ((13 * s, 40 * s), (14 * s, 33 * s), (24 * s, 43 * s))
    masks = _box_masks(n, [b1, b2])
    f = masks[2]
    R = 16.0 * s
    cx, cy, cz = 80.0 * s, 94.0 * s, 134.0 * s
    (x0, x1), (y0, y1), (z0, z1) = [(a * 4, b * 4) for a, b in b2]
    xs = np.arange(x0, x1) + 0.5 - cx
    ys = np.arange(y0, y1) + 0.5 - cy
    zs = np.arange(z0, z1) + 0.5 - cz
    inside = (xs[:, None, None] ** 2 + ys[None, :, None] ** 2 + zs[None, None, :] ** 2) < R * R
    f[x0:x1, y0:y1, z0:z1][inside] = CLS_WALL
    nu2 = 0.05 * R / re
    nu0 = nu2 / 4.0
    return Problem(
        name=f"sphere_tab1_s{s}" + ("" if (collision, Q) == ("kbc", 27) else f"_{collision}{Q}"),
        nx=n[0], ny=n[1], nz=n[2], masks=masks,
        face_bc=(CLS_LID, CLS_OUT, CLS_WALL, CLS_WALL, CLS_WALL, CLS_WALL),
        Q=Q, collision=collision, omega0=1.0 / (3 * nu0 + 0.5),
        bc={CLS_WALL: (BC_NOSLIP, (0.0, 0.0, 0.0)), CLS_LID: (BC_VELOCITY, (0.05, 0.0, 0.0)),
            CLS_OUT: (BC_OUTFLOW, (0.0, 0.0, 0.0))},
        uniform_u=(0.05, 0.0, 0.0),
    )


# Tab. I: leaves (finest, middle, coarse) in millions and the
# paper's A100 fp64 MLUPS of its modified baseline (Fig. 4b) and optimised
# (Fig. 4f) implementations — context for bench.py's vs_baseline.
TAB1 = {
    1: dict(leaves_M=(0.602, 0.296, 0.175), baseline_mlups=482.63, ours_mlups=1081.67),
    2: dict(leaves_M=(4.81, 2.37, 1.40), baseline_mlups=1115.80, ours_mlups=1646.37),
    3: dict(leaves_M=(16.25, 8.0, 4.74), baseline_mlups=1299.7, ours_mlups=1805.03),
}


CONFIGS = {
    "cavity2": cavity2,
    "uniform512": uniform,
    "sphere3": sphere3,
    "cavity4_kbc": cavity4_kbc,
    "tunnel4": tunnel4,
    "sphere_tab1": sphere_tab1,
}


# ---------------------------------------------------------------------------
# random strong-2:1 grids for brute-force and parity tests
# ---------------------------------------------------------------------------

def _neighbour_max(a: np.ndarray, periodic: Sequence[int]) -> np.ndarray:
    """max over the 26-neighbourhood (and self) of an integer field."""
    out = a.copy()
    for ax in range(3):
        if periodic[ax]:
            lo = np.roll(out, 1, axis=ax)
            hi = np.roll(out, -1, axis=ax)
        else:
            lo = out.copy()
            hi = out.copy()
            sl = [slice(None)] * 3
            sl2 = [slice(None)] * 3
            sl[ax] = slice(1, None)
            sl2[ax] = slice(None, -1)
            lo[tuple(sl)] = out[tuple(sl2)]
            hi[tuple(sl2)] = out[tuple(sl)]
        out = np.maximum(out, np.maximum(lo, hi))
    return out


def random_balanced(seed: int, n=(4, 4, 4), levels: int = 3, p_refine: float = 0.35,
                    p_bc: float = 0.06, periodic=None, Q: int = 19, collision: str = "bgk",
                    omega0: Optional[float] = None, random_init: bool = True) -> Problem:
    """Random strong-2:1 balanced multi-level grid with random BC leaves.

    Built on the finest-resolution "leaf level" field: random leaves are
    refined level by level and the 26-neighbour 2:1 rule is enforced by
    refining the coarser side until stable.  BC classes: 2 no-slip,
    3 moving wall u=(0.03,-0.02,0.01), 4 outflow.
    """
    rng = np.random.default_rng(seed)
    if periodic is None:
        periodic = tuple(int(v) for v in rng.integers(0, 2, size=3))
    F = levels - 1
    fshape = (n[0] << F, n[1] << F, n[2] << F)
    lev = np.zeros(fshape, dtype=np.int32)

    def coarse_view(field, L):
        # reshape finest field into level-L cells x (2^(F-L))^3 sub-cells
        k = 1 << (F - L)
        return field.reshape(n[0] << L, k, n[1] << L, k, n[2] << L, k)

    for L in range(levels - 1):
        # leaves at level L: cells whose whole region has lev == L
        v = coarse_view(lev, L)
        is_leaf = (v.min(axis=(1, 3, 5)) == L) & (v.max(axis=(1, 3, 5)) == L)
        # only refine leaves with no coarser 26-neighbour (keeps the mix of
        # levels; the balance loop below then only repairs corner cases)
        lowest = -_neighbour_max(-lev, periodic)
        safe = coarse_view(lowest, L).min(axis=(1, 3, 5)) >= L
        pick = is_leaf & safe & (rng.random(is_leaf.shape) < p_refine)
        k = 1 << (F - L)
        up = np.repeat(np.repeat(np.repeat(pick, k, 0), k, 1), k, 2)
        lev[up] = L + 1
        # enforce strong 2:1 balance: a cell's level must be >= max(neighbours)-1
        while True:
            need = _neighbour_max(lev, periodic) - 1
            bad = lev < need
            if not bad.any():
                break
            # refine whole leaves of the offending cells by one level
            for M in range(levels - 1):
                vM = coarse_view(lev, M)
                badM = coarse_view(bad, M).any(axis=(1, 3, 5))
                leafM = (vM.min(axis=(1, 3, 5)) == M) & (vM.max(axis=(1, 3, 5)) == M)
                sel = badM & leafM
                if sel.any():
                    kk = 1 << (F - M)
                    upM = np.repeat(np.repeat(np.repeat(sel, kk, 0), kk, 1), kk, 2)
                    lev[upM] = M + 1
    masks = []
    for L in range(levels):
        v = coarse_view(lev, L)
        leaf = (v.min(axis=(1, 3, 5)) == L) & (v.max(axis=(1, 3, 5)) == L)
        m = leaf.astype(np.uint8)
        bcsel = leaf & (rng.random(leaf.shape) < p_bc)
        cls = rng.integers(2, 5, size=leaf.shape).astype(np.uint8)
        m[bcsel] = cls[bcsel]
        masks.append(m)
    face = tuple(int(c) for c in rng.integers(2, 5, size=6))
    if omega0 is None:
        omega0 = float(rng.uniform(0.6, 1.8))
    p = Problem(
        name=f"random{seed}", nx=n[0], ny=n[1], nz=n[2], masks=masks, periodic=tuple(periodic),
        face_bc=face, Q=Q, collision=collision, omega0=omega0,
        bc={CLS_WALL: (BC_NOSLIP, (0.0, 0.0, 0.0)), CLS_LID: (BC_VELOCITY, (0.03, -0.02, 0.01)),
            CLS_OUT: (BC_OUTFLOW, (0.0, 0.0, 0.0))},
    )
    if random_init:
        p.init_rho, p.init_u = [], []
        for L in range(levels):
            shape = p.level_shape(L)
            p.init_rho.append(1.0 + 0.01 * rng.uniform(-1, 1, size=shape))
            p.init_u.append(0.02 * rng.uniform(-1, 1, size=shape + (3,)))
    return p


def planar_slab(levels: int = 2, n=(16, 8, 8), Q: int = 19, collision: str = "bgk",
                omega0: float = 1.2, seed: int = 7) -> Problem:
    """Fully periodic box refined in planar slabs along x (interfaces are planes
    normal to x): level >= k+1 for coarse x in [2+2k, n0-2-2k)."""
    boxes = []
    for k in range(levels - 1):
        boxes.append(((2 + 2 * k, n[0] - 2 - 2 * k), (0, n[1]), (0, n[2])))
    masks = _box_masks(n, boxes)
    p = Problem(name=f"slab{levels}", nx=n[0], ny=n[1], nz=n[2], masks=masks, periodic=(1, 1, 1),
                Q=Q, collision=collision, omega0=omega0)
    rng = np.random.default_rng(seed)
    p.init_rho, p.init_u = [], []
    for L in range(levels):
        shape = p.level_shape(L)
        p.init_rho.append(1.0 + 0.01 * rng.uniform(-1, 1, size=shape))
        p.init_u.append(0.03 * rng.uniform(-1, 1, size=shape + (3,)))
    return p


def refined_box(levels: int = 2, n=(8, 8, 8), Q: int = 19, collision: str = "bgk",
                omega0: float = 1.3, periodic=(1, 1, 1)) -> Problem:
    """Periodic box with a nested refined cube in the middle (interface edges
    and corners)."""
    boxes = []
    for k in range(levels - 1):
        lo, hi = 2 + k, n[0] - 2 - k
        boxes.append(((lo, hi), (lo, hi), (lo, hi)))
    masks = _box_masks(n, boxes)
    return Problem(name=f"box{levels}", nx=n[0], ny=n[1], nz=n[2], masks=masks, periodic=tuple(periodic),
                   Q=Q, collision=collision, omega0=omega0)


def couette(levels: int = 1, H: int = 16, n_xz: int = 8, U: float = 0.02, omega0: float = 1.0,
            both_walls: bool = True) -> Problem:
    """Plane Couette flow: periodic in x and z, no-slip at -y, moving wall
    u=(U,0,0) at +y.  Refined wall layers (planar): level >= k+1 for coarse y
    within w_k = 2 (levels-1-k) coarse cells of a wall (both walls, or the
    bottom wall only), so the finest level touches the wall."""
    masks = []
    for L in range(levels):
        shape = (n_xz << L, H << L, n_xz << L)
        y = (np.arange(H << L) + 0.5) / (1 << L)  # coarse units
        lev_of_y = np.zeros_like(y, dtype=int)
        for k in range(levels - 1):
            lo, hi = 2 * (levels - 1 - k), H - 2 * (levels - 1 - k)
            if both_walls:
                lev_of_y[(y < lo) | (y > hi)] = k + 1
            else:
                lev_of_y[y < lo] = k + 1
        m = np.zeros(shape, dtype=np.uint8)
        m[:, lev_of_y == L, :] = 1
        masks.append(m)
    return Problem(name=f"couette{levels}", nx=n_xz, ny=H, nz=n_xz, masks=masks, periodic=(1, 0, 1),
                   face_bc=(CLS_WALL, CLS_WALL, CLS_WALL, CLS_LID, CLS_WALL, CLS_WALL),
                   Q=19, collision="bgk", omega0=omega0,
                   bc={CLS_WALL: (BC_NOSLIP, (0.0, 0.0, 0.0)), CLS_LID: (BC_VELOCITY, (U, 0.0, 0.0))})
