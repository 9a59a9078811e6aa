"""Thin ctypes binding of liblbmr.so (include/lbmr.h).

Argument marshalling only: every step of the hot path runs in the library's
sm_100a kernels.  There is no CPU fallback: if the library is missing, or no
CUDA device is present when a grid is created, the call raises.
"""
from __future__ import annotations

import ctypes
import os
from typing import Optional, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("LBMR_LIB") or os.path.join(_HERE, "_lib", "liblbmr.so")

LBM_OK = 0
STATUS = {0: "LBM_OK", 1: "LBM_E_INVAL", 2: "LBM_E_TILING", 3: "LBM_E_UNBALANCED", 4: "LBM_E_OOM",
          5: "LBM_E_CUDA", 6: "LBM_E_COMM", 7: "LBM_E_STATE", 8: "LBM_E_UNSUPPORTED"}
D3Q19, D3Q27 = 19, 27
BGK, KBC = 0, 1
FP32, FP64 = 0, 1
BC_NOSLIP, BC_VELOCITY, BC_OUTFLOW = 0, 1, 2
SCHED_FUSED, SCHED_UNFUSED, SCHED_NO_GRAPH = 0, 1, 2
SCHED_SPLIT_E, SCHED_SPLIT_A, SCHED_ATOMIC_A, SCHED_SPLIT_O = 4, 8, 16, 32
SCHED_CTA_GATHER = 64
# the paper's Fig. 4 configurations as schedule bit sets
FIG4 = {
    "4b": SCHED_UNFUSED | SCHED_SPLIT_E | SCHED_SPLIT_A | SCHED_SPLIT_O,  # modified baseline: C, A, S, E, O
    "4c": SCHED_UNFUSED | SCHED_SPLIT_E | SCHED_ATOMIC_A | SCHED_SPLIT_O,  # CA fused (atomic Accumulate)
    "4d": SCHED_UNFUSED | SCHED_SPLIT_A | SCHED_SPLIT_O,  # SE fused
    "4e": SCHED_UNFUSED | SCHED_ATOMIC_A,  # CA, SE and SO fused
    "4f": SCHED_ATOMIC_A,  # CASE and SO fused (the paper's design)
    "product": SCHED_FUSED,  # fused level kernels, warp-cooperative A+A+O gather kernel (deterministic)
    "cta_gather": SCHED_CTA_GATHER,  # A+A+O gathered inside F_L^k by each CTA (no gather kernel)
}
VARIANT_PAPER, VARIANT_VOLUMETRIC = 0, 1


class LBMError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


class GridDesc(ctypes.Structure):
    _fields_ = [
        ("nx", ctypes.c_int32), ("ny", ctypes.c_int32), ("nz", ctypes.c_int32),
        ("periodic", ctypes.c_int32 * 3),
        ("face_bc", ctypes.c_uint8 * 6), ("pad_", ctypes.c_uint8 * 2),
        ("lattice", ctypes.c_int32), ("collision", ctypes.c_int32), ("precision", ctypes.c_int32),
        ("omega0", ctypes.c_double),
        ("n_ranks", ctypes.c_int32), ("rank", ctypes.c_int32),
        ("stream", ctypes.c_void_p),
        ("variant", ctypes.c_int32),
    ]


class GridInfo(ctypes.Structure):
    _fields_ = [
        ("levels", ctypes.c_int32), ("Q", ctypes.c_int32), ("precision", ctypes.c_int32),
        ("kernels_per_step", ctypes.c_int32),
        ("leaves", ctypes.c_int64 * 16), ("blocks", ctypes.c_int64 * 16),
        ("special_blocks", ctypes.c_int64 * 16), ("special_cells", ctypes.c_int64 * 16),
        ("total_blocks", ctypes.c_int64 * 16),
        ("device_bytes", ctypes.c_int64), ("steps_done", ctypes.c_int64),
        ("launches_per_step", ctypes.c_int64),
        ("block_offset", (ctypes.c_int32 * 3) * 16),
        ("coal_links", ctypes.c_int64 * 16), ("coal_wide", ctypes.c_int64 * 16),
    ]


EXPORTS = ["lbm_grid_create", "lbm_set_bc", "lbm_init_equilibrium", "lbm_init_uniform", "lbm_step",
           "lbm_macroscopic", "lbm_stats", "lbm_grid_get_info", "lbm_profile_levels", "lbm_synchronize",
           "lbm_grid_destroy", "lbm_last_error", "lbm_version", "lbm_grid_analyze", "lbm_schedule",
           "lbm_lattice_table", "lbm_omega_level", "lbm_partition_cuts", "lbm_grid_slab", "lbm_halo_export",
           "lbm_halo_connect", "lbm_halo_connect_local", "lbm_halo_plan", "lbm_set_schedule",
           "lbm_checkpoint_size", "lbm_checkpoint_save", "lbm_checkpoint_load", "lbm_probe", "lbm_debug_flags", "lbm_profile_step"]

_lib = None


def load_library(path: str = LIB_PATH):
    """Load liblbmr.so; raises if it is missing (no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise ImportError(f"liblbmr.so not built ({path}); run __graft_entry__.build()")
    lib = ctypes.CDLL(path)
    P = ctypes.c_void_p
    dp = ctypes.POINTER(ctypes.c_double)
    lp = ctypes.POINTER(ctypes.c_int64)
    lib.lbm_grid_create.argtypes = [ctypes.POINTER(GridDesc), ctypes.c_int32, ctypes.POINTER(ctypes.c_void_p),
                                    ctypes.POINTER(P)]
    lib.lbm_set_bc.argtypes = [P, ctypes.c_int32, ctypes.c_int32, dp]
    lib.lbm_init_equilibrium.argtypes = [P, ctypes.c_int32, dp, dp]
    lib.lbm_init_uniform.argtypes = [P, ctypes.c_double, dp]
    lib.lbm_step.argtypes = [P, ctypes.c_int32]
    lib.lbm_macroscopic.argtypes = [P, ctypes.c_int32, dp, dp]
    lib.lbm_stats.argtypes = [P, lp, dp]
    lib.lbm_grid_get_info.argtypes = [P, ctypes.POINTER(GridInfo)]
    lib.lbm_profile_levels.argtypes = [P, ctypes.c_int32, dp, lp]
    lib.lbm_profile_step.argtypes = [P, ctypes.c_int32, dp, dp, lp]
    lib.lbm_synchronize.argtypes = [P]
    lib.lbm_grid_destroy.argtypes = [P]
    lib.lbm_grid_destroy.restype = None
    lib.lbm_grid_analyze.argtypes = [ctypes.POINTER(GridDesc), ctypes.c_int32, ctypes.POINTER(ctypes.c_void_p),
                                     ctypes.POINTER(GridInfo)]
    lib.lbm_schedule.argtypes = [ctypes.c_int32, ctypes.c_int64, lp, ctypes.c_int32]
    lib.lbm_schedule.restype = ctypes.c_int32
    lib.lbm_lattice_table.argtypes = [ctypes.c_int32, ctypes.POINTER(ctypes.c_int32), dp]
    lib.lbm_lattice_table.restype = ctypes.c_int32
    lib.lbm_omega_level.argtypes = [ctypes.c_double, ctypes.c_int32]
    lib.lbm_omega_level.restype = ctypes.c_double
    PP = ctypes.POINTER(ctypes.c_void_p)
    i32p = ctypes.POINTER(ctypes.c_int32)
    lib.lbm_partition_cuts.argtypes = [ctypes.POINTER(GridDesc), ctypes.c_int32, PP, ctypes.c_int32, i32p]
    lib.lbm_grid_slab.argtypes = [P, i32p, i32p]
    lib.lbm_halo_export.argtypes = [P, ctypes.c_int32, ctypes.c_void_p, ctypes.c_int64, lp]
    lib.lbm_halo_connect.argtypes = [P, ctypes.c_int32, ctypes.c_void_p, ctypes.c_int64]
    lib.lbm_halo_connect_local.argtypes = [P, ctypes.c_int32, P]
    lib.lbm_halo_plan.argtypes = [ctypes.POINTER(GridDesc), ctypes.c_int32, PP, ctypes.c_int32, ctypes.c_int32, lp, lp,
                                  ctypes.c_int64, lp, lp]
    lib.lbm_set_schedule.argtypes = [P, ctypes.c_int32]
    lib.lbm_probe.argtypes = [P, ctypes.c_int32, ctypes.c_int64, lp, dp, dp]
    lib.lbm_checkpoint_size.argtypes = [P, lp]
    lib.lbm_checkpoint_save.argtypes = [P, ctypes.c_void_p, ctypes.c_int64]
    lib.lbm_checkpoint_load.argtypes = [P, ctypes.c_void_p, ctypes.c_int64]
    lib.lbm_debug_flags.argtypes = [P, ctypes.POINTER(ctypes.c_ulonglong)]
    lib.lbm_last_error.restype = ctypes.c_char_p
    lib.lbm_version.restype = ctypes.c_char_p
    for name in EXPORTS:
        f = getattr(lib, name)
        if f.restype is ctypes.c_int:
            f.restype = ctypes.c_int
    _lib = lib
    return lib


def _check(st: int):
    if st != LBM_OK:
        raise LBMError(st, _lib.lbm_last_error().decode())


def _dp(a: Optional[np.ndarray]):
    if a is None:
        return None
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_double))


def make_desc(nx, ny, nz, periodic=(0, 0, 0), face_bc=(0,) * 6, lattice=D3Q19, collision=BGK, precision=FP32,
              omega0=1.0, stream=None, n_ranks=1, rank=0, variant=VARIANT_PAPER) -> GridDesc:
    d = GridDesc()
    d.nx, d.ny, d.nz = nx, ny, nz
    for a in range(3):
        d.periodic[a] = int(periodic[a])
    for f in range(6):
        d.face_bc[f] = int(face_bc[f])
    d.lattice, d.collision, d.precision = int(lattice), int(collision), int(precision)
    d.omega0 = float(omega0)
    d.n_ranks, d.rank = int(n_ranks), int(rank)
    d.stream = stream
    d.variant = int(variant)
    return d


def analyze(nx, ny, nz, masks, **kw) -> GridInfo:
    """Host-only validation + block tables (no GPU): returns the grid counts."""
    lib = load_library()
    ms = [np.ascontiguousarray(m, dtype=np.uint8) for m in masks]
    d = make_desc(nx, ny, nz, **kw)
    ptrs = (ctypes.c_void_p * len(ms))(*[m.ctypes.data for m in ms])
    gi = GridInfo()
    _check(lib.lbm_grid_analyze(ctypes.byref(d), len(ms), ptrs, ctypes.byref(gi)))
    return gi


def analyze_problem(prob, precision=FP32) -> GridInfo:
    return analyze(prob.nx, prob.ny, prob.nz, prob.masks, periodic=prob.periodic, face_bc=prob.face_bc,
                   lattice=prob.Q, collision=KBC if prob.collision == "kbc" else BGK, precision=precision,
                   omega0=prob.omega0)


def _mask_ptrs(masks):
    ms = [np.ascontiguousarray(m, dtype=np.uint8) for m in masks]
    return ms, (ctypes.c_void_p * len(ms))(*[m.ctypes.data for m in ms])


def _problem_kw(prob, precision=FP32):
    return dict(periodic=prob.periodic, face_bc=prob.face_bc, lattice=prob.Q,
                collision=KBC if prob.collision == "kbc" else BGK, precision=precision, omega0=prob.omega0)


def partition_cuts(prob, n_ranks: int):
    """Balanced level-0 x cuts (n_ranks + 1 entries), host only."""
    lib = load_library()
    ms, ptrs = _mask_ptrs(prob.masks)
    d = make_desc(prob.nx, prob.ny, prob.nz, **_problem_kw(prob))
    cuts = np.zeros(n_ranks + 1, dtype=np.int32)
    _check(lib.lbm_partition_cuts(ctypes.byref(d), len(ms), ptrs, int(n_ranks),
                                  cuts.ctypes.data_as(ctypes.POINTER(ctypes.c_int32))))
    return [int(c) for c in cuts]


def halo_plan(prob, n_ranks: int, rank: int, side: int, level: int):
    """Global (x, y, z) of the cells rank sends across `side` and of its halo
    cells there, at `level` (host only)."""
    lib = load_library()
    ms, ptrs = _mask_ptrs(prob.masks)
    d = make_desc(prob.nx, prob.ny, prob.nz, n_ranks=n_ranks, rank=rank, **_problem_kw(prob))
    ns, nh = ctypes.c_int64(), ctypes.c_int64()
    lp = ctypes.POINTER(ctypes.c_int64)
    _check(lib.lbm_halo_plan(ctypes.byref(d), len(ms), ptrs, side, level, None, None, 0, ctypes.byref(ns),
                             ctypes.byref(nh)))
    cap = max(ns.value, nh.value, 1)
    a = np.zeros((cap, 3), dtype=np.int64)
    b = np.zeros((cap, 3), dtype=np.int64)
    _check(lib.lbm_halo_plan(ctypes.byref(d), len(ms), ptrs, side, level, a.ctypes.data_as(lp),
                             b.ctypes.data_as(lp), cap, ctypes.byref(ns), ctypes.byref(nh)))
    return a[:ns.value].copy(), b[:nh.value].copy()


def schedule(levels: int, n: int = 0):
    """Pipelined launch order [(L, k), ...] of coarse step n."""
    lib = load_library()
    cap = (1 << levels) + 1
    buf = np.zeros(2 * cap, dtype=np.int64)
    m = lib.lbm_schedule(int(levels), int(n), buf.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)), cap)
    if m < 0:
        raise ValueError("bad levels")
    return [(int(buf[2 * i]), int(buf[2 * i + 1])) for i in range(m)]


def lattice_table(Q: int):
    lib = load_library()
    e = np.zeros(3 * Q, dtype=np.int32)
    w = np.zeros(Q)
    if lib.lbm_lattice_table(Q, e.ctypes.data_as(ctypes.POINTER(ctypes.c_int32)), _dp(w)) != Q:
        raise ValueError("bad Q")
    return e.reshape(Q, 3), w


def omega_level(omega0: float, level: int) -> float:
    return load_library().lbm_omega_level(float(omega0), int(level))


class Grid:
    """A multi-level LBM grid on the current CUDA device (one per rank)."""

    def __init__(self, nx: int, ny: int, nz: int, masks: Sequence[np.ndarray], *, periodic=(0, 0, 0),
                 face_bc=(0, 0, 0, 0, 0, 0), lattice: int = D3Q19, collision: int = BGK,
                 precision: int = FP32, omega0: float = 1.0, stream: Optional[int] = None,
                 n_ranks: int = 1, rank: int = 0, variant: int = VARIANT_PAPER):
        lib = load_library()
        self.lib = lib
        self.shape0 = (nx, ny, nz)
        self.levels = len(masks)
        self._masks = [np.ascontiguousarray(m, dtype=np.uint8) for m in masks]
        for L, m in enumerate(self._masks):
            if m.shape != (nx << L, ny << L, nz << L):
                raise ValueError(f"mask {L} has shape {m.shape}, expected {(nx << L, ny << L, nz << L)}")
        d = make_desc(nx, ny, nz, periodic, face_bc, lattice, collision, precision, omega0, stream, n_ranks, rank,
                      variant)
        self.n_ranks, self.rank = n_ranks, rank
        self._periodic_x = bool(periodic[0])
        ptrs = (ctypes.c_void_p * self.levels)(*[m.ctypes.data for m in self._masks])
        h = ctypes.c_void_p()
        _check(lib.lbm_grid_create(ctypes.byref(d), self.levels, ptrs, ctypes.byref(h)))
        self.h = h
        self._masks = None  # the library copied what it needs

    # -- lifecycle -------------------------------------------------------
    def close(self):
        if getattr(self, "h", None) is not None and self.h.value:
            self.lib.lbm_grid_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    # -- API -----------------------------------------------------------------
    def set_bc(self, cls: int, kind: int, u=(0.0, 0.0, 0.0)):
        u = np.ascontiguousarray(u, dtype=np.float64)
        _check(self.lib.lbm_set_bc(self.h, int(cls), int(kind), _dp(u)))

    def slab(self):
        """Owned level-0 x range [begin, end) (the whole domain on one rank)."""
        a, b = ctypes.c_int32(), ctypes.c_int32()
        _check(self.lib.lbm_grid_slab(self.h, ctypes.byref(a), ctypes.byref(b)))
        return a.value, b.value

    def level_shape(self, L: int):
        """Shape of the dense per-level arrays this grid takes and returns
        (the owned slab on a partitioned grid)."""
        nx, ny, nz = self.shape0
        if self.n_ranks > 1:
            b, e = self.slab()
            nx = e - b
        return (nx << L, ny << L, nz << L)

    def halo_export(self, side: int) -> bytes:
        n = ctypes.c_int64()
        _check(self.lib.lbm_halo_export(self.h, int(side), None, 0, ctypes.byref(n)))
        buf = ctypes.create_string_buffer(n.value)
        _check(self.lib.lbm_halo_export(self.h, int(side), buf, n.value, ctypes.byref(n)))
        return buf.raw

    def halo_connect(self, side: int, blob: bytes):
        _check(self.lib.lbm_halo_connect(self.h, int(side), blob, len(blob)))

    def halo_connect_local(self, side: int, peer: "Grid"):
        _check(self.lib.lbm_halo_connect_local(self.h, int(side), peer.h))

    def init_equilibrium(self, L: int, rho: Optional[np.ndarray] = None, u: Optional[np.ndarray] = None):
        shape = self.level_shape(L)
        r = None if rho is None else np.ascontiguousarray(rho, dtype=np.float64).reshape(shape)
        v = None if u is None else np.ascontiguousarray(u, dtype=np.float64).reshape(shape + (3,))
        _check(self.lib.lbm_init_equilibrium(self.h, int(L), _dp(r), _dp(v)))

    def init_uniform(self, rho0: float = 1.0, u0=(0.0, 0.0, 0.0)):
        u = np.ascontiguousarray(u0, dtype=np.float64)
        _check(self.lib.lbm_init_uniform(self.h, float(rho0), _dp(u)))

    def step(self, n_coarse: int = 1):
        _check(self.lib.lbm_step(self.h, int(n_coarse)))

    def synchronize(self):
        _check(self.lib.lbm_synchronize(self.h))

    def macroscopic(self, L: int):
        shape = self.level_shape(L)
        rho = np.empty(shape)
        u = np.empty(shape + (3,))
        _check(self.lib.lbm_macroscopic(self.h, int(L), _dp(rho), _dp(u)))
        return rho, u

    def probe(self, L: int, xyz):
        """(rho[n], u[n,3]) at GLOBAL level-L cells xyz[n,3]; NaN off this
        rank's fluid leaves."""
        xyz = np.ascontiguousarray(xyz, dtype=np.int64).reshape(-1, 3)
        rho = np.empty(len(xyz))
        u = np.empty((len(xyz), 3))
        _check(self.lib.lbm_probe(self.h, int(L), len(xyz), xyz.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
                                  _dp(rho), _dp(u)))
        return rho, u

    def stats(self):
        leaves = np.zeros(self.levels, dtype=np.int64)
        mass = ctypes.c_double()
        _check(self.lib.lbm_stats(self.h, leaves.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
                                  ctypes.byref(mass)))
        return leaves, mass.value

    def info(self) -> GridInfo:
        gi = GridInfo()
        _check(self.lib.lbm_grid_get_info(self.h, ctypes.byref(gi)))
        return gi

    def set_schedule(self, mode: int):
        """Bit flags SCHED_* (lbmr.h lbm_set_schedule); FIG4 names the paper's
        Fig. 4 configurations."""
        _check(self.lib.lbm_set_schedule(self.h, int(mode)))

    def checkpoint_size(self) -> int:
        n = ctypes.c_int64()
        _check(self.lib.lbm_checkpoint_size(self.h, ctypes.byref(n)))
        return n.value

    def save_checkpoint(self) -> np.ndarray:
        """The grid's state as a host byte array (opaque; see lbmr.h)."""
        buf = np.empty(self.checkpoint_size(), dtype=np.uint8)
        _check(self.lib.lbm_checkpoint_save(self.h, buf.ctypes.data, buf.nbytes))
        return buf

    def load_checkpoint(self, buf: np.ndarray):
        buf = np.ascontiguousarray(buf, dtype=np.uint8)
        _check(self.lib.lbm_checkpoint_load(self.h, buf.ctypes.data, buf.nbytes))

    def debug_flags(self):
        """Halo-protocol counters of a partitioned grid (lbm_debug_flags)."""
        out = (ctypes.c_ulonglong * 4)()
        _check(self.lib.lbm_debug_flags(self.h, out))
        return [int(v) for v in out]

    def profile_step(self, n_coarse: int):
        """(level_ms[L], gather_ms[L], launches[L]) summed over n_coarse
        instrumented coarse steps (lbm_profile_step)."""
        lms = np.zeros(self.levels)
        gms = np.zeros(self.levels)
        cnt = np.zeros(self.levels, dtype=np.int64)
        _check(self.lib.lbm_profile_step(self.h, int(n_coarse), _dp(lms), _dp(gms),
                                         cnt.ctypes.data_as(ctypes.POINTER(ctypes.c_int64))))
        return lms, gms, cnt

    def profile_levels(self, n_coarse: int):
        ms = np.zeros(self.levels)
        cnt = np.zeros(self.levels, dtype=np.int64)
        _check(self.lib.lbm_profile_levels(self.h, int(n_coarse), _dp(ms),
                                           cnt.ctypes.data_as(ctypes.POINTER(ctypes.c_int64))))
        return ms, cnt


def grid_from_problem(prob, precision: int = FP32, stream: Optional[int] = None, init: bool = True,
                      n_ranks: int = 1, rank: int = 0, variant: int = VARIANT_PAPER) -> Grid:
    """Build a Grid from an ``lbm_inputs.Problem`` (masks, BCs, initial state);
    with n_ranks > 1 the grid holds rank's x-slab (connect its halos before
    stepping)."""
    g = Grid(prob.nx, prob.ny, prob.nz, prob.masks, stream=stream, n_ranks=n_ranks, rank=rank, variant=variant,
             **_problem_kw(prob, precision))
    for cls, (kind, u) in prob.bc.items():
        g.set_bc(cls, kind, u)
    if init:
        init_from_problem(g, prob)
    return g


def init_from_problem(g: Grid, prob):
    if prob.init_rho is None and prob.init_u is None:
        g.init_uniform(prob.uniform_rho, prob.uniform_u)
        return
    b, e = g.slab() if g.n_ranks > 1 else (0, prob.nx)
    for L in range(prob.levels):
        rho, u = prob.init_fields(L)
        g.init_equilibrium(L, rho[b << L:e << L], u[b << L:e << L])


class PartitionedGrid:
    """P x-slab grids of one problem in ONE process (emulated multi-GPU on one
    device, or one grid per visible device).  Each slab runs on its own CUDA
    stream; the halo protocol orders the slabs on the device, so stepping is
    just issuing lbm_step on every slab."""

    def __init__(self, prob, n_ranks: int, precision: int = FP32, devices=None):
        import torch
        self.prob, self.P = prob, n_ranks
        self.grids, self.streams = [], []
        for r in range(n_ranks):
            dev = devices[r] if devices else torch.cuda.current_device()
            with torch.cuda.device(dev):
                s = torch.cuda.Stream()
                self.streams.append(s)
                self.grids.append(grid_from_problem(prob, precision, stream=s.cuda_stream, n_ranks=n_ranks, rank=r))
        for r, g in enumerate(self.grids):
            left, right = (r - 1) % n_ranks, (r + 1) % n_ranks
            if g_has(g, 0):
                g.halo_connect_local(0, self.grids[left])
            if g_has(g, 1):
                g.halo_connect_local(1, self.grids[right])

    def step(self, n: int = 1):
        for g in self.grids:
            g.step(n)

    def synchronize(self):
        for g in self.grids:
            g.synchronize()

    def macroscopic(self, L: int):
        parts = [g.macroscopic(L) for g in self.grids]
        return np.concatenate([p[0] for p in parts], axis=0), np.concatenate([p[1] for p in parts], axis=0)

    def close(self):
        # every slab's last kernels may still be storing into a neighbour's
        # buffers: wait for all of them before freeing any
        for g in self.grids:
            if g.h is not None:
                g.synchronize()
        for g in self.grids:
            g.close()


def g_has(g: Grid, side: int) -> bool:
    """Whether partitioned grid g has a neighbour on `side` (0: -x, 1: +x)."""
    b, e = g.slab()
    per = g._periodic_x
    return (b > 0 or per) if side == 0 else (e < g.shape0[0] or per)
