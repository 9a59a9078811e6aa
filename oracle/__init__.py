"""fp64 CPU oracle for multi-level grid-refinement LBM (TEST INFRASTRUCTURE).

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` legs may import this package.  The product path
(``paper_conf_ipps_mahmoudsm24_b200``) never does, and this package never
imports the product.  Both consume problem descriptions from ``lbm_inputs``.

``Oracle`` wraps ``liboracle.so`` (compiled from ``lbm_oracle.cpp``: the
literal Algorithm 1 recursion).  ``brute`` is an independent numpy
per-link point-location definition for tiny grids.
See the header of lbm_oracle.cpp for the per-function pin status.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "lbm_oracle.cpp")
_LIB = os.path.join(_HERE, "liboracle.so")

_lib = None


def build(force: bool = False) -> str:
    """Compile liboracle.so with g++ (OpenMP).  Building is not using it."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        cmd = ["g++", "-O2", "-std=c++17", "-fopenmp", "-fPIC", "-shared", "-o", _LIB, _SRC]
        subprocess.check_call(cmd)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        # ORACLE_LIB: a separately built copy (tools/mutation_test.py loads
        # deliberately mutated oracles to show that the pins catch them)
        path = os.environ.get("ORACLE_LIB")
        if not path:
            path = build()
        lib = ctypes.CDLL(path)
        P = ctypes.c_void_p
        dp = ctypes.POINTER(ctypes.c_double)
        ip = ctypes.POINTER(ctypes.c_int)
        lib.ora_lattice.argtypes = [ctypes.c_int, ip, dp, ip]
        lib.ora_lattice.restype = ctypes.c_int
        lib.ora_omega_level.argtypes = [ctypes.c_double, ctypes.c_int]
        lib.ora_omega_level.restype = ctypes.c_double
        lib.ora_collide_cell.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_double, dp, dp, ctypes.c_int]
        lib.ora_equilibrium.argtypes = [ctypes.c_int, ctypes.c_double, dp, dp]
        lib.ora_create.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                   ctypes.POINTER(ctypes.c_void_p), ip, ctypes.POINTER(ctypes.c_uint8),
                                   ctypes.c_int, ctypes.c_int, ctypes.c_double, ip, dp,
                                   ctypes.c_char_p, ctypes.c_int]
        lib.ora_create.restype = P
        lib.ora_destroy.argtypes = [P]
        lib.ora_force_gamma2.argtypes = [P, ctypes.c_int]
        lib.ora_set_variant.argtypes = [P, ctypes.c_int]
        lib.ora_num_leaves.argtypes = [P, ctypes.c_int]
        lib.ora_num_leaves.restype = ctypes.c_int64
        lib.ora_init_equilibrium.argtypes = [P, ctypes.c_int, dp, dp]
        lib.ora_init_uniform.argtypes = [P, ctypes.c_double, dp]
        lib.ora_step.argtypes = [P, ctypes.c_int]
        lib.ora_macroscopic.argtypes = [P, ctypes.c_int, dp, dp]
        lib.ora_get_f.argtypes = [P, ctypes.c_int, dp]
        lib.ora_probe.argtypes = [P, ctypes.c_int, ctypes.c_int64, ctypes.POINTER(ctypes.c_int64), dp, dp]
        lib.ora_set_f.argtypes = [P, ctypes.c_int, dp]
        _lib = lib
    return _lib


def _dp(a):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_double))


def lattice(Q: int):
    """(e[Q,3] int, w[Q], opp[Q]) in the oracle's own direction order."""
    lib = _load()
    e = np.zeros(Q * 3, dtype=np.int32)
    w = np.zeros(Q)
    opp = np.zeros(Q, dtype=np.int32)
    lib.ora_lattice(Q, e.ctypes.data_as(ctypes.POINTER(ctypes.c_int)), _dp(w),
                    opp.ctypes.data_as(ctypes.POINTER(ctypes.c_int)))
    return e.reshape(Q, 3), w, opp


def omega_level(omega0: float, L: int) -> float:
    return _load().ora_omega_level(float(omega0), int(L))


def collide_cell(Q: int, collision: str, omega: float, f, force_gamma2: bool = False):
    lib = _load()
    f = np.ascontiguousarray(f, dtype=np.float64)
    out = np.zeros(Q)
    lib.ora_collide_cell(Q, 1 if collision == "kbc" else 0, float(omega), _dp(f), _dp(out), int(force_gamma2))
    return out


def equilibrium(Q: int, rho: float, u):
    lib = _load()
    u = np.ascontiguousarray(u, dtype=np.float64)
    out = np.zeros(Q)
    lib.ora_equilibrium(Q, float(rho), _dp(u), _dp(out))
    return out


class Oracle:
    """The oracle grid for one ``lbm_inputs.Problem``."""

    def __init__(self, prob, init: bool = True):
        lib = _load()
        self.lib = lib
        self.prob = prob
        self.Q = prob.Q
        self._masks = [np.ascontiguousarray(m, dtype=np.uint8) for m in prob.masks]
        ptrs = (ctypes.c_void_p * len(self._masks))(*[m.ctypes.data for m in self._masks])
        per = (ctypes.c_int * 3)(*[int(v) for v in prob.periodic])
        face = (ctypes.c_uint8 * 6)(*[int(v) for v in prob.face_bc])
        kind, u = prob.bc_arrays()
        err = ctypes.create_string_buffer(256)
        h = lib.ora_create(prob.nx, prob.ny, prob.nz, prob.levels, ptrs, per, face, prob.Q,
                           1 if prob.collision == "kbc" else 0, float(prob.omega0),
                           kind.ctypes.data_as(ctypes.POINTER(ctypes.c_int)), _dp(u), err, 256)
        if not h:
            raise ValueError("oracle: " + err.value.decode())
        self.h = ctypes.c_void_p(h)
        if init:
            if prob.init_rho is None and prob.init_u is None:
                u0 = np.ascontiguousarray(prob.uniform_u, dtype=np.float64)
                lib.ora_init_uniform(self.h, float(prob.uniform_rho), _dp(u0))
            else:
                for L in range(prob.levels):
                    rho, uu = prob.init_fields(L)
                    self.init_equilibrium(L, rho, uu)

    def __del__(self):
        h = getattr(self, "h", None)
        if h is not None and h.value:
            self.lib.ora_destroy(h)
            self.h = None

    def set_variant(self, variant: str):
        """"paper" (default) or "volumetric" (ghost advection)."""
        self.lib.ora_set_variant(self.h, {"paper": 0, "volumetric": 1}[variant])

    def force_gamma2(self, on: bool = True):
        self.lib.ora_force_gamma2(self.h, int(on))

    def num_leaves(self, L: int) -> int:
        return int(self.lib.ora_num_leaves(self.h, L))

    def init_equilibrium(self, L, rho=None, u=None):
        r = None if rho is None else np.ascontiguousarray(rho, dtype=np.float64)
        v = None if u is None else np.ascontiguousarray(u, dtype=np.float64)
        self.lib.ora_init_equilibrium(self.h, L, _dp(r) if r is not None else None,
                                      _dp(v) if v is not None else None)

    def step(self, n: int = 1):
        self.lib.ora_step(self.h, int(n))

    def macroscopic(self, L: int):
        shape = self.prob.level_shape(L)
        rho = np.empty(shape)
        u = np.empty(shape + (3,))
        self.lib.ora_macroscopic(self.h, L, _dp(rho), _dp(u))
        return rho, u

    def probe(self, L: int, xyz):
        """(rho[n], u[n,3]) at level-L cells xyz[n,3]; NaN off fluid leaves."""
        xyz = np.ascontiguousarray(xyz, dtype=np.int64).reshape(-1, 3)
        rho = np.empty(len(xyz))
        u = np.empty((len(xyz), 3))
        self.lib.ora_probe(self.h, L, len(xyz), xyz.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)), _dp(rho), _dp(u))
        return rho, u

    def get_f(self, L: int):
        shape = self.prob.level_shape(L)
        out = np.empty(shape + (self.Q,))
        self.lib.ora_get_f(self.h, L, _dp(out))
        return out

    def set_f(self, L: int, f):
        f = np.ascontiguousarray(f, dtype=np.float64)
        self.lib.ora_set_f(self.h, L, _dp(f))
