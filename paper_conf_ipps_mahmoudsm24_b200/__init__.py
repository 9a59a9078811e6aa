"""B200-native multi-level grid-refinement LBM (Mahmoud et al., IPDPS 2024).

The hot path lives in ``_lib/liblbmr.so`` (C ABI, include/lbmr.h; sm_100a
kernels in csrc/).  ``lbmr`` is the thin ctypes binding.
"""
from . import lbmr  # noqa: F401
from .lbmr import Grid, LBMError, grid_from_problem, load_library  # noqa: F401

__all__ = ["lbmr", "Grid", "LBMError", "grid_from_problem", "load_library"]
