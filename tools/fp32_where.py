"""Where the fp32 trajectory departs from fp64 (diagnostic, run under gpurun):
the CUDA path in fp32 and fp64 on one problem, n coarse steps; per level the
largest |u32 - u64| (normalised like tests/_parity.py: by the field maximum of
|u| over all levels), its cell and |u| there, and the error histogram by the
cell's distance to the nearest non-fluid cell.
  python tools/fp32_where.py [problem=tunnel4_s5] [steps=100]
"""
import os
import sys

sys.path.insert(0, os.getcwd())
import numpy as np  # noqa: E402


def main():
    from tools.parity_growth import PROBLEMS
    from paper_conf_ipps_mahmoudsm24_b200 import lbmr
    from scipy import ndimage
    name = sys.argv[1] if len(sys.argv) > 1 else "tunnel4_s5"
    steps = [int(s) for s in sys.argv[2:]] or [25, 50, 100]
    prob = PROBLEMS[name]()
    gs = {p: lbmr.grid_from_problem(prob, precision=p) for p in (lbmr.FP32, lbmr.FP64)}
    done = 0
    for n in steps:
        for g in gs.values():
            g.step(n - done)
        done = n
        out = {p: [g.macroscopic(L) for L in range(prob.levels)] for p, g in gs.items()}
        umax = max(np.nanmax(np.abs(u)) for _, u in out[lbmr.FP64])
        print(f"== {name} after {n} coarse steps, |u|max {umax:.4g}")
        for L in range(prob.levels):
            r32, u32 = out[lbmr.FP32][L]
            r64, u64 = out[lbmr.FP64][L]
            e = np.abs(u32 - u64).max(axis=-1) / umax if u32.ndim == 4 else np.abs(u32 - u64) / umax
            fluid = ~np.isnan(r64)
            if not fluid.any():
                continue
            e = np.where(fluid, e, 0.0)
            i = np.unravel_index(np.argmax(e), e.shape)
            dist = ndimage.distance_transform_cdt(fluid, metric="chessboard")
            sp = np.linalg.norm(u64[i]) if u64.ndim == 4 else abs(u64[i])
            print(f"  L{L}: max err {e[i]:.3e} at {tuple(int(x) for x in i)} |u| {sp:.4g} dist-to-nonfluid {dist[i]}"
                  f"  shape {e.shape}")
            for d in (1, 2, 3, 5, 8):
                m = fluid & (dist == d) if d < 8 else fluid & (dist >= d)
                if m.any():
                    print(f"      dist {'>=' if d == 8 else '=='}{d}: max {e[m].max():.3e} mean {e[m].mean():.3e}"
                          f" cells {int(m.sum())}")


if __name__ == "__main__":
    main()
