"""Where does the e2e step's host time go? (per-step wall clock of set_bc / step / probe)"""
import sys, time
sys.path.insert(0, '.')
import numpy as np
import torch
import lbm_inputs as I
from paper_conf_ipps_mahmoudsm24_b200 import lbmr

prob = I.tunnel4()
stream = torch.cuda.Stream()
g = lbmr.grid_from_problem(prob, precision=lbmr.FP32, stream=stream.cuda_stream)
g.step(5); g.synchronize()
u_in = prob.bc.get(I.CLS_LID, (1, (0.0, 0.0, 0.0)))[1]
Lf = prob.levels - 1
fl = np.flatnonzero(prob.masks[Lf] == 1)
pick = np.random.default_rng(3).choice(fl, size=4096, replace=False)
probes = np.stack(np.unravel_index(pick, prob.masks[Lf].shape), axis=1).astype(np.int64)
N = 30
def run(label, fn):
    g.synchronize(); t0 = time.perf_counter()
    for _ in range(N): fn()
    g.synchronize(); dt = (time.perf_counter() - t0) / N
    print(f"{label:40s} {dt*1e3:8.3f} ms/step", flush=True)
run("step only (async)", lambda: g.step(1))
run("step + synchronize", lambda: (g.step(1), g.synchronize()))
run("set_bc + step + sync", lambda: (g.set_bc(I.CLS_LID, lbmr.BC_VELOCITY, u_in), g.step(1), g.synchronize()))
run("step + probe", lambda: (g.step(1), g.probe(Lf, probes)))
run("set_bc + step + probe (bench e2e)", lambda: (g.set_bc(I.CLS_LID, lbmr.BC_VELOCITY, u_in), g.step(1), g.probe(Lf, probes)))
t0 = time.perf_counter()
for _ in range(N): g.probe(Lf, probes)
print("probe alone", (time.perf_counter() - t0) / N * 1e3, "ms")
