#!/usr/bin/env python
"""Benchmark: MLUPS (fine-equivalent) of the multi-level LBM coarse step on B200.

Default workload: BASELINE configs[4] / SURVEY cfg5 "tunnel4" — D3Q19 BGK,
4 levels, 200x105x105 coarse = 1600x840x840 finest-equivalent, fp32 (shifted
populations), the configuration the metric's 1/2/4/8-GPU target is quoted on
(it fits one B200: 7.3 GB of populations).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                  [--config tunnel4|sphere3|cavity4_kbc|uniform512|cavity2]

MLUPS = sum_L V_L 2^L K / T[us] (reading R-A13), V_L = fluid leaves of
level L.  T is measured with CUDA events on the grid's stream around K graph
replays (inputs resident in HBM; the 7.3 GB working set exceeds the 126 MB L2,
so no flush is needed), max over ranks.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import lbm_inputs as I  # noqa: E402

METRIC = "MLUPS (fine-equivalent) per step at 1/2/4/8 B200 and % of HBM roofline"

CONFIGS = {
    "tunnel4": (lambda: I.tunnel4(), "cfg5 tunnel4: D3Q19 BGK, 4 levels, 200x105x105 coarse (1600x840x840 eff.)"),
    "sphere3": (lambda: I.sphere3(), "cfg3 sphere3: D3Q19 BGK, 3 levels, 256x128x128 coarse, Re=3700"),
    "cavity4_kbc": (lambda: I.cavity4_kbc(), "cfg4 cavity4: D3Q27 KBC, 4 levels, 384^3 effective"),
    "cavity4_bgk": (lambda: I.cavity4_kbc(collision="bgk"), "cfg4 geometry with D3Q27 BGK (KBC cost reference)"),
    "uniform512": (lambda: I.uniform(512), "cfg2 uniform512: D3Q19 BGK, single level 512^3 periodic"),
    "cavity2": (lambda: I.cavity2(), "cfg1 cavity2: D3Q19 BGK, 2 levels, 32^3 coarse"),
}
# the paper's Tab. I sphere sweep (D3Q27 KBC, 3 levels, fp64 like the paper)
for _s in (1, 2, 3):
    CONFIGS[f"sphere_tab1_s{_s}"] = (
        (lambda s=_s: I.sphere_tab1(s)),
        f"Tab. I sphere row {_s}: D3Q27 KBC, 3 levels, {272 * _s}x{192 * _s}x{272 * _s} finest-equivalent, Re=4000")
DEFAULT_PRECISION = {f"sphere_tab1_s{_s}": "fp64" for _s in (1, 2, 3)}
# the paper's own number for exactly this metric and workload (A100, fp64), Tab. I
PAPER_MLUPS = {f"sphere_tab1_s{_s}": I.TAB1[_s]["ours_mlups"] for _s in (1, 2, 3)}
# lbm_set_schedule bit sets (lbmr.h): the product, the C/S split, the graph-free
# launch path, and the paper's Fig. 4 fusion configurations (lbmr.FIG4)
SCHEDULES = {"fused": 0, "unfused": 1, "nograph": 2, "unfused_nograph": 3,
             "fig4b": 1 | 4 | 8 | 32, "fig4c": 1 | 4 | 16 | 32, "fig4d": 1 | 8 | 32, "fig4e": 1 | 16, "fig4f": 16,
             "cta_gather": 64}  # A+A+O gathered inside F_L^k by each CTA (no gather kernel)
N_PROBE = 4096  # e2e monitoring cells
# bounded oracle sample for --impl reference (one coarse step per timed step)
REF_SAMPLE = {
    "tunnel4": (lambda: I.tunnel4(scale=5), "tunnel4 geometry at 1/5 scale (40x21x21 coarse, 4 levels)"),
    "sphere3": (lambda: I.sphere3(scale=4), "sphere3 geometry at 1/4 scale (64x32x32 coarse, 3 levels)"),
    "cavity4_kbc": (lambda: I.cavity4_kbc("mini"), "cavity4 KBC at 16^3 coarse, 4 levels"),
    "cavity4_bgk": (lambda: I.cavity4_kbc("mini", collision="bgk"), "cavity4 geometry D3Q27 BGK at 16^3 coarse"),
    "uniform512": (lambda: I.uniform(64), "uniform periodic 64^3"),
    "cavity2": (lambda: I.cavity2(), "cavity2 (full size)"),
}
for _s in (1, 2, 3):
    REF_SAMPLE[f"sphere_tab1_s{_s}"] = (lambda: I.sphere_tab1(1), "Tab. I sphere row 1 (272x192x272 finest-equivalent)")


def updates_per_step(leaves):
    return sum(int(v) << L for L, v in enumerate(leaves))


def peak_hbm():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""

    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, device_index: int):
        self.proc = None
        self.dev = device_index

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.dev), f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                 "-lms", "50"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.proc = None
        time.sleep(0.3)

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.1)
        self.proc.terminate()
        out, _ = self.proc.communicate(timeout=10)
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in out.strip().splitlines():
            parts = [p.strip() for p in line.split(",")]
            if len(parts) < 7:
                continue
            try:
                sm.append(float(parts[0]))
                mx = float(parts[1])
            except ValueError:
                continue
            for n, v in zip(names, parts[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        load = [s for s in sm if mx and s > 0.5 * mx] or sm
        return {"sm_mhz": statistics.median(load) if load else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm)}


def dist_setup():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def run_reference(args, ws, rank):
    """The oracle (fp64 CPU) as it stands, timed on the host cores."""
    import oracle
    if rank != 0:
        return
    build_fn, sample = REF_SAMPLE[args.config]
    prob = build_fn()
    o = oracle.Oracle(prob)
    upd = updates_per_step(prob.fluid_leaves())
    for _ in range(args.warmup):
        o.step(1)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        o.step(1)
    dt = time.perf_counter() - t0
    value = upd * args.steps / (dt * 1e6)
    cores = len(os.sched_getaffinity(0))
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "MLUPS", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt * 1e3 / args.steps,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
        "data": "synthetic", "config": {"workload": CONFIGS[args.config][1], "sample": sample},
        "cpu_baseline": {"value": value, "unit": "MLUPS", "cores": cores, "kind": "oracle",
                         "sample": f"{sample}; one oracle coarse step per timed step"},
        "e2e": {"value": value, "unit": "MLUPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def cpu_baseline(prob):
    """Oracle (as it stands) on the same workload, one coarse step, host cores."""
    import oracle
    o = oracle.Oracle(prob)
    t0 = time.perf_counter()
    o.step(1)
    dt = time.perf_counter() - t0
    del o
    upd = updates_per_step(prob.fluid_leaves())
    return {"value": upd / (dt * 1e6), "unit": "MLUPS", "cores": len(os.sched_getaffinity(0)), "kind": "oracle",
            "sample": "one coarse step of the same workload (fp64 C++ OpenMP oracle, literal Alg.1)",
            "seconds": dt}


def lib_build_id():
    """sha256 prefix of the liblbmr.so this run loads (labels measurements
    taken from another process, e.g. the ncu traffic capture)."""
    import hashlib
    from paper_conf_ipps_mahmoudsm24_b200 import lbmr
    with open(lbmr.LIB_PATH, "rb") as f:
        return hashlib.sha256(f.read()).hexdigest()[:16]


def level_profile(g, prob, prec, lbmr, profile_steps, leaves_local):
    """Per-level device time of the level kernels (lbm_profile_step: the
    coarse step captured into an instrumented CUDA graph with event nodes
    around every level kernel and its coalescence gather, so no host launch
    gaps are timed) and the roofline object of the dominant kernel.  `frac`
    is the level kernel's own; `frac_incl_gather` charges the level with the
    gather kernel that feeds it."""
    ms_lvl, gather_ms, cnt_lvl = g.profile_step(profile_steps)
    tsz = 4 if prec == lbmr.FP32 else 8
    bpu = 2 * prob.Q * tsz
    dom = int(np.argmax(ms_lvl))
    per_launch_ms = ms_lvl[dom] / max(cnt_lvl[dom], 1)
    achieved = leaves_local[dom] * bpu / (per_launch_ms * 1e-3) / 1e9
    peak, peak_src = peak_hbm()
    per_level = []
    for L in range(prob.levels):
        pl = ms_lvl[L] / max(cnt_lvl[L], 1)
        gbs = leaves_local[L] * bpu / (pl * 1e-3) / 1e9 if pl > 0 else None
        gl = gather_ms[L] / max(cnt_lvl[L], 1)
        per_level.append({"level": L, "leaves": leaves_local[L], "launches": int(cnt_lvl[L]), "ms_per_launch": pl,
                          "GBs": gbs, "frac": gbs / peak if gbs else None,
                          "gather_ms_per_launch": gl,
                          "frac_incl_gather": leaves_local[L] * bpu / ((pl + gl) * 1e-3) / 1e9 / peak if pl > 0 else None,
                          "share_of_step": (ms_lvl[L] + gather_ms[L]) / max(ms_lvl.sum() + gather_ms.sum(), 1e-12)})
    roof = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
            "kernel": f"level_step L{dom}", "bytes_per_update": bpu, "peak_source": peak_src,
            "algorithmic_bytes_per_launch": leaves_local[dom] * bpu, "ms_per_launch": per_launch_ms}
    return roof, per_level, dom


def ncu_traffic(config, precision, levels, timeout=240):
    """DRAM bytes (dram__bytes_read.sum + dram__bytes_write.sum) of one launch
    of the dominant (finest-level) kernel, measured now by ncu in a child
    process running this same workload (first finest launch of the second
    coarse step).  None if ncu is unavailable or fails."""
    import csv
    import io
    import shutil
    ncu = shutil.which("ncu") or "/usr/local/cuda/bin/ncu"
    if not os.path.exists(ncu):
        return None, "ncu not found"
    skip = (1 << levels) - 1  # level_step_all launches of the first coarse step
    cmd = [ncu, "--metrics", "dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum",
           "--clock-control", "none", "-k", "regex:level_step_all", "-s", str(skip), "-c", "1", "--csv",
           sys.executable, os.path.abspath(__file__), "--traffic-child", "--config", config, "--precision", precision]
    try:
        r = subprocess.run(cmd, capture_output=True, text=True, timeout=timeout, cwd=ROOT)
    except Exception as e:  # noqa: BLE001
        return None, f"ncu failed: {e!r}"[:200]
    vals = {}
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith('"')]
    for row in csv.reader(io.StringIO("\n".join(lines))):
        if len(row) > 14 and row[12] in ("dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__time_duration.sum"):
            unit = row[13]
            scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "B": 1, "KB": 1e3, "MB": 1e6, "GB": 1e9,
                     "nsecond": 1e-3, "usecond": 1, "msecond": 1e3, "ns": 1e-3, "us": 1, "ms": 1e3}.get(unit, 1)
            vals[row[12]] = float(row[14].replace(",", "")) * scale
    if "dram__bytes_read.sum" not in vals:
        return None, ("ncu gave no metrics: " + (r.stderr or r.stdout)[-200:]).replace("\n", " ")
    return {"dram_bytes_per_launch": vals["dram__bytes_read.sum"] + vals.get("dram__bytes_write.sum", 0.0),
            "duration_us_under_ncu": vals.get("gpu__time_duration.sum")}, "ncu, this run (child process, same build)"


def traffic_child(args):
    """The workload ncu_traffic() profiles: build, prologue, two coarse steps."""
    from paper_conf_ipps_mahmoudsm24_b200 import lbmr
    prob = CONFIGS[args.config][0]()
    prec = lbmr.FP32 if args.precision == "fp32" else lbmr.FP64
    g = lbmr.grid_from_problem(prob, precision=prec)
    g.step(2)
    g.synchronize()
    g.close()


def secondary_block(name, prob, prec, lbmr, steps, warmup, profile_steps, paper_mlups=None):
    """One more workload timed in the same run (N = 1 only): MLUPS over
    `steps` graph replays (CUDA events), the dominant kernel's roofline and
    per-level fractions."""
    import torch
    stream = torch.cuda.Stream()
    g = lbmr.grid_from_problem(prob, precision=prec, stream=stream.cuda_stream)
    info = g.info()
    leaves = [int(info.leaves[L]) for L in range(prob.levels)]
    upd = updates_per_step(leaves)
    g.step(warmup)
    g.synchronize()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    ev0.record(stream)
    g.step(steps)
    ev1.record(stream)
    torch.cuda.synchronize()
    ms = ev0.elapsed_time(ev1)
    value = upd * steps / (ms * 1e3)
    roof, per_level, _ = level_profile(g, prob, prec, lbmr, profile_steps, leaves)
    bpu = roof["bytes_per_update"]
    roof["step_frac"] = value * 1e6 * bpu / 1e9 / roof["peak"]
    g.close()
    del g
    out = {"workload": name, "value": value, "unit": "MLUPS", "ms_per_step": ms / steps, "steps": steps,
           "dtype": "f32" if prec == lbmr.FP32 else "f64", "leaves": leaves, "updates_per_step": upd,
           "roofline": roof, "per_level": per_level}
    if paper_mlups:
        out["paper_a100_mlups"] = paper_mlups
        out["vs_paper_a100"] = value / paper_mlups
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="tunnel4", choices=sorted(CONFIGS))
    ap.add_argument("--precision", default=None, choices=["fp32", "fp64"],
                    help="default fp32 (fp64 for the Tab. I sphere configs, the paper's precision)")
    ap.add_argument("--variant", default="paper", choices=["paper", "volumetric"],
                    help="interface transport: the paper's method (default) or the volumetric "
                         "ghost-advection variant (DESIGN.md §16)")
    ap.add_argument("--schedule", default="fused", choices=sorted(SCHEDULES),
                    help="fusion ablation (lbm_set_schedule); the default is the product schedule")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--profile-steps", type=int, default=10)
    ap.add_argument("--no-secondary", action="store_true",
                    help="skip the secondary blocks (cfg5 fp64, Tab. I s3 fp64 KBC) of the default run")
    ap.add_argument("--no-ncu-traffic", action="store_true", help="skip the in-run ncu DRAM-traffic capture")
    ap.add_argument("--traffic-child", action="store_true", help=argparse.SUPPRESS)
    args = ap.parse_args()
    if args.traffic_child:
        if args.precision is None:
            args.precision = DEFAULT_PRECISION.get(args.config, "fp32")
        traffic_child(args)
        return
    args.warmup = max(args.warmup, 3)
    if args.precision is None:
        args.precision = DEFAULT_PRECISION.get(args.config, "fp32")
    ws, rank, local = dist_setup()

    if args.impl == "reference":
        run_reference(args, ws, rank)
        return

    import torch
    # LBMR_BENCH_SHARE_DEVICE=1: every rank on cuda:0 with gloo (exercises the
    # N>1 code path on a one-GPU box; its timing is not a scaling number)
    share = os.environ.get("LBMR_BENCH_SHARE_DEVICE") == "1"
    torch.cuda.set_device(0 if share else local)
    if ws > 1:
        import torch.distributed as dist
        if share:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    from paper_conf_ipps_mahmoudsm24_b200 import lbmr

    build_fn, desc = CONFIGS[args.config]
    prob = build_fn()
    prec = lbmr.FP32 if args.precision == "fp32" else lbmr.FP64
    stream = torch.cuda.Stream()
    t0 = time.perf_counter()
    # N > 1: rank's x-slab of the SAME workload (strong scaling), halos written
    # into the neighbour GPUs' buffers by the level kernels (CUDA IPC / NVLink)
    g = lbmr.grid_from_problem(prob, precision=prec, stream=stream.cuda_stream, init=False, n_ranks=ws, rank=rank,
                               variant=lbmr.VARIANT_VOLUMETRIC if args.variant == "volumetric" else lbmr.VARIANT_PAPER)
    if ws > 1:
        import torch.distributed as dist
        blobs = {side: (g.halo_export(side) if lbmr.g_has(g, side) else None) for side in (0, 1)}
        allb = [None] * ws
        dist.all_gather_object(allb, blobs)
        for side in (0, 1):
            if lbmr.g_has(g, side):
                g.halo_connect(side, allb[(rank + (1 if side else -1)) % ws][1 - side])
    lbmr.init_from_problem(g, prob)
    g.set_schedule(SCHEDULES[args.schedule])
    setup_s = time.perf_counter() - t0
    info = g.info()
    leaves_local = [int(info.leaves[L]) for L in range(prob.levels)]
    leaves = list(leaves_local)
    if ws > 1:
        t = torch.tensor(leaves, device="cpu" if share else "cuda", dtype=torch.int64)
        torch.distributed.all_reduce(t)
        leaves = [int(v) for v in t.tolist()]
    upd = updates_per_step(leaves)
    launches_per_step = int(info.launches_per_step)  # for the schedule set above (lbm_grid_get_info)

    g.step(args.warmup)
    g.synchronize()

    def barrier():
        if ws > 1:
            torch.distributed.barrier()

    sampler = ClockSampler(0 if share else local)
    sampler.start()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    barrier()
    torch.cuda.synchronize()
    ev0.record(stream)
    g.step(args.steps)
    ev1.record(stream)
    torch.cuda.synchronize()
    barrier()
    clocks = sampler.stop()
    ms = ev0.elapsed_time(ev1)
    if ws > 1:
        t = torch.tensor([ms], device="cpu" if share else "cuda", dtype=torch.float64)
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
        ms = float(t.item())
    value = upd * args.steps / (ms * 1e3)  # all ranks' updates / max-over-ranks time

    # per-level device time of the level kernels (instrumented graph, CUDA events)
    roof, per_level, dom = level_profile(g, prob, prec, lbmr, args.profile_steps, leaves_local)
    bpu = roof["bytes_per_update"]
    peak = roof["peak"]

    # e2e through the public API with host buffers: per step an H2D BC update
    # (inlet velocity) and a D2H read of the step's result at monitoring
    # points (lbm_probe of N_PROBE finest-level fluid cells, like the paper's
    # Fig. 7 probes; the probe list itself is copied H2D every step too)
    n_e2e = args.steps  # same number of coarse steps as the device-timed region
    u_in = prob.bc.get(I.CLS_LID, (1, (0.0, 0.0, 0.0)))[1]
    Lf = prob.levels - 1
    fl = np.flatnonzero(prob.masks[Lf] == 1)
    pick = np.random.default_rng(3).choice(fl, size=min(N_PROBE, fl.size), replace=False)
    probes = np.stack(np.unravel_index(pick, prob.masks[Lf].shape), axis=1).astype(np.int64)
    torch.cuda.synchronize()
    barrier()
    t0 = time.perf_counter()
    for _ in range(n_e2e):
        g.set_bc(I.CLS_LID, lbmr.BC_VELOCITY, u_in)
        g.step(1)
        pr, _ = g.probe(Lf, probes)
    e2e_s = time.perf_counter() - t0
    if ws > 1:
        t = torch.tensor([e2e_s], device="cpu" if share else "cuda", dtype=torch.float64)
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
        e2e_s = float(t.item())
    e2e = {"value": upd * n_e2e / (e2e_s * 1e6), "unit": "MLUPS",
           "h2d_bytes_per_step": 32 + 27 + 8 * len(probes),
           "d2h_bytes_per_step": 32 * len(probes),
           "steps": n_e2e, "what": f"per step: lbm_set_bc (H2D) + lbm_step(1) + lbm_probe of {len(probes)} "
                                   "finest-level monitoring cells (H2D list, D2H rho/u), wall clock"}

    gi = g.info()
    dev_bytes = int(gi.device_bytes)
    g.close()
    del g
    # DRAM traffic of the dominant kernel, measured by ncu in this run (N = 1)
    traffic, traffic_src = None, "not measured (N > 1: ncu never wraps a multi-rank run)"
    if rank == 0 and ws == 1 and not args.no_ncu_traffic:
        t, traffic_src = ncu_traffic(args.config, args.precision, prob.levels)
        if t:
            traffic = t["dram_bytes_per_launch"]
            roof["traffic_duration_us_under_ncu"] = t["duration_us_under_ncu"]
    roof["traffic"] = traffic
    roof["traffic_source"] = traffic_src
    roof["traffic_over_algorithmic"] = traffic / roof["algorithmic_bytes_per_launch"] if traffic else None
    roof["build_id"] = lib_build_id()
    # secondary workloads of the default run (N = 1): the paper's precision on
    # the headline config, and the paper's own Tab. I workload at its largest size
    secondary = None
    if rank == 0 and ws == 1 and not args.no_secondary and args.config == "tunnel4" and args.schedule == "fused" \
            and args.variant == "paper":
        secondary = {}
        try:
            secondary["tunnel4_fp64"] = secondary_block(CONFIGS["tunnel4"][1] + ", fp64", prob, lbmr.FP64, lbmr,
                                                        max(5, args.steps // 2), 3, 4)
        except Exception as e:  # noqa: BLE001
            secondary["tunnel4_fp64"] = {"error": repr(e)[:300]}
        try:
            p3 = I.sphere_tab1(3)
            secondary["sphere_tab1_s3_fp64"] = secondary_block(CONFIGS["sphere_tab1_s3"][1] + ", fp64 (P:L258)", p3,
                                                               lbmr.FP64, lbmr, max(5, args.steps // 2), 3, 4,
                                                               PAPER_MLUPS["sphere_tab1_s3"])
            del p3
        except Exception as e:  # noqa: BLE001
            secondary["sphere_tab1_s3_fp64"] = {"error": repr(e)[:300]}
    cpu = None
    if rank == 0 and ws == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(prob)

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "MLUPS", "n_gpus": ws, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True,
            "scaling": "strong",
            # the paper's Tab. I number is fp64 on one GPU: only that run is the same workload
            "vs_baseline": (value / PAPER_MLUPS[args.config])
            if args.config in PAPER_MLUPS and ws == 1 and prec == lbmr.FP64 else None,
            "dtype": "f32" if prec == lbmr.FP32 else "f64", "data": "synthetic",
            "config": {"workload": desc, "levels": prob.levels, "leaves": leaves, "updates_per_step": upd,
                       "parallelism": f"x-slabs x{ws} (halo peer stores over NVLink)" if ws > 1 else "single",
                       "l2": f"working set {dev_bytes / 1e9:.2f} GB > 126 MB L2 (no flush needed)",
                       "precision": args.precision, "schedule": args.schedule, "variant": args.variant,
                       "setup_s": round(setup_s, 2),
                       **({"paper_a100_fp64_mlups": PAPER_MLUPS[args.config]} if args.config in PAPER_MLUPS else {})},
            "roofline": {**roof, "step_frac": value * 1e6 / ws * bpu / 1e9 / peak,
                         "note": "achieved / per_level are this rank's (rank 0) kernels" if ws > 1 else None},
            "per_level": per_level,
            "secondary": secondary,
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": launches_per_step * args.steps,
            "clocks": clocks,
        }
        print(json.dumps(line), flush=True)
    if ws > 1:
        torch.distributed.destroy_process_group()


if __name__ == "__main__":
    main()
