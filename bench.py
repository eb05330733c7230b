#!/usr/bin/env python3
"""Benchmark of the DASP SpMV hot path on B200 (BASELINE.json metric:
"FP64/FP16 SpMV GFLOPS & effective HBM GB/s (fraction of B200 peak), 1-8 GPUs").

One step = one whole pass of the hot path, y = alpha*A*x through dasp_spmv (the long-row
phase-1 kernel, then the main kernel: long phase 2 + empty rows, medium row-blocks, short tiles)
over one synthetic matrix; for N > 1 also the NCCL all-gather of the next x (iterated SpMV,
SURVEY.md §8(e)).

Workloads (BASELINE.json configs):
  N = 1 (default): configs[2] C3, power-law rows, 12.5M rows, 2.07e8 nnz, FP64 -- the >= 1e8-nnz
                   headline of north_star; the same line carries configs[3] C3 in FP16 ("fp16")
                   and the >= 1e8-nnz stencil C2+ in FP64 ("c2big") as sub-objects.
  N > 1          : configs[4] C5, mixed classes, 62.5M rows, 4.29e9 nnz, FP64, row slabs + NCCL
                   all-gather.  Without WORLD_SIZE in the environment, `--gpus N` re-launches this
                   script under torch.distributed.run with N ranks (one per GPU).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config c3] [--dtype f64|f16|f32]
                    [--variant mma|cudacore] [--impl dasp|reference]

--impl reference times the CPU oracle (oracle/, test infrastructure) on a bounded sample of the
same workload: this tier has no runnable reference implementation.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "FP64/FP16 SpMV GFLOPS & effective HBM GB/s (fraction of B200 peak), 1-8 GPUs"
CONFIG_DOC = {
    "c1a": "random CSR n=4096, Poisson(16) row lengths (configs[0])",
    "c1b": "class-coverage mix n=4096 (configs[0] variant)",
    "c2": "3D 27-point stencil 128^3, 55,742,968 nnz (configs[1])",
    "c2big": "3D 27-point stencil 162^3, 113,379,904 nnz (C2+, configs[1] at >= 1e8 nnz)",
    "c3": "power-law row lengths gamma=1.86 on [1,1e5] + 8 rows of 1e5, 12.5M rows, ~2.07e8 nnz (configs[2])",
    "c5": "mixed-class, mean row length ~64, 62.5M rows, ~4.29e9 nnz, row-partitioned (configs[4])",
    "c6": "short rows only, len U{1..4} (mc2depi-like)",
    "c7": "long rows only, lengths log-uniform [257, 2e4] (per-class probe)",
}
SIZES = {"f64": (8, 8, 8, 8), "f16": (2, 2, 4, 4), "f32": (4, 4, 4, 8)}   # s_v, s_x, s_y, s_a (partials)


def parse(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=1000)   # the paper averages 1000 runs
    ap.add_argument("--warmup", type=int, default=20)
    ap.add_argument("--config", default=None, help="default: c3 at N = 1, c5 at N > 1")
    ap.add_argument("--scale", type=float, default=1.0)
    ap.add_argument("--dtype", default="f64", choices=["f64", "f16", "f32"])
    ap.add_argument("--variant", default="cudacore", choices=["mma", "cudacore"])
    ap.add_argument("--impl", default="dasp", choices=["dasp", "reference"])
    ap.add_argument("--rbw", type=int, default=0, help="medium row-blocks per warp (LOOP_NUM); 0 = auto")
    ap.add_argument("--panel-rows", type=int, default=0, help="rows per panel (0 auto, -1 one global panel)")
    ap.add_argument("--max-len", type=int, default=0, help="MAX_LEN (P:L152): long iff len > max_len; 0 = auto")
    ap.add_argument("--tau", type=float, default=0.75, help="regular-block threshold tau (P:L158)")
    ap.add_argument("--x-stage", type=int, default=0, help="x-window staging: 0 auto, 1 off, 2 on")
    ap.add_argument("--iterate", action="store_true", help="N=1: run the row-slab iteration (x <- alpha*A*x)")
    ap.add_argument("--halo", action="store_true", help="slab mode: sparse halo exchange (all_to_all of the referenced "
                    "remote x only) overlapped with the local sub-matrix SpMV (SURVEY.md 8(f) f1)")
    ap.add_argument("--fused", action="store_true", help="slab mode: fuse the x all-gather into the SpMV "
                    "epilogue (symmetric memory + dasp_spmv_scatter)")
    ap.add_argument("--no-sub", action="store_true", help="skip the fp16 / c2big sub-measurements")
    ap.add_argument("--sub-steps", type=int, default=300)
    ap.add_argument("--no-compare", action="store_true", help="skip timing the other compute variant")
    ap.add_argument("--no-graph", action="store_true", help="skip the CUDA-graph replay measurement (N=1 SpMV)")
    ap.add_argument("--no-triad", action="store_true")
    ap.add_argument("--no-gpu-build", action="store_true", help="skip timing the device-side builder")
    ap.add_argument("--e2e-steps", type=int, default=40)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-budget-s", type=float, default=12.0)
    # launcher test hook (tests/test_bench_launcher.py): gloo on CPU, the slab SpMV replaced by a
    # torch CSR product -- exercises --gpus N -> N ranks without a GPU; never a bench number
    ap.add_argument("--cpu-stub", action="store_true", help=argparse.SUPPRESS)
    args = ap.parse_args(argv)
    if args.config is None:
        args.config = "c3" if args.gpus <= 1 else "c5"
    return args


def dist_env():
    return int(os.environ.get("RANK", "0")), int(os.environ.get("WORLD_SIZE", "1")), int(os.environ.get("LOCAL_RANK", "0"))


def relaunch(args, argv):
    """`--gpus N` without a torchrun environment: run this script as N ranks (one per GPU) under
    torch.distributed.run on 127.0.0.1; rank 0 prints the JSON line."""
    import socket
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    env = dict(os.environ)
    if not args.cpu_stub:
        env.setdefault("NCCL_DEBUG", "INFO")            # communicator size / NVLS / channels on stderr
        env.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__)] + argv
    return subprocess.call(cmd, env=env)


# ----------------------------------------------------------------------------------------------
# clocks sampled DURING the timed region (B200_PROFILING.md clocks line)
# ----------------------------------------------------------------------------------------------
class ClockSampler:
    REASONS = {0x8: "hw_slowdown", 0x40: "hw_thermal_slowdown", 0x20: "sw_thermal_slowdown", 0x4: "sw_power_cap",
               0x80: "hw_power_brake_slowdown", 0x100: "display_clock", 0x2: "applications_clocks_setting",
               0x1: "gpu_idle"}

    def __init__(self, index):
        self.index = index
        self.samples, self.reasons = [], set()
        self.max_mhz = None
        self._stop = threading.Event()
        self.ok = True
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nvml = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.ok = False

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nvml.nvmlDeviceGetClockInfo(self.h, self.nvml.NVML_CLOCK_SM))
                r = self.nvml.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in self.REASONS.items():
                    if r & bit and name != "gpu_idle":
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(0.02)

    def __enter__(self):
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        if self.ok:
            self._stop.set()
            self.t.join()

    def result(self):
        if not self.ok or not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": 0}
        return {"sm_mhz": float(np.median(self.samples)), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


# ----------------------------------------------------------------------------------------------
# bytes per launch
# ----------------------------------------------------------------------------------------------
def byte_model(info, dtype, beta_nonzero=False):
    """Algorithmic bytes per launch of each kernel, B_alg as SURVEY.md §8(d) writes it:
    slots * (s_v + 4) + groupPtr 8(row_long+1) + 2 s_a per long group (partial written by the long
    kernel, read by phase 2) + rowblockPtr 8(rowblocks+1) + irregPtr 4(row_medium+1) + outRow 4 per
    output slot + y s_y per row (x2 if beta != 0) + x s_x per column once.  What the format moves on
    top of that (irr_ptr is int64 over the 8 slots of every row-block, the long-unit schedule) is
    `overhead`, reported beside it and not counted as achieved bandwidth."""
    sv, sx, sy, sa = SIZES[dtype]
    b1 = 2 if beta_nonzero else 1
    m, n, nnz = info["m"], info["n"], info["nnz"]
    G = 128 if dtype == "f16" else 64
    ngp, nrb, rl = info["n_groups_padded"], info["rowblocks"], info["row_long"]
    nout_short = 64 * info["tiles_13"] + 32 * info["tiles_4"] + 64 * info["tiles_22"] + 128 * info["tiles_single"]
    long_ = ngp * G * (sv + 4) + ngp * sa
    phase2 = 8 * (rl + 1) + ngp * sa + 4 * rl + rl * sy * b1        # groupPtr, partials, outRow, y of long rows
    main = ((info["nnz_reg_new"] + info["nnz_irreg"] + info["nnz_short_new"]) * (sv + 4)
            + 8 * (nrb + 1) + 4 * (info["row_medium"] + 1)
            + 4 * (8 * nrb + nout_short + info["n_empty"])                  # outRow of every other output slot
            + (m - rl) * sy * b1 + n * sx)
    overhead = {"irr_ptr_int64_all_slots": 8 * (8 * nrb + 1) - 4 * (info["row_medium"] + 1),
                "long_unit_schedule": 4 * (ngp // 4)}
    csr_equiv = nnz * (sv + 4) + (m + 1) * 8 + n * sx + m * sy * b1
    return {"dasp_long_kernel": long_, "dasp_main_kernel": main + phase2, "total": long_ + main + phase2,
            "overhead": overhead, "csr_equiv": csr_equiv}


def load_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy burst)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def load_traffic(workload, dtype, variant, kernel, what=""):
    """ncu DRAM bytes (read + write) per launch recorded by scripts/ncu_summary.py (what="": bytes;
    "l2_read_requests": L1 -> L2 read requests per launch)."""
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_traffic.json")) as f:
            return json.load(f).get(f"{workload}/{dtype}/{variant}/{kernel}" + (f"/{what}" if what else ""))
    except Exception:
        return None


def load_l2_ceiling():
    """Measured ceiling of scattered 8-B gathers served by L2 (one 32-B sector request each):
    profiles/l2_gather_ceiling.json, written from scripts/probe/l2peak.py on this pool's B200s."""
    try:
        with open(os.path.join(ROOT, "profiles", "l2_gather_ceiling.json")) as f:
            return float(json.load(f)["Grequests_per_s"])
    except Exception:
        return None


def stream_triad(dev, n=1 << 28, reps=20):
    """STREAM triad a = b + s*c in FP64 on this GPU (3 x 2 GiB, 24 B per element), best of `reps`."""
    import torch
    b = torch.rand(n, dtype=torch.float64, device=dev)
    c = torch.rand(n, dtype=torch.float64, device=dev)
    a = torch.empty_like(b)
    best = float("inf")
    for _ in range(3):
        torch.add(b, c, alpha=3.0, out=a)
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        torch.add(b, c, alpha=3.0, out=a)
        e1.record()
        e1.synchronize()
        best = min(best, e0.elapsed_time(e1))
    del a, b, c
    torch.cuda.empty_cache()
    return 24.0 * n / (best * 1e-3) / 1e9


def roofline(info, dtype, kern, ms_step, workload, variant, peak, peak_src, triad=None):
    """Per-kernel algorithmic GB/s from the CUDA-event launch times; the dominant kernel (largest
    share of the step) is the line's roofline kernel."""
    bm = byte_model(info, dtype)
    per = {k: (ms, n) for k, (ms, n) in kern.items() if n}
    kernels = {}
    for k, (ms, nl) in per.items():
        avg = ms / nl
        alg = bm.get(k)
        tr = load_traffic(workload, dtype, variant, k)
        req = load_traffic(workload, dtype, variant, k, "l2_read_requests")
        ceil = load_l2_ceiling()
        kernels[k] = {"avg_ms": avg, "launches": nl, "share_of_step": avg / ms_step, "alg_bytes": alg,
                      "alg_gbs": alg / (avg * 1e-3) / 1e9 if alg else None,
                      "frac": alg / (avg * 1e-3) / 1e9 / peak if alg else None,
                      "traffic": tr, "traffic_over_alg": tr / alg if (tr and alg) else None,
                      # second roofline axis: L1 -> L2 read requests (ncu, per launch) over this launch's
                      # time, against the measured scattered-gather ceiling
                      "l2_requests": ({"per_launch": req, "achieved_G_per_s": req / (avg * 1e-3) / 1e9,
                                       "ceiling_G_per_s": ceil, "frac": req / (avg * 1e-3) / 1e9 / ceil}
                                      if (req and ceil) else None)}
    dom = max(per, key=lambda k: per[k][0]) if per else "dasp_main_kernel"
    d = kernels.get(dom, {})
    ach = d.get("alg_gbs")
    return {"kernel": dom, "bound": "hbm", "achieved": ach, "peak": peak, "unit": "GB/s",
            "frac": ach / peak if ach else None, "traffic": d.get("traffic"),
            "traffic_over_alg": d.get("traffic_over_alg"), "alg_bytes_per_launch": d.get("alg_bytes"),
            "avg_launch_ms": d.get("avg_ms"), "share_of_step": d.get("share_of_step"), "peak_source": peak_src,
            "stream_triad_gbs": triad, "frac_of_triad": ach / triad if (ach and triad) else None,
            "step": {"alg_bytes": bm["total"], "alg_gbs": bm["total"] / (ms_step * 1e-3) / 1e9,
                     "frac": bm["total"] / (ms_step * 1e-3) / 1e9 / peak, "overhead_bytes": bm["overhead"]},
            "kernels": kernels}


# ----------------------------------------------------------------------------------------------
# CPU oracle timing (cpu_baseline and --impl reference): bounded, strided row sample
# ----------------------------------------------------------------------------------------------
def row_sample(A, target_nnz):
    if A.nnz <= target_nnz:
        return A, 1
    stride = int(np.ceil(A.nnz / target_nnz))
    return row_sample_rows(A, np.arange(0, A.m, stride)), stride


def row_sample_rows(A, rows):
    """The sub-CSR of the given rows (all columns)."""
    import synth
    starts, ends = A.row_ptr[rows], A.row_ptr[rows + 1]
    lens = ends - starts
    rp = np.zeros(len(rows) + 1, dtype=np.int64)
    np.cumsum(lens, out=rp[1:])
    idx = np.repeat(starts - rp[:-1], lens) + np.arange(rp[-1])
    return synth.CSR(len(rows), A.n, rp, A.col[idx], A.val[idx])


def time_oracle(A, x, dtype, budget_s):
    import oracle
    narrow = {"f64": np.float64, "f16": np.float16, "f32": np.float32}[dtype]
    val = A.val.astype(narrow).astype(np.float64)
    xv = x.astype(narrow).astype(np.float64)
    oracle.spmv(A.row_ptr[:2], A.col[:1], val[:1], xv)  # load the library
    reps, t_total = 0, 0.0
    while t_total < budget_s and reps < 50:
        t0 = time.perf_counter()
        oracle.spmv(A.row_ptr, A.col, val, xv)
        t_total += time.perf_counter() - t0
        reps += 1
    threads = len(os.sched_getaffinity(0))
    oracle.spmv_mt(A.row_ptr, A.col, val, xv, threads=threads)
    reps_mt, t_mt, used = 0, 0.0, threads
    while t_mt < budget_s / 4 and reps_mt < 200:
        t0 = time.perf_counter()
        _, _, used = oracle.spmv_mt(A.row_ptr, A.col, val, xv, threads=threads)
        t_mt += time.perf_counter() - t0
        reps_mt += 1
    return t_total / reps, reps, t_mt / reps_mt, reps_mt, used


# ----------------------------------------------------------------------------------------------
# single GPU: plan, timed steps, per-kernel timing
# ----------------------------------------------------------------------------------------------
def make_plan(A, dtype, dev_index, variant, args):
    from paper_conf_sc_lu023_b200 import dasp
    val = A.val.astype({"f64": np.float64, "f16": np.float16, "f32": np.float32}[dtype])
    return dasp.dasp_plan_create(A.row_ptr, A.col, val, A.m, A.n, dtype, device=dev_index, variant=variant,
                                 medium_rb_per_warp=args.rbw, panel_rows=args.panel_rows,
                                 max_len=args.max_len, threshold=args.tau, x_stage=args.x_stage)


def timed_steps(step, plan, steps, warmup, dev, stream, clocks=True):
    """W untimed steps, then K steps between CUDA events on the launch stream (synchronize on both
    sides); per-kernel launch times from the plan's own events."""
    import torch
    from paper_conf_sc_lu023_b200 import dasp
    for _ in range(max(warmup, 3)):
        step()
    torch.cuda.synchronize(dev)
    dasp.dasp_plan_set_timing(plan, steps)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    clk = ClockSampler(dev.index or 0) if clocks else None
    if clk:
        clk.__enter__()
    torch.cuda.synchronize(dev)
    ev0.record(stream)
    for _ in range(steps):
        step()
    ev1.record(stream)
    torch.cuda.synchronize(dev)
    if clk:
        clk.__exit__()
    kern = dasp.dasp_plan_read_timing(plan)
    return ev0.elapsed_time(ev1), kern, (clk.result() if clk else None)


def sub_measure(workload, dtype, args, dev, local, peak, peak_src):
    """A second N = 1 workload in the same line (value, ms/step, per-kernel roofline)."""
    import torch
    import synth
    from paper_conf_sc_lu023_b200 import dasp
    spec = synth.config(workload)
    A = synth.generate(spec)
    variant = dasp.DASP_VARIANT_MMA if args.variant == "mma" else dasp.DASP_VARIANT_CUDACORE
    plan = make_plan(A, dtype, local, variant, args)
    xdt = {"f64": torch.float64, "f16": torch.float16, "f32": torch.float32}[dtype]
    xd = torch.from_numpy(synth.vector(101, spec.n)).to(xdt).to(dev)
    yd = torch.zeros(A.m, dtype=torch.float64 if dtype == "f64" else torch.float32, device=dev)
    stream = torch.cuda.current_stream(dev)

    def step():
        dasp.dasp_spmv(plan, xd, yd, 1.0, 0.0, stream, variant=variant, check=False)
    ms, kern, clk = timed_steps(step, plan, args.sub_steps, args.warmup, dev, stream)
    info = plan.info
    ms_step = ms / args.sub_steps
    out = {"workload": workload, "matrix": CONFIG_DOC.get(workload), "dtype": dtype, "nnz": A.nnz,
           "value": 2.0 * A.nnz / (ms_step * 1e-3) / 1e9, "unit": "GFLOPS", "ms_per_step": ms_step,
           "steps": args.sub_steps, "effective_gbs": byte_model(info, dtype)["csr_equiv"] / (ms_step * 1e-3) / 1e9,
           "roofline": roofline(info, dtype, kern, ms_step, workload, args.variant, peak, peak_src), "clocks": clk,
           "gpu_launches": int(info["launches_per_spmv"]) * args.sub_steps}
    plan.destroy()
    del xd, yd, A
    torch.cuda.empty_cache()
    return out


def main():
    argv = sys.argv[1:]
    args = parse(argv)
    rank, world, local = dist_env()
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(relaunch(args, argv))
    if args.impl == "reference":
        return run_reference(args, rank, world)
    if args.cpu_stub:
        return run_cpu_stub(args, rank, world)
    if world > 1 or args.iterate:
        return run_slab(args, rank, world, local)
    return run_single(args, local)


def run_single(args, local):
    import torch
    import synth
    from paper_conf_sc_lu023_b200 import dasp

    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    variant = dasp.DASP_VARIANT_MMA if args.variant == "mma" else dasp.DASP_VARIANT_CUDACORE
    spec = synth.config(args.config, scale=args.scale)
    workload = args.config if args.scale == 1.0 else f"{args.config}@{args.scale}"
    t0 = time.perf_counter()
    A = synth.generate(spec)
    gen_s = time.perf_counter() - t0
    x_global = synth.vector(101, spec.n)
    t1 = time.perf_counter()
    plan = make_plan(A, args.dtype, local, variant, args)
    plan_s = time.perf_counter() - t1
    info = plan.info
    xdt = {"f64": torch.float64, "f16": torch.float16, "f32": torch.float32}[args.dtype]
    ydt = torch.float64 if args.dtype == "f64" else torch.float32
    xd = torch.from_numpy(x_global).to(xdt).to(dev)
    yd = torch.zeros(A.m, dtype=ydt, device=dev)
    stream = torch.cuda.current_stream(dev)

    def step():
        dasp.dasp_spmv(plan, xd, yd, 1.0, 0.0, stream, variant=variant, check=False)
    ms_total, kern, clocks = timed_steps(step, plan, args.steps, args.warmup, dev, stream)
    ms_step = ms_total / args.steps
    nnz = A.nnz
    flops = 2.0 * nnz
    gflops = flops / (ms_step * 1e-3) / 1e9
    peak, peak_src = load_peaks()
    triad = None if args.no_triad else stream_triad(dev)
    roof = roofline(info, args.dtype, kern, ms_step, workload, args.variant, peak, peak_src, triad)
    bm = byte_model(info, args.dtype)

    # the other compute variant on the same plan (north_star: the MMA block-dot path is justified, or
    # not, against the CUDA-core variant of the same format)
    compare = None
    if not args.no_compare:
        other = dasp.DASP_VARIANT_CUDACORE if variant == dasp.DASP_VARIANT_MMA else dasp.DASP_VARIANT_MMA
        vname = {dasp.DASP_VARIANT_MMA: "mma", dasp.DASP_VARIANT_CUDACORE: "cudacore"}
        nrep = max(10, args.steps // 4)
        oms, okern, _ = timed_steps(lambda: dasp.dasp_spmv(plan, xd, yd, 1.0, 0.0, stream, variant=other, check=False),
                                    plan, nrep, 5, dev, stream, clocks=False)
        oms /= nrep
        compare = {vname[variant]: {"GFLOPS": gflops, "ms_per_step": ms_step},
                   vname[other]: {"GFLOPS": flops / (oms * 1e-3) / 1e9, "ms_per_step": oms, "steps": nrep,
                                  "kernels_ms": {k: v[0] / v[1] for k, v in okern.items() if v[1]}}}

    # the same K SpMVs captured once into a CUDA graph and replayed (launch gaps removed)
    graph = None
    if not args.no_graph:
        try:
            gs = torch.cuda.Stream(dev)
            gs.wait_stream(stream)
            g = torch.cuda.CUDAGraph()
            with torch.cuda.stream(gs):
                dasp.dasp_spmv(plan, xd, yd, 1.0, 0.0, gs, variant=variant, check=False)
                with torch.cuda.graph(g, stream=gs):
                    for _ in range(args.steps):
                        dasp.dasp_spmv(plan, xd, yd, 1.0, 0.0, gs, variant=variant, check=False)
            torch.cuda.synchronize(dev)
            g.replay()
            torch.cuda.synchronize(dev)
            g0, g1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            g0.record(stream)
            g.replay()
            g1.record(stream)
            torch.cuda.synchronize(dev)
            gms = g0.elapsed_time(g1) / args.steps
            graph = {"ms_per_step": gms, "GFLOPS": flops / (gms * 1e-3) / 1e9,
                     "kernel_nodes": int(info["launches_per_spmv"]) * args.steps}
            del g
        except Exception as exc:   # reported, not fatal
            graph = {"error": str(exc)[:200]}

    # e2e: the same metric through the C-ABI with HOST buffers -- dasp_spmv_host_stream copies every
    # step's own x_j in (pinned) and y_j out; neighbouring steps' copies overlap SpMV j
    e2e = None
    if args.e2e_steps > 0:
        xdt_np = {"f64": np.float64, "f16": np.float16, "f32": np.float32}[args.dtype]
        x1 = torch.from_numpy(x_global.astype(xdt_np))
        nv = max(2, min(args.e2e_steps, (2 << 30) // max(1, x1.numel() * x1.element_size())))
        xh = torch.empty((nv, x1.numel()), dtype=x1.dtype).pin_memory()
        for j in range(nv):
            xh[j].copy_(x1 if j == 0 else x1 * (1.0 + j / 64.0))      # distinct x per step
        yh = torch.empty((nv, A.m), dtype=ydt).pin_memory()
        dasp.dasp_spmv_host_stream(plan, xh, x1.numel(), yh, A.m, nv, 1.0, 0.0, stream)
        torch.cuda.synchronize(dev)
        done, t0 = 0, time.perf_counter()
        while done < args.e2e_steps:
            k = min(nv, args.e2e_steps - done)
            dasp.dasp_spmv_host_stream(plan, xh, x1.numel(), yh, A.m, k, 1.0, 0.0, stream)
            done += k
        dt = (time.perf_counter() - t0) / args.e2e_steps
        y_last = yh[(args.e2e_steps - 1) % nv].numpy()
        if not np.isfinite(y_last).all():
            raise RuntimeError("e2e result is not finite")
        dasp.dasp_spmv_host(plan, xh[0], yh[0], 1.0, 0.0, stream)
        t1 = time.perf_counter()
        for j in range(args.e2e_steps):
            dasp.dasp_spmv_host(plan, xh[j % nv], yh[j % nv], 1.0, 0.0, stream)
        dt1 = (time.perf_counter() - t1) / args.e2e_steps
        e2e = {"value": flops / dt / 1e9, "unit": "GFLOPS", "ms_per_step": dt * 1e3,
               "h2d_bytes_per_step": int(x1.numel() * x1.element_size()),
               "d2h_bytes_per_step": int(A.m * yh.element_size()), "api": "dasp_spmv_host_stream",
               "steps": args.e2e_steps, "distinct_x": nv, "h2d": "copy engine (pinned host)",
               "single_call": {"api": "dasp_spmv_host", "value": flops / dt1 / 1e9, "ms_per_step": dt1 * 1e3}}
        del xh, yh

    # preprocessing cost (Fig. 13): host builder vs the device builder (f2)
    gpu_build = None
    if not args.no_gpu_build:
        try:
            d_rp = torch.from_numpy(A.row_ptr).to(dev)
            d_col = torch.from_numpy(np.ascontiguousarray(A.col)).to(dev)
            d_val = torch.from_numpy(np.ascontiguousarray(A.val)).to(xdt).to(dev)
            builds = []
            for _ in range(2):   # the first call also pays CUDA lazy loading of the builder kernels
                torch.cuda.synchronize(dev)
                tb = time.perf_counter()
                dplan = dasp.dasp_plan_create_device(d_rp, d_col, d_val, A.m, A.n, args.dtype, device=local,
                                                     panel_rows=args.panel_rows)
                builds.append((dplan.info["build_ms"], (time.perf_counter() - tb) * 1e3))
                dplan.destroy()
            (cold_ms, _), (warm_ms, wall) = builds
            gpu_build = {"gpu_build_ms": warm_ms, "wall_ms": wall, "first_call_ms": cold_ms,
                         "host_build_ms": info["build_ms"], "host_upload_ms": info["upload_ms"],
                         "spmv_equivalents": warm_ms / ms_step,
                         "host_spmv_equivalents": (info["build_ms"] + info["upload_ms"]) / ms_step}
            del d_rp, d_col, d_val
            torch.cuda.empty_cache()
        except Exception as exc:   # reported, not fatal
            gpu_build = {"error": str(exc)[:200]}

    plan.destroy()
    del xd, yd
    torch.cuda.empty_cache()

    # the fp16 (configs[3]) and >= 1e8-nnz stencil sub-measurements of the same line
    subs = {}
    if not args.no_sub and args.config == "c3" and args.scale == 1.0 and args.dtype == "f64":
        subs["fp16"] = sub_measure("c3", "f16", args, dev, local, peak, peak_src)
        subs["c2big"] = sub_measure("c2big", "f64", args, dev, local, peak, peak_src)

    # CPU oracle on the host cores (rank 0, N = 1): a bounded row sample of the same workload
    cpu = None
    if not args.no_cpu_baseline:
        S, stride = row_sample(A, max(1, int(min(A.nnz, 1.5e8))))
        per, reps, per_mt, reps_mt, used = time_oracle(S, x_global, args.dtype, args.cpu_budget_s)
        cpu = {"value": 2.0 * S.nnz / per_mt / 1e9, "unit": "GFLOPS", "cores": used, "kind": "oracle",
               "sample": f"every {stride}th row of {workload} ({S.m} rows, {S.nnz} nnz), {reps_mt} reps, "
                         f"double-double CSR loop, rows split over {used} OpenMP threads (oracle_spmv_mt)",
               "single_thread": {"value": 2.0 * S.nnz / per / 1e9, "cores": 1, "reps": reps}}

    line = {
        "metric": METRIC, "value": gflops, "unit": "GFLOPS", "n_gpus": 1, "steps": args.steps,
        "warmup": max(args.warmup, 3), "ms_per_step": ms_step, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": args.dtype, "data": "synthetic",
        "config": {"workload": workload, "matrix": CONFIG_DOC.get(args.config, args.config),
                   "m": int(spec.m), "n": int(spec.n), "nnz": nnz, "variant": args.variant,
                   "panel_rows": info["panel_rows"], "parallelism": "single GPU",
                   "l2": "inputs larger than L2 (packed A, 2.8 GB for C3 FP64, streamed every step); x stays "
                         "L2-resident across steps as in the paper's averaged back-to-back runs (P:L567)"},
        "effective_gbs": bm["csr_equiv"] / (ms_step * 1e-3) / 1e9,
        "effective_frac_of_peak": bm["csr_equiv"] / (ms_step * 1e-3) / 1e9 / peak,
        "alg_gbs_step": bm["total"] / (ms_step * 1e-3) / 1e9,
        "alg_frac_step": bm["total"] / (ms_step * 1e-3) / 1e9 / peak,
        "gpu_launches": int(info["launches_per_spmv"]) * args.steps,
        "gpu_launches_per_step": int(info["launches_per_spmv"]),
        "roofline": roof, "cpu_baseline": cpu, "e2e": e2e, "clocks": clocks,
        "fp16": subs.get("fp16"), "c2big": subs.get("c2big"),
        "variant_compare": compare, "cuda_graph": graph, "preprocessing": gpu_build,
        "plan": {"build_ms": info["build_ms"], "upload_ms": info["upload_ms"], "gen_s": gen_s, "plan_s": plan_s,
                 "rows": {"empty": info["n_empty"], "short": info["n_len1"] + info["n_len2"] + info["n_len3"]
                          + info["n_len4"], "medium": info["row_medium"], "long": info["row_long"]},
                 "nnz": {"short": info["nnz_short"], "medium": info["nnz_medium"], "long": info["nnz_long"]},
                 "fill_rate": (info["nnz_long_new"] + info["nnz_reg_new"] + info["nnz_irreg"]
                               + info["nnz_short_new"]) / max(info["nnz"], 1) - 1.0,
                 "medium_rb_per_warp": info["medium_rb_per_warp"], "x_stage_blocks": info.get("x_stage_blocks")},
    }
    print(json.dumps(line))


# ----------------------------------------------------------------------------------------------
# row-slab iteration: N ranks (NCCL all-gather of x), or N = 1 with --iterate
# ----------------------------------------------------------------------------------------------
def run_slab(args, rank, world, local):
    import torch
    import torch.distributed as dist
    import synth
    from paper_conf_sc_lu023_b200 import dasp
    from paper_conf_sc_lu023_b200.multigpu import HaloSlabSpMV, SlabSpMV, build_slab

    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    elif args.fused:   # symmetric memory rendezvouses over a process group
        import socket
        with socket.socket() as sk:
            sk.bind(("127.0.0.1", 0))
            port = sk.getsockname()[1]
        dist.init_process_group("nccl", init_method=f"tcp://127.0.0.1:{port}", rank=0, world_size=1, device_id=dev)
    if args.dtype == "f16":
        raise SystemExit("the row-slab iteration needs x and y of one type (f64 or f32); FP16 writes f32 y")
    variant = dasp.DASP_VARIANT_MMA if args.variant == "mma" else dasp.DASP_VARIANT_CUDACORE
    spec = synth.config(args.config, scale=args.scale)
    workload = args.config if args.scale == 1.0 else f"{args.config}@{args.scale}"

    def reduce(v, op):
        if world == 1:
            return v
        t = torch.tensor([float(v)], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=op)
        return float(t.item())

    t0 = time.perf_counter()
    lens = synth.row_lengths(spec)
    slab = build_slab(lambda r0, nr: synth.generate(spec, r0, nr), lens, rank, world,
                      lambda v: reduce(v, dist.ReduceOp.MAX), need_norm=True, remap=not args.halo)
    if args.dtype == "f32":
        slab.val = slab.val.astype(np.float32)
    gen_s = time.perf_counter() - t0
    x_global = synth.vector(101, spec.n)
    t1 = time.perf_counter()
    if args.halo:
        it = HaloSlabSpMV(slab, world, rank, dev, args.dtype, variant=variant)
    else:
        it = SlabSpMV(slab, world, rank, dev, args.dtype, variant=variant, fused=args.fused)
    plan_s = time.perf_counter() - t1
    it.set_x(x_global)
    alpha = 1.0 / max(slab.inf_norm, 1e-300)   # ||A||_inf-normalised: the iteration stays bounded
    stream = torch.cuda.current_stream(dev)
    info = it.plan.info
    launches = int(info["launches_per_spmv"])
    if args.halo and it.plan_rem is not None:
        launches += int(it.plan_rem.info["launches_per_spmv"]) + 1

    for _ in range(max(args.warmup, 3)):
        it.step(alpha)
    torch.cuda.synchronize(dev)
    if world > 1:
        dist.barrier()
    dasp.dasp_plan_set_timing(it.plan, args.steps)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(local) as clk:
        torch.cuda.synchronize(dev)
        if world > 1:
            dist.barrier()
        ev0.record(stream)
        for _ in range(args.steps):
            it.step(alpha)
        ev1.record(stream)
        torch.cuda.synchronize(dev)
    ms_step = reduce(ev0.elapsed_time(ev1), dist.ReduceOp.MAX) / args.steps
    kern = dasp.dasp_plan_read_timing(it.plan)
    kern_ms = sum(ms for ms, n in kern.values()) / args.steps           # this rank's slab SpMV kernels
    kern_ms_max = reduce(kern_ms, dist.ReduceOp.MAX)
    bm = byte_model(info, args.dtype)
    alg_all = reduce(bm["total"], dist.ReduceOp.SUM)
    nnz_total = int(lens.sum())
    peak, peak_src = load_peaks()
    roof = roofline(info, args.dtype, kern, kern_ms, workload, args.variant, peak, peak_src)

    e2e = None
    if args.e2e_steps > 0:
        # per step: this rank's x slab host->device, assemble x (all-gather), SpMV, y slab device->host
        S0 = slab.S
        tnp = np.float64 if args.dtype == "f64" else np.float32
        xh = torch.from_numpy(x_global[slab.row0:slab.row0 + slab.rows].astype(tnp)).pin_memory()
        yh = torch.empty(slab.rows, dtype=xh.dtype).pin_memory()
        times = []
        for k in range(args.e2e_steps + 1):
            torch.cuda.synchronize(dev)
            if world > 1:
                dist.barrier()
            te = time.perf_counter()
            if args.halo:
                it.my_x().copy_(xh, non_blocking=True)
                it.step(alpha)
                yh.copy_(it.my_x(), non_blocking=True)
            else:
                it.x[it.cur][rank * S0: rank * S0 + slab.rows].copy_(xh, non_blocking=True)
                if world > 1 and not args.fused:
                    dist.all_gather_into_tensor(it.x[it.cur], it.x[it.cur][rank * S0:(rank + 1) * S0])
                it.step(alpha)
                yh.copy_(it.x[it.cur][rank * S0: rank * S0 + slab.rows], non_blocking=True)
            torch.cuda.synchronize(dev)
            if k:
                times.append(time.perf_counter() - te)
        dt = reduce(max(times), dist.ReduceOp.MAX)
        e2e = {"value": 2.0 * nnz_total / dt / 1e9, "unit": "GFLOPS", "ms_per_step": dt * 1e3,
               "h2d_bytes_per_step": int(reduce(xh.numel() * xh.element_size(), dist.ReduceOp.SUM)),
               "d2h_bytes_per_step": int(reduce(yh.numel() * yh.element_size(), dist.ReduceOp.SUM)),
               "api": "dasp_spmv" + ("_scatter" if args.fused else "") + (" + dasp_gather_halo" if args.halo else "")
                      + " (row-slab iteration)"}

    nccl = None
    if world > 1:
        try:
            nccl = {"backend": dist.get_backend(), "world": dist.get_world_size(),
                    "version": ".".join(map(str, torch.cuda.nccl.version()))}
        except Exception as exc:
            nccl = {"error": str(exc)[:100]}
    if rank == 0:
        line = {
            "metric": METRIC, "value": 2.0 * nnz_total / (ms_step * 1e-3) / 1e9, "unit": "GFLOPS", "n_gpus": world,
            "steps": args.steps, "warmup": max(args.warmup, 3), "ms_per_step": ms_step, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": args.dtype, "data": "synthetic",
            "config": {"workload": workload, "matrix": CONFIG_DOC.get(args.config, args.config), "m": int(spec.m),
                       "n": int(spec.n), "nnz": nnz_total, "variant": args.variant,
                       "parallelism": f"row-slab x{world}" + (
                           " + fused NVLink scatter of y into every rank's x" if args.fused else
                           " + sparse halo all_to_all overlapped with the local sub-matrix" if args.halo else
                           " + NCCL all-gather of x"),
                       "l2": "inputs larger than L2 (each slab's packed A streamed every step)"},
            "kernel_only": {"alg_gbs_aggregate": alg_all / (kern_ms_max * 1e-3) / 1e9, "ms_max_over_ranks": kern_ms_max,
                            "frac_of_peak_per_gpu": alg_all / (kern_ms_max * 1e-3) / 1e9 / world / peak},
            "per_iteration": {"alg_gbs_aggregate": alg_all / (ms_step * 1e-3) / 1e9,
                              "exchange_ms": max(0.0, ms_step - kern_ms_max)},
            "gpu_launches": launches * args.steps, "gpu_launches_per_step": launches,
            "roofline": roof, "cpu_baseline": None, "e2e": e2e, "clocks": clk.result(), "nccl": nccl,
            "plan": {"gen_s": gen_s, "plan_s": plan_s, "slab_rows_rank0": slab.rows, "slab_nnz_rank0": slab.nnz},
        }
        print(json.dumps(line))
    if dist.is_initialized():
        dist.destroy_process_group()


def run_cpu_stub(args, rank, world):
    """Launcher test only (gloo, CPU): the slab iteration with a torch CSR product as the local
    SpMV, printing the same JSON keys; the numbers mean nothing."""
    import torch
    import torch.distributed as dist
    import synth
    from paper_conf_sc_lu023_b200.multigpu import SlabSpMV, build_slab
    if world > 1:
        dist.init_process_group("gloo")
    spec = synth.config(args.config, scale=args.scale)
    lens = synth.row_lengths(spec)

    def red(v):
        t = torch.tensor([v], dtype=torch.float64)
        if world > 1:
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())
    slab = build_slab(lambda r0, nr: synth.generate(spec, r0, nr), lens, rank, world, red)
    Acsr = torch.sparse_csr_tensor(torch.from_numpy(slab.row_ptr), torch.from_numpy(slab.col.astype(np.int64)),
                                   torch.from_numpy(slab.val), size=(slab.rows, world * slab.S))

    def local(x, y, alpha):
        y.copy_(alpha * torch.mv(Acsr, x))
    it = SlabSpMV(slab, world, rank, "cpu", local_spmv=local)
    it.set_x(synth.vector(101, spec.n))
    t0 = time.perf_counter()
    for _ in range(args.steps):
        it.step(1.0 / slab.inf_norm)
    dt = red(time.perf_counter() - t0) / max(args.steps, 1)
    if rank == 0:
        print(json.dumps({"metric": METRIC, "value": 2.0 * float(lens.sum()) / dt / 1e9, "unit": "GFLOPS",
                          "n_gpus": world, "steps": args.steps, "ms_per_step": dt * 1e3, "cpu_stub": True,
                          "config": {"workload": args.config if args.scale == 1.0 else f"{args.config}@{args.scale}"}}))
    if dist.is_initialized():
        dist.destroy_process_group()


def run_reference(args, rank, world):
    """--impl reference: the CPU oracle, bounded per-step sample of the same workload (rank 0 only)."""
    if rank != 0:
        return
    import oracle
    import synth
    spec = synth.config(args.config, scale=args.scale)
    workload = args.config if args.scale == 1.0 else f"{args.config}@{args.scale}"
    lens = synth.row_lengths(spec)
    nnz = int(lens.sum())
    total = args.steps + max(args.warmup, 3)
    per_step_nnz = int(np.clip(90.0 * 2.5e8 / total, 2e5, nnz))   # ~90 s of oracle work in all
    # a strided row sample, generated chunk by chunk (C5 does not fit the host twice)
    stride = max(1, int(np.ceil(nnz / per_step_nnz)))
    parts, chunk = [], 1 << 22
    for r0 in range(0, spec.m, chunk):
        C = synth.generate(spec, r0, min(chunk, spec.m - r0))
        keep = np.arange((-r0) % stride, C.m, stride)
        parts.append(row_sample_rows(C, keep))
    rows_n = sum(p.m for p in parts)
    rp = np.zeros(rows_n + 1, dtype=np.int64)
    np.cumsum(np.concatenate([np.diff(p.row_ptr) for p in parts]), out=rp[1:])
    narrow = {"f64": np.float64, "f16": np.float16, "f32": np.float32}[args.dtype]
    col = np.concatenate([p.col for p in parts])
    val = np.concatenate([p.val for p in parts]).astype(narrow).astype(np.float64)
    xv = synth.vector(101, spec.n).astype(narrow).astype(np.float64)
    threads = len(os.sched_getaffinity(0))   # the box's host cores (the oracle's OpenMP row split)
    used = threads
    for _ in range(max(args.warmup, 3)):
        _, _, used = oracle.spmv_mt(rp, col, val, xv, threads=threads)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        oracle.spmv_mt(rp, col, val, xv, threads=threads)
    dt = (time.perf_counter() - t0) / args.steps
    v = 2.0 * int(rp[-1]) / dt / 1e9
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "GFLOPS", "n_gpus": world,
            "steps": args.steps, "warmup": max(args.warmup, 3), "ms_per_step": dt * 1e3, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": args.dtype, "data": "synthetic",
            "config": {"workload": workload, "matrix": CONFIG_DOC.get(args.config, args.config),
                       "m": int(spec.m), "n": int(spec.n), "nnz": nnz, "variant": "oracle (double-double CSR loop)",
                       "panel_rows": None, "parallelism": f"host CPU, rows over {used} OpenMP threads",
                       "l2": "n/a (CPU); a strided row sample of the workload per step"},
            "cpu_baseline": {"value": v, "unit": "GFLOPS", "cores": used, "kind": "oracle",
                             "sample": f"every {stride}th row ({rows_n} rows, {int(rp[-1])} nnz) per step, "
                                       f"double-double CSR loop over {used} OpenMP threads"},
            "e2e": {"value": v, "unit": "GFLOPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line))


if __name__ == "__main__":
    main()
