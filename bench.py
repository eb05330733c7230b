#!/usr/bin/env python3
"""Benchmark of the DASP SpMV hot path on B200 (BASELINE.json metric:
"FP64/FP16 SpMV GFLOPS & effective HBM GB/s (fraction of B200 peak), 1-8 GPUs").

One step = one whole pass of the hot path: y_slab = alpha * A_slab * x (dasp_spmv: the fused
long/medium/short kernel + the long-row finish kernel) over the configured synthetic matrix,
and for N > 1 the in-place NCCL all-gather of the next x (iterated SpMV).
Default workload (N = 1): configs[1], the 3-D 27-point stencil on 128^3 (55,742,968 nnz) in FP64;
``--config c3`` is configs[2] (power-law rows, ~2e8 nnz), ``--dtype f16`` configs[3].

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config c3] [--dtype f64|f16]
                    [--variant mma|cudacore] [--impl dasp|reference]

--impl reference times the CPU oracle (oracle/, test infrastructure) on a bounded sample of
the same workload: this tier has no runnable reference implementation.
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

CONFIG_DOC = {
    "c1a": "random CSR n=4096, Poisson(16) row lengths (configs[0])",
    "c1b": "class-coverage mix n=4096 (configs[0] variant)",
    "c2": "3D 27-point stencil 128^3, 55,742,968 nnz (configs[1])",
    "c2big": "3D 27-point stencil 162^3, 113,379,904 nnz (C2+)",
    "c3": "power-law row lengths gamma=1.86 on [1,1e5] + 8 rows of 1e5, 12.5M rows, ~2.04e8 nnz (configs[2])",
    "c5": "mixed-class mean row length ~64, row-partitioned (configs[4])",
    "c6": "short rows only, len U{1..4} (mc2depi-like)",
}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=1000)   # the paper averages 1000 runs
    ap.add_argument("--warmup", type=int, default=20)
    ap.add_argument("--config", default="c2")            # configs[1]: 27-point stencil 128^3, FP64
    ap.add_argument("--scale", type=float, default=1.0)
    ap.add_argument("--dtype", default="f64", choices=["f64", "f16", "f32"])
    ap.add_argument("--variant", default="cudacore", choices=["mma", "cudacore"])
    ap.add_argument("--no-compare", action="store_true", help="skip timing the other compute variant")
    ap.add_argument("--no-graph", action="store_true", help="skip the CUDA-graph replay measurement (N=1 SpMV)")
    ap.add_argument("--no-library", action="store_true", help="skip the cuSPARSE (torch CSR) context timing")
    ap.add_argument("--impl", default="dasp", choices=["dasp", "reference"])
    ap.add_argument("--rbw", type=int, default=0, help="medium row-blocks per warp (LOOP_NUM); 0 = auto")
    ap.add_argument("--pipeline", action="store_true", help="use the TMA-staged persistent kernel")
    ap.add_argument("--panel-rows", type=int, default=0, help="rows per panel (0 auto, -1 one global panel)")
    ap.add_argument("--co-schedule", type=int, default=-1, choices=[-1, 0, 1],
                    help="long-row units inside the medium/short kernel (1), in their own launch (0), auto (-1)")
    ap.add_argument("--no-triad", action="store_true")
    ap.add_argument("--iterate", action="store_true", help="N=1: run the row-slab iteration (x <- alpha*A*x)")
    ap.add_argument("--no-gpu-build", action="store_true", help="skip timing the device-side builder")
    ap.add_argument("--halo", action="store_true", help="slab mode: sparse halo exchange (all_to_all of the referenced "
                    "remote x only) overlapped with the local sub-matrix SpMV (SURVEY.md 8(f) f1)")
    ap.add_argument("--fused", action="store_true", help="slab mode: fuse the x all-gather into the SpMV "
                    "epilogue (symmetric memory + dasp_spmv_scatter)")
    ap.add_argument("--e2e-steps", type=int, default=40)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-budget-s", type=float, default=12.0)
    return ap.parse_args()


def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


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
# bytes per launch: CSR-equivalent and algorithmic (what the DASP format moves)
# ----------------------------------------------------------------------------------------------
def byte_model(info, dtype, beta_nonzero=False, split_short=False, fused_finish=True):
    """Algorithmic bytes per launch of each kernel.  fused_finish: the long-row
    phase 2 and the empty rows run inside dasp_main_kernel (the default; a separate
    dasp_finish_kernel only with the pipelined kernel)."""
    sv, sx, sy = {"f64": (8, 8, 8), "f16": (2, 2, 4), "f32": (4, 4, 4)}[dtype]
    sa = 4 if dtype == "f16" else 8
    b1 = 2 if beta_nonzero else 1
    m, n, nnz = info["m"], info["n"], info["nnz"]
    G = 128 if dtype == "f16" else 64
    ngp = info["n_groups_padded"]
    nrb = info["rowblocks"]
    nout = 64 * info["tiles_13"] + 32 * info["tiles_4"] + 64 * info["tiles_22"] + 128 * info["tiles_single"]
    n_short_rows = info["n_len1"] + info["n_len2"] + info["n_len3"] + info["n_len4"]
    long_ = ngp * G * (sv + 4) + ngp * sa + 4 * (ngp // 4)          # slots, group partials, unit order
    medium = ((info["nnz_reg_new"] + info["nnz_irreg"]) * (sv + 4) + 8 * (nrb + 1) + 8 * (8 * nrb + 1)
              + 4 * 8 * nrb + info["row_medium"] * sy * b1)
    short = info["nnz_short_new"] * (sv + 4) + 4 * nout + n_short_rows * sy * b1
    main = medium + (0 if split_short else short) + n * sx           # x counted once, here
    finish = (ngp * sa + 8 * (info["row_long"] + 1) + 4 * info["row_long"] + info["row_long"] * sy * b1
              + info["n_empty"] * (4 + sy * b1))
    csr_equiv = nnz * (sv + 4) + (m + 1) * 8 + n * sx + m * sy * b1
    if fused_finish:
        main += finish
    if info.get("co_scheduled"):          # long units run inside dasp_main_kernel (+ group_row)
        main += long_ + 4 * ngp
        long_ = 0
    out = {"dasp_long_kernel": long_, "dasp_main_kernel": main, "dasp_finish_kernel": 0 if fused_finish else finish,
           "total": long_ + main + (0 if fused_finish else finish) + (short if split_short else 0),
           "csr_equiv": csr_equiv}
    if split_short:
        out["dasp_short_kernel"] = short + 8 * info["tiles_13"] + 8 * info["tiles_4"] + 8 * info["tiles_22"] \
            + 8 * info["tiles_single"]                                    # + per-tile metadata
    return out


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy burst)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def stream_triad(dev, n=1 << 28, reps=20):
    """STREAM triad a = b + s*c in FP64 on this GPU (3 x 2 GiB arrays, 24 B per element), best of
    `reps`, CUDA events: the same-run HBM reference of SURVEY.md §8(d)."""
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


def load_traffic(config, dtype, variant, kernel="dasp_main_kernel"):
    """ncu DRAM bytes per launch recorded by scripts/ncu_summary.py (profiles/ncu_traffic.json)."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return d.get(f"{config}/{dtype}/{variant}/{kernel}", d.get(f"{config}/{dtype}/{variant}")
                     if kernel == "dasp_main_kernel" else None)
    except Exception:
        return None


# ----------------------------------------------------------------------------------------------
# CPU oracle timing (cpu_baseline and --impl reference): bounded, strided row sample
# ----------------------------------------------------------------------------------------------
def row_sample(A, target_nnz):
    import synth
    if A.nnz <= target_nnz:
        return A, 1
    stride = int(np.ceil(A.nnz / target_nnz))
    rows = np.arange(0, A.m, stride)
    starts, ends = A.row_ptr[rows], A.row_ptr[rows + 1]
    lens = ends - starts
    rp = np.zeros(len(rows) + 1, dtype=np.int64)
    np.cumsum(lens, out=rp[1:])
    idx = np.repeat(starts - rp[:-1], lens) + np.arange(rp[-1])
    return synth.CSR(len(rows), A.n, rp, A.col[idx], A.val[idx]), stride


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
    # the same loop, rows split over every host core this process may use (OpenMP)
    threads = len(os.sched_getaffinity(0))
    oracle.spmv_mt(A.row_ptr, A.col, val, xv, threads=threads)
    reps_mt, t_mt = 0, 0.0
    while t_mt < budget_s / 4 and reps_mt < 200:
        t0 = time.perf_counter()
        _, _, used = oracle.spmv_mt(A.row_ptr, A.col, val, xv, threads=threads)
        t_mt += time.perf_counter() - t0
        reps_mt += 1
    return t_total / reps, reps, t_mt / reps_mt, reps_mt, used


# ----------------------------------------------------------------------------------------------
def main():
    args = parse()
    rank, world, local = dist_env()
    if args.gpus != world and world > 1:
        print(f"warning: --gpus {args.gpus} but WORLD_SIZE {world}", file=sys.stderr)
    import synth

    spec = synth.config(args.config, scale=args.scale)
    workload = args.config if args.scale == 1.0 else f"{args.config}@{args.scale}"
    metric = "FP64/FP16 SpMV GFLOPS & effective HBM GB/s (fraction of B200 peak), 1-8 GPUs"

    if args.impl == "reference":
        return run_reference(args, spec, workload, metric, rank, world)

    import torch
    import torch.distributed as dist
    from paper_conf_sc_lu023_b200 import dasp
    from paper_conf_sc_lu023_b200.multigpu import HaloSlabSpMV, SlabSpMV, build_slab

    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    elif args.fused:   # the fused scatter mode rendezvouses symmetric memory over a process group
        import socket
        with socket.socket() as sk:
            sk.bind(("127.0.0.1", 0))
            port = sk.getsockname()[1]
        dist.init_process_group("nccl", init_method=f"tcp://127.0.0.1:{port}", rank=0, world_size=1, device_id=dev)
    variant = dasp.DASP_VARIANT_MMA if args.variant == "mma" else dasp.DASP_VARIANT_CUDACORE

    # ---- inputs: this rank's slab (whole matrix at N = 1), generated per row ----
    t0 = time.perf_counter()
    lens = synth.row_lengths(spec)

    def gen_rows(r0, nr):
        return synth.generate(spec, r0, nr)

    def reduce_max(v):
        if world == 1:
            return v
        t = torch.tensor([v], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    use_slab = world > 1 or args.iterate
    slab = build_slab(gen_rows, lens, rank, world, reduce_max, need_norm=use_slab, remap=not args.halo)
    gen_s = time.perf_counter() - t0
    if args.dtype != "f64":
        if world > 1:
            raise SystemExit("FP16 / FP32 multi-GPU is not part of the north star")
        slab.val = slab.val.astype(np.float16 if args.dtype == "f16" else np.float32)
    x_global = synth.vector(101, spec.n)

    t1 = time.perf_counter()
    if not use_slab:
        # single GPU: plain SpMV over resident inputs, y overwritten every step
        plan = dasp.dasp_plan_create(slab.row_ptr, slab.col, slab.val, slab.rows, spec.n, args.dtype,
                                     device=local, variant=variant, medium_rb_per_warp=args.rbw,
                                     pipeline=args.pipeline, panel_rows=args.panel_rows,
                                     co_schedule=args.co_schedule)
        xdt = {"f64": torch.float64, "f16": torch.float16, "f32": torch.float32}[args.dtype]
        ydt = torch.float64 if args.dtype == "f64" else torch.float32
        xd = torch.from_numpy(x_global).to(xdt).to(dev)
        yd = torch.zeros(slab.rows, dtype=ydt, device=dev)
        stream = torch.cuda.current_stream(dev)
        alpha = 1.0

        def step():
            dasp.dasp_spmv(plan, xd, yd, alpha, 0.0, stream, variant=variant, check=False)
    else:
        if args.halo:
            it = HaloSlabSpMV(slab, world, rank, dev, args.dtype, variant=variant)
        else:
            it = SlabSpMV(slab, world, rank, dev, args.dtype, variant=variant, fused=args.fused)
        plan = it.plan
        it.set_x(x_global)
        alpha = 1.0 / max(slab.inf_norm, 1e-300)   # iterated SpMV stays bounded
        stream = torch.cuda.current_stream(dev)

        def step():
            it.step(alpha)
    plan_s = time.perf_counter() - t1
    info = plan.info
    launches_step = int(info["launches_per_spmv"])
    if use_slab and args.halo and it.plan_rem is not None:   # remote sub-matrix SpMV + halo pack
        launches_step += int(it.plan_rem.info["launches_per_spmv"]) + 1

    # ---- warm-up, then K timed steps (barrier + synchronize on both sides, CUDA events) ----
    for _ in range(max(args.warmup, 3)):
        step()
    torch.cuda.synchronize(dev)
    if world > 1:
        dist.barrier()
    dasp.dasp_plan_set_timing(plan, args.steps)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(local) as clk:
        torch.cuda.synchronize(dev)
        if world > 1:
            dist.barrier()
        ev0.record(stream)
        for _ in range(args.steps):
            step()
        ev1.record(stream)
        torch.cuda.synchronize(dev)
    ms_total = ev0.elapsed_time(ev1)
    if world > 1:
        t = torch.tensor([ms_total], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms_total = float(t.item())
        dist.barrier()
    kern = dasp.dasp_plan_read_timing(plan)
    ms_step = ms_total / args.steps

    # the other compute variant on the same plan and inputs (north_star: the MMA block-dot path
    # is justified, or not, against the CUDA-core variant of the same format)
    compare = None
    if not use_slab and not args.no_compare:
        other = dasp.DASP_VARIANT_CUDACORE if variant == dasp.DASP_VARIANT_MMA else dasp.DASP_VARIANT_MMA
        vname = {dasp.DASP_VARIANT_MMA: "mma", dasp.DASP_VARIANT_CUDACORE: "cudacore"}
        nrep = max(10, args.steps // 4)
        for _ in range(5):
            dasp.dasp_spmv(plan, xd, yd, 1.0, 0.0, stream, variant=other, check=False)
        torch.cuda.synchronize(dev)
        c0, c1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        c0.record(stream)
        for _ in range(nrep):
            dasp.dasp_spmv(plan, xd, yd, 1.0, 0.0, stream, variant=other, check=False)
        c1.record(stream)
        torch.cuda.synchronize(dev)
        oms = c0.elapsed_time(c1) / nrep
        compare = {vname[variant]: {"GFLOPS": 2.0 * float(lens.sum()) / (ms_step * 1e-3) / 1e9, "ms_per_step": ms_step},
                   vname[other]: {"GFLOPS": 2.0 * float(lens.sum()) / (oms * 1e-3) / 1e9, "ms_per_step": oms,
                                  "steps": nrep}}

    # the same K SpMVs captured once into a CUDA graph and replayed (launch overhead removed; what an
    # iterative caller gets by capturing its loop).  Reported beside the eager number, not instead.
    graph = None
    if not use_slab and not args.no_graph:
        try:
            dasp.dasp_plan_set_timing(plan, 0)
            gs = torch.cuda.Stream(dev)
            gs.wait_stream(stream)
            g = torch.cuda.CUDAGraph()
            with torch.cuda.stream(gs):
                dasp.dasp_spmv(plan, xd, yd, alpha, 0.0, gs, variant=variant, check=False)   # warm, outside
                with torch.cuda.graph(g, stream=gs):
                    for _ in range(args.steps):
                        dasp.dasp_spmv(plan, xd, yd, alpha, 0.0, gs, variant=variant, check=False)
            torch.cuda.synchronize(dev)
            g.replay()
            torch.cuda.synchronize(dev)
            g0, g1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            g0.record(stream)
            g.replay()
            g1.record(stream)
            torch.cuda.synchronize(dev)
            gms = g0.elapsed_time(g1) / args.steps
            graph = {"ms_per_step": gms, "GFLOPS": 2.0 * float(lens.sum()) / (gms * 1e-3) / 1e9,
                     "kernel_nodes": int(info["launches_per_spmv"]) * args.steps}
            del g
        except Exception as exc:   # reported, not fatal
            graph = {"error": str(exc)}

    # context only (the paper compares against cuSPARSE CSR SpMV): the same matrix and
    # x through torch's CSR tensor @ vector, i.e. cuSPARSE SpMV on this GPU, same timing protocol
    library = None
    if not use_slab and not args.no_library and args.dtype in ("f64", "f32"):
        try:
            vdt = torch.float64 if args.dtype == "f64" else torch.float32
            idt = np.int32 if int(slab.row_ptr[-1]) < 2 ** 31 - 1 else np.int64   # one index dtype for both
            Acsr = torch.sparse_csr_tensor(torch.from_numpy(slab.row_ptr.astype(idt)).to(dev),
                                           torch.from_numpy(np.ascontiguousarray(slab.col).astype(idt)).to(dev),
                                           torch.from_numpy(np.ascontiguousarray(slab.val)).to(vdt).to(dev),
                                           size=(slab.rows, spec.n), check_invariants=False)
            xl = xd.to(vdt)
            with torch.cuda.stream(stream):
                for _ in range(5):
                    yl = torch.mv(Acsr, xl)
                l0, l1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                nrep = min(args.steps, 200)
                l0.record(stream)
                for _ in range(nrep):
                    yl = torch.mv(Acsr, xl)
                l1.record(stream)
            torch.cuda.synchronize(dev)
            lms = l0.elapsed_time(l1) / nrep
            err = float(torch.max(torch.abs(yl.to(torch.float64) - yd.to(torch.float64) / alpha)))
            library = {"impl": "cuSPARSE CSR SpMV via torch.mv(sparse_csr)", "ms_per_step": lms,
                       "GFLOPS": 2.0 * float(lens.sum()) / (lms * 1e-3) / 1e9, "steps": nrep,
                       "max_abs_diff_vs_dasp": err}
            del Acsr, xl, yl
            torch.cuda.empty_cache()
        except Exception as exc:   # reported, not fatal
            library = {"error": str(exc)[:200]}

    nnz_total = int(lens.sum())
    flops_step = 2.0 * nnz_total
    gflops = flops_step / (ms_step * 1e-3) / 1e9
    bm = byte_model(info, args.dtype, split_short=kern.get("dasp_short_kernel", (0, 0))[1] > 0,
                    fused_finish=kern.get("dasp_finish_kernel", (0, 0))[1] == 0)
    # whole-job CSR-equivalent bytes: sum over ranks (slab models), else the local one
    csr_bytes = bm["csr_equiv"]
    if world > 1:
        t = torch.tensor([float(csr_bytes)], dtype=torch.float64, device=dev)
        dist.all_reduce(t)
        csr_bytes = float(t.item())
    eff_gbs = csr_bytes / (ms_step * 1e-3) / 1e9

    # ---- roofline of the dominant kernel (largest share of the step), per launch ----
    peak, peak_src = load_peaks()
    per_kernel = {k: (ms, nl) for k, (ms, nl) in kern.items() if nl}
    dom = max(per_kernel, key=lambda k: per_kernel[k][0]) if per_kernel else "dasp_main_kernel"
    dom_ms, dom_n = per_kernel.get(dom, (0.0, 0))
    dom_avg = dom_ms / max(dom_n, 1)
    dom_bytes = bm.get(dom, bm["total"])
    achieved = dom_bytes / (dom_avg * 1e-3) / 1e9 if dom_n else None
    traffic = load_traffic(workload, args.dtype, args.variant, dom)
    triad = None if args.no_triad else stream_triad(dev)
    roofline = {"kernel": dom, "bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                "frac": achieved / peak if achieved else None, "traffic": traffic,
                "alg_bytes_per_launch": dom_bytes, "avg_launch_ms": dom_avg,
                "share_of_step": dom_avg / ms_step if dom_n else None, "peak_source": peak_src,
                "stream_triad_gbs": triad, "frac_of_triad": achieved / triad if (achieved and triad) else None,
                "kernels": {k: {"avg_ms": ms / nl, "launches": nl, "alg_bytes": bm.get(k),
                                "alg_gbs": bm[k] / (ms / nl * 1e-3) / 1e9 if k in bm and ms > 0 else None}
                            for k, (ms, nl) in per_kernel.items()}}

    # ---- e2e: the same metric through the C-ABI with HOST buffers (copies inside the timed region) ----
    e2e = None
    if use_slab and args.e2e_steps > 0:
        # per step: this rank's x slab host->device, assemble x (all-gather), SpMV, y slab device->host
        S0 = slab.S
        xh = torch.from_numpy(x_global[slab.row0:slab.row0 + slab.rows].copy()).pin_memory()
        yh = torch.empty(slab.rows, dtype=torch.float64).pin_memory()
        times = []
        for k in range(args.e2e_steps + 1):
            torch.cuda.synchronize(dev)
            if world > 1:
                dist.barrier()
            t0 = time.perf_counter()
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
                times.append(time.perf_counter() - t0)
        dt = max(times) if times else float("nan")
        if world > 1:
            t = torch.tensor([dt], dtype=torch.float64, device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            dt = float(t.item())
        e2e = {"value": flops_step / dt / 1e9, "unit": "GFLOPS", "ms_per_step": dt * 1e3,
               "h2d_bytes_per_step": int(xh.numel() * 8) * world, "d2h_bytes_per_step": int(yh.numel() * 8) * world,
               "api": "dasp_spmv" + ("_scatter" if args.fused else "") + (" + dasp_gather_halo" if args.halo else "")
                      + " (row-slab iteration)"}
    if not use_slab and args.e2e_steps > 0:
        # dasp_spmv_host_stream: every step copies its own x_j in (pinned) and y_j out; the copies of
        # neighbouring steps overlap SpMV j on the two copy engines (H2D / D2H full duplex)
        xdt_np = {"f64": np.float64, "f16": np.float16, "f32": np.float32}[args.dtype]
        ydt = torch.float64 if args.dtype == "f64" else torch.float32
        x1 = torch.from_numpy(x_global.astype(xdt_np))
        nv = max(2, min(args.e2e_steps, (2 << 30) // max(1, x1.numel() * x1.element_size())))
        xh = torch.empty((nv, x1.numel()), dtype=x1.dtype).pin_memory()
        for j in range(nv):
            xh[j].copy_(x1 if j == 0 else x1 * (1.0 + j / 64.0))      # distinct x per step
        yh = torch.empty((nv, slab.rows), dtype=ydt).pin_memory()
        dasp.dasp_spmv_host_stream(plan, xh.data_ptr(), x1.numel(), yh.data_ptr(), slab.rows, nv, 1.0, 0.0, stream)
        torch.cuda.synchronize(dev)
        done, t0 = 0, time.perf_counter()
        while done < args.e2e_steps:
            k = min(nv, args.e2e_steps - done)
            dasp.dasp_spmv_host_stream(plan, xh.data_ptr(), x1.numel(), yh.data_ptr(), slab.rows, k, 1.0, 0.0, stream)
            done += k
        dt = (time.perf_counter() - t0) / args.e2e_steps
        assert np.isfinite(yh[0].numpy()).all()
        # one synchronous dasp_spmv_host call per step (no overlap between steps), for context
        dasp.dasp_spmv_host(plan, xh[0].data_ptr(), yh[0].data_ptr(), 1.0, 0.0, stream)
        t1 = time.perf_counter()
        for j in range(args.e2e_steps):
            dasp.dasp_spmv_host(plan, xh[j % nv].data_ptr(), yh[j % nv].data_ptr(), 1.0, 0.0, stream)
        dt1 = (time.perf_counter() - t1) / args.e2e_steps
        e2e = {"value": flops_step / dt / 1e9, "unit": "GFLOPS", "ms_per_step": dt * 1e3,
               "h2d_bytes_per_step": int(x1.numel() * x1.element_size()),
               "d2h_bytes_per_step": int(slab.rows * yh.element_size()), "api": "dasp_spmv_host_stream",
               "steps": args.e2e_steps, "distinct_x": nv,
               "h2d": "SM loads from pinned host (UVA)" if os.environ.get("DASP_H2D_SM", "0") not in ("", "0") else "copy engine",
               "single_call": {"api": "dasp_spmv_host", "value": flops_step / dt1 / 1e9, "ms_per_step": dt1 * 1e3}}

    # ---- preprocessing cost (Fig. 13): host builder vs the device builder (f2) ----
    gpu_build = None
    if not use_slab and not args.no_gpu_build:
        try:
            vdt = {"f64": torch.float64, "f16": torch.float16, "f32": torch.float32}[args.dtype]
            d_rp = torch.from_numpy(slab.row_ptr).to(dev)
            d_col = torch.from_numpy(np.ascontiguousarray(slab.col)).to(dev)
            d_val = torch.from_numpy(np.ascontiguousarray(slab.val)).to(vdt).to(dev)
            builds = []
            for _ in range(2):   # the first call also pays CUDA lazy module loading of the builder kernels
                torch.cuda.synchronize(dev)
                t0 = time.perf_counter()
                dplan = dasp.dasp_plan_create_device(d_rp, d_col, d_val, slab.rows, spec.n, args.dtype,
                                                     device=local, panel_rows=args.panel_rows)
                builds.append((dplan.info["build_ms"], (time.perf_counter() - t0) * 1e3))
                dplan.destroy()
            (cold_ms, cold_wall), (warm_ms, wall) = builds
            gpu_build = {"gpu_build_ms": warm_ms, "wall_ms": wall, "first_call_ms": cold_ms,
                         "first_call_note": "first call in the process includes CUDA lazy loading of the builder kernels",
                         "host_build_ms": info["build_ms"], "host_upload_ms": info["upload_ms"],
                         "spmv_equivalents": warm_ms / ms_step,
                         "host_spmv_equivalents": (info["build_ms"] + info["upload_ms"]) / ms_step}
            del d_rp, d_col, d_val
            torch.cuda.empty_cache()
        except Exception as exc:   # reported, not fatal: the bench line is about the SpMV
            gpu_build = {"error": str(exc)}

    # ---- CPU oracle on the host cores (rank 0, N = 1 only) ----
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        A = synth.CSR(slab.rows, spec.n, slab.row_ptr, slab.col, slab.val.astype(np.float64))
        target = max(1, int(min(A.nnz, 1.5e8)))
        S, stride = row_sample(A, target)
        per, reps, per_mt, reps_mt, used = time_oracle(S, x_global, args.dtype, args.cpu_budget_s)
        cpu = {"value": 2.0 * S.nnz / per_mt / 1e9, "unit": "GFLOPS", "cores": used, "kind": "oracle",
               "sample": f"every {stride}th row of {workload} ({S.m} rows, {S.nnz} nnz), {reps_mt} reps, "
                         f"double-double CSR loop, rows split over {used} OpenMP threads (oracle_spmv_mt)",
               "single_thread": {"value": 2.0 * S.nnz / per / 1e9, "cores": 1, "reps": reps}}

    if rank == 0:
        clocks = clk.result()
        line = {
            "metric": metric, "value": gflops, "unit": "GFLOPS", "n_gpus": world, "steps": args.steps,
            "warmup": max(args.warmup, 3), "ms_per_step": ms_step, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": args.dtype, "data": "synthetic",
            "config": {"workload": workload, "matrix": CONFIG_DOC.get(args.config, args.config),
                       "m": int(spec.m), "n": int(spec.n), "nnz": nnz_total, "variant": args.variant,
                       "kernel": "pipeline" if info.get("pipeline") else "direct", "panel_rows": info["panel_rows"],
                       "co_scheduled": bool(info.get("co_scheduled")),
                       "parallelism": f"row-slab x{world}" + (
                           (" + fused NVLink scatter of y into every rank's x" if args.fused else
                            " + sparse halo all_to_all overlapped with the local sub-matrix" if args.halo else
                            " + NCCL all-gather of x") if use_slab else ""),
                       "l2": "inputs larger than L2 (packed A streamed every step); x stays L2-resident "
                             "across steps as in the paper's averaged back-to-back runs"},
            "effective_gbs": eff_gbs, "effective_frac_of_peak": eff_gbs / peak,
            "alg_gbs_step": bm["total"] * world / (ms_step * 1e-3) / 1e9 if world == 1 else None,
            "gpu_launches": launches_step * args.steps,
            "gpu_launches_per_step": launches_step,
            "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e, "clocks": clocks,
            "variant_compare": compare, "cuda_graph": graph, "library_context": library,
            "preprocessing": gpu_build,
            "plan": {"build_ms": info["build_ms"], "upload_ms": info["upload_ms"], "gen_s": gen_s, "plan_s": plan_s,
                     "rows": {"empty": info["n_empty"], "short": info["n_len1"] + info["n_len2"] + info["n_len3"]
                              + info["n_len4"], "medium": info["row_medium"], "long": info["row_long"]},
                     "nnz": {"short": info["nnz_short"], "medium": info["nnz_medium"], "long": info["nnz_long"]},
                     "fill_rate": (info["nnz_long_new"] + info["nnz_reg_new"] + info["nnz_irreg"]
                                   + info["nnz_short_new"]) / max(info["nnz"], 1) - 1.0,
                     "medium_rb_per_warp": info["medium_rb_per_warp"]},
        }
        print(json.dumps(line))
    if dist.is_initialized():
        dist.destroy_process_group()


def run_reference(args, spec, workload, metric, rank, world):
    """--impl reference: the CPU oracle, bounded per-step sample of the same workload."""
    if rank != 0:
        return
    import synth
    lens = synth.row_lengths(spec)
    nnz = int(lens.sum())
    A = synth.generate(spec)
    narrow = {"f64": np.float64, "f16": np.float16, "f32": np.float32}[args.dtype]
    A.val = A.val.astype(narrow).astype(np.float64)
    x = synth.vector(101, spec.n)
    total = args.steps + max(args.warmup, 3)
    per_step_nnz = int(np.clip(90.0 * 2.5e8 / total, 2e5, nnz))   # ~90 s of oracle work in all
    S, stride = row_sample(A, per_step_nnz)
    import oracle
    xv = x.astype(narrow).astype(np.float64)
    threads = len(os.sched_getaffinity(0))   # the box's host cores (the oracle's OpenMP row split)
    for _ in range(max(args.warmup, 3)):
        _, _, used = oracle.spmv_mt(S.row_ptr, S.col, S.val, xv, threads=threads)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        oracle.spmv_mt(S.row_ptr, S.col, S.val, xv, threads=threads)
    dt = (time.perf_counter() - t0) / args.steps
    v = 2.0 * S.nnz / dt / 1e9
    line = {"impl": "reference", "metric": metric, "value": v, "unit": "GFLOPS", "n_gpus": world,
            "steps": args.steps, "warmup": max(args.warmup, 3), "ms_per_step": dt * 1e3, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": args.dtype, "data": "synthetic",
            "config": {"workload": workload, "matrix": CONFIG_DOC.get(args.config, args.config), "nnz": nnz},
            "cpu_baseline": {"value": v, "unit": "GFLOPS", "cores": used, "kind": "oracle",
                             "sample": f"every {stride}th row ({S.m} rows, {S.nnz} nnz) per step, "
                                       f"double-double CSR loop over {used} OpenMP threads"},
            "e2e": {"value": v, "unit": "GFLOPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line))


if __name__ == "__main__":
    main()
