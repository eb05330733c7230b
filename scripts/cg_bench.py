#!/usr/bin/env python3
"""f4 measurement: conjugate gradient on the SPD 27-point stencil (C2 pattern,
VAL_SPD values), end to end including the format build, with the SpMV's share of the solve.

    python scripts/cg_bench.py [--scale S] [--tol T]   -> one JSON line on stdout
"""
import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--scale", type=float, default=1.0)
    ap.add_argument("--tol", type=float, default=1e-10)
    ap.add_argument("--maxiter", type=int, default=2000)
    args = ap.parse_args()
    import torch
    import synth
    from paper_conf_sc_lu023_b200 import dasp
    from paper_conf_sc_lu023_b200.solvers import conjugate_gradient
    dev = torch.device("cuda", 0)
    spec = synth.config("c2", val_mode=synth.VAL_SPD, scale=args.scale)
    A = synth.generate(spec)
    d_rp = torch.from_numpy(A.row_ptr).to(dev)
    d_col = torch.from_numpy(A.col).to(dev)
    d_val = torch.from_numpy(A.val).to(dev)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    plan = dasp.dasp_plan_create_device(d_rp, d_col, d_val, A.m, A.n, "f64", device=0)
    torch.cuda.synchronize()
    first_build_wall = time.perf_counter() - t0       # includes CUDA lazy loading of the builder kernels
    first_build_ms = plan.info["build_ms"]
    plan.destroy()
    t0 = time.perf_counter()
    plan = dasp.dasp_plan_create_device(d_rp, d_col, d_val, A.m, A.n, "f64", device=0)
    torch.cuda.synchronize()
    build_wall = time.perf_counter() - t0
    del d_rp, d_col, d_val
    t0 = time.perf_counter()
    hplan = dasp.dasp_plan_create(A.row_ptr, A.col, A.val, A.m, A.n, "f64", device=0)
    host_build_wall = time.perf_counter() - t0
    hplan.destroy()
    ones = torch.ones(A.m, dtype=torch.float64, device=dev)
    b = torch.empty_like(ones)
    dasp.dasp_spmv(plan, ones, b)                     # b = A*1: the solution is all ones
    conjugate_gradient(plan, b, tol=args.tol, maxiter=5)   # warm-up (allocator, kernels)
    torch.cuda.synchronize()
    dasp.dasp_plan_set_timing(plan, args.maxiter + 10)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    res = conjugate_gradient(plan, b, tol=args.tol, maxiter=args.maxiter)
    e1.record()
    torch.cuda.synchronize()
    solve_ms = e0.elapsed_time(e1)
    kern = dasp.dasp_plan_read_timing(plan)
    spmv_ms = sum(ms for ms, n in kern.values())
    err = float(torch.max(torch.abs(res.x - ones)))
    line = {"workload": f"CG on c2{'' if args.scale == 1.0 else '@' + str(args.scale)} (VAL_SPD: -1 off-diagonal, "
                        "L+0.5 diagonal)", "m": A.m, "nnz": A.nnz, "iterations": res.iterations,
            "converged": res.converged, "residual": res.residual_norm, "max_abs_error_vs_ones": err,
            "gpu_build_ms": plan.info["build_ms"], "gpu_build_wall_ms": build_wall * 1e3,
            "first_gpu_build_ms": first_build_ms, "first_gpu_build_wall_ms": first_build_wall * 1e3,
            "host_build_wall_ms": host_build_wall * 1e3, "solve_ms": solve_ms,
            "ms_per_iteration": solve_ms / max(res.iterations, 1),
            "spmv_ms_total": spmv_ms, "spmv_share_of_solve": spmv_ms / solve_ms,
            "spmv_gflops": 2.0 * A.nnz * res.iterations / (spmv_ms * 1e-3) / 1e9 if spmv_ms else None,
            "end_to_end_ms_incl_gpu_build": solve_ms + plan.info["build_ms"],
            "build_share_of_end_to_end": plan.info["build_ms"] / (solve_ms + plan.info["build_ms"])}
    print(json.dumps(line))


if __name__ == "__main__":
    main()
