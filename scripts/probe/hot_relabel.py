"""Probe: does compacting the most-referenced ("hot") columns of x cut C3's x re-fetch?

Relabels the columns of the C3 matrix so the H most referenced columns take ids 0..H-1 (in
ascending original order) and the others keep their relative order after them; x is permuted
the same way, so y is unchanged.  Times dasp_long_kernel / dasp_main_kernel on the original and
on each relabelled matrix, and the cost of a device gather of H entries (what a plan-side "hot
x" copy would cost per SpMV).  Experiment only: prints one JSON line per case.
"""
import json
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.join(os.path.dirname(__file__), "..", ".."))
import synth  # noqa: E402
from paper_conf_sc_lu023_b200 import dasp  # noqa: E402


def time_plan(A, x, dtype, steps=200):
    plan = dasp.dasp_plan_create(A.row_ptr, A.col, A.val, A.m, A.n, dtype, device=0)
    xd = torch.from_numpy(x).cuda()
    yd = torch.zeros(A.m, dtype=torch.float64, device="cuda")
    s = torch.cuda.current_stream()
    for _ in range(10):
        dasp.dasp_spmv(plan, xd, yd, 1.0, 0.0, s, check=False)
    torch.cuda.synchronize()
    dasp.dasp_plan_set_timing(plan, steps)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    for _ in range(steps):
        dasp.dasp_spmv(plan, xd, yd, 1.0, 0.0, s, check=False)
    e1.record(s)
    torch.cuda.synchronize()
    k = dasp.dasp_plan_read_timing(plan)
    out = {"ms_step": e0.elapsed_time(e1) / steps}
    for name, (ms, n) in k.items():
        if n:
            out[name] = ms / n
    y = yd.cpu().numpy()
    plan.destroy()
    return out, y


def main():
    cfg = sys.argv[1] if len(sys.argv) > 1 else "c3"
    scale = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
    hs = [int(h) for h in sys.argv[3].split(",")] if len(sys.argv) > 3 else [250_000, 1_000_000, 2_000_000, 4_000_000]
    A = synth.generate(synth.config(cfg, scale=scale))
    x = synth.vector(101, A.n)
    base, y0 = time_plan(A, x, "f64")
    print(json.dumps({"case": "original", **base}), flush=True)
    cnt = np.bincount(A.col, minlength=A.n)
    order = np.argsort(-cnt, kind="stable")
    lens = np.diff(A.row_ptr)
    rows = torch.repeat_interleave(torch.arange(A.m, device="cuda"), torch.from_numpy(lens).cuda())
    for H in hs:
        hot = np.sort(order[:H])
        is_hot = np.zeros(A.n, dtype=bool)
        is_hot[hot] = True
        newid = np.empty(A.n, dtype=np.int64)
        newid[hot] = np.arange(H)
        cold = np.nonzero(~is_hot)[0]
        newid[cold] = H + np.arange(len(cold))
        nc = torch.from_numpy(newid[A.col]).cuda()
        key = rows * (1 << 24) + nc
        key, perm = torch.sort(key)
        col2 = (key & ((1 << 24) - 1)).to(torch.int32).cpu().numpy()
        val2 = A.val[perm.cpu().numpy()]
        inv = np.empty(A.n, dtype=np.int64)
        inv[newid] = np.arange(A.n)
        x2 = x[inv]
        B = synth.CSR(A.m, A.n, A.row_ptr, col2, val2)
        t, y = time_plan(B, x2, "f64")
        err = float(np.max(np.abs(y - y0)))
        # per-SpMV cost of building a compact hot copy on the device: xh[k] = x[hot[k]]
        xd = torch.from_numpy(x).cuda()
        hd = torch.from_numpy(hot.astype(np.int64)).cuda()
        for _ in range(5):
            torch.index_select(xd, 0, hd)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(50):
            torch.index_select(xd, 0, hd)
        e1.record()
        torch.cuda.synchronize()
        print(json.dumps({"case": f"hot {H}", **t, "max_abs_diff": err,
                          "hot_gather_ms": e0.elapsed_time(e1) / 50}), flush=True)
        del nc, key, perm


if __name__ == "__main__":
    main()
