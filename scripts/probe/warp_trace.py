"""Probe (experiment build DASP_EXP_TRACE=1): per-warp phase timestamps of dasp_main_kernel.

For each main-kernel warp the first work item records clock64 at start, when its stream loads
have landed, when its x gathers have landed (first row-block / pass / tile pair), at the end,
plus globaltimer start / end and the SM.  Prints per-kind medians / percentiles in microseconds.

    DASP_LIB=build/libdasp_DASP_EXP_TRACE=1.so python scripts/probe/warp_trace.py c3
"""
import ctypes
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.join(os.path.dirname(__file__), "..", ".."))
import synth  # noqa: E402
from paper_conf_sc_lu023_b200 import dasp  # noqa: E402

KIND = {1: "short pair", 2: "wide medium", 3: "narrow (lane/row)", 4: "mid (2 lanes/row)"}


def main():
    cfg = sys.argv[1] if len(sys.argv) > 1 else "c3"
    scale = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
    A = synth.generate(synth.config(cfg, scale=scale))
    plan = dasp.dasp_plan_create(A.row_ptr, A.col, A.val, A.m, A.n, "f64", device=0)
    xd = torch.from_numpy(synth.vector(101, A.n)).cuda()
    yd = torch.zeros(A.m, dtype=torch.float64, device="cuda")
    lib = dasp.lib()
    rd = lib.dasp_exp_trace_read
    rd.argtypes = [ctypes.c_void_p, ctypes.c_int64, ctypes.c_int]
    nwarps = 1 << 20
    buf = np.zeros(nwarps * 8, dtype=np.uint64)
    for _ in range(5):
        dasp.dasp_spmv(plan, xd, yd)
    torch.cuda.synchronize()
    assert rd(buf.ctypes.data, buf.nbytes, 1) == 0
    dasp.dasp_spmv(plan, xd, yd)
    torch.cuda.synchronize()
    assert rd(buf.ctypes.data, buf.nbytes, 0) == 0
    T = buf.reshape(nwarps, 8).astype(np.int64)
    T = T[T[:, 0] > 0]
    clk_mhz = torch.cuda.clock_rate() if hasattr(torch.cuda, "clock_rate") else 1965
    # cycles -> us at the SM clock inferred from globaltimer over the same spans
    span_ns = (T[:, 6] - T[:, 5]).astype(np.float64)
    span_cyc = (T[:, 4] - T[:, 1]).astype(np.float64)
    ok = span_ns > 500
    ghz = np.median(span_cyc[ok] / span_ns[ok]) if ok.any() else clk_mhz / 1e3
    t0 = T[:, 5].min()
    out = {"config": cfg, "warps_traced": int(len(T)), "sm_ghz_inferred": float(ghz),
           "kernel_span_us": float((T[:, 6].max() - t0) / 1e3)}
    for k, name in KIND.items():
        S = T[T[:, 0] == k]
        if not len(S):
            continue
        d_stream = (S[:, 2] - S[:, 1]) / ghz / 1e3
        d_gather = (S[:, 3] - S[:, 2]) / ghz / 1e3
        d_total = (S[:, 4] - S[:, 1]) / ghz / 1e3
        start = (S[:, 5] - t0) / 1e3

        def q(a):
            return [round(float(v), 3) for v in np.percentile(a, [10, 50, 90, 99])]
        out[name] = {"warps": int(len(S)), "stream_us_p10_50_90_99": q(d_stream), "gather_us": q(d_gather),
                     "warp_total_us": q(d_total), "start_us_min_max": [float(start.min()), float(start.max())]}
    # resident warps over time (globaltimer): how many warps are alive at each microsecond
    edges = np.arange(0, out["kernel_span_us"] + 1, 1.0)
    alive = np.zeros(len(edges))
    s_us, e_us = (T[:, 5] - t0) / 1e3, (T[:, 6] - t0) / 1e3
    for a, b in zip(s_us, e_us):
        alive[int(a):int(b) + 1] += 1
    out["alive_warps_p10_50_90"] = [float(v) for v in np.percentile(alive[: max(1, len(alive) - 1)], [10, 50, 90])]
    print(json.dumps(out))


if __name__ == "__main__":
    main()
