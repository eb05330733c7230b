"""Random 8-byte gather throughput (G gathers/s = G sectors/s) vs the gathered footprint, on B200.
The ceiling of scattered x gathers: every gather is one 32-B sector request to L2."""
import ctypes
import json
import os
import subprocess

import torch

HERE = os.path.dirname(os.path.abspath(__file__))
SO = os.path.join(HERE, "libl2peak.so")
if not os.path.exists(SO):
    subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-shared", "-Xcompiler",
                           "-fPIC", "-o", SO, os.path.join(HERE, "l2peak.cu")])
lib = ctypes.CDLL(SO)
lib.l2peak_run.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_void_p,
                           ctypes.c_void_p]
out = torch.zeros(1, dtype=torch.float64, device="cuda")
s = torch.cuda.current_stream()
res = []
for mb in (4, 16, 32, 48, 64, 96, 128, 256, 1024):
    n = mb * (1 << 20) // 8
    x = torch.rand(n, dtype=torch.float64, device="cuda")
    for mlp in (8, 16):
        for bps in (8, 16):
            blocks, iters = 148 * bps, 64
            lib.l2peak_run(x.data_ptr(), n, blocks, 4, mlp, out.data_ptr(), s.cuda_stream)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            lib.l2peak_run(x.data_ptr(), n, blocks, iters, mlp, out.data_ptr(), s.cuda_stream)
            e1.record()
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1)
            g = blocks * 256 * iters * mlp / (ms * 1e-3) / 1e9
            res.append({"footprint_mb": mb, "mlp": mlp, "blocks_per_sm": bps, "ms": ms, "Ggathers_per_s": g,
                        "sector_TBps": g * 32 / 1e3})
            print(json.dumps(res[-1]), flush=True)
    del x
