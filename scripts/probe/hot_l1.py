"""Probe (experiment build DASP_EXP_HOT=1): compact the H most referenced columns of C3 into
x[0..H) (offline relabel, as scripts/probe/hot_relabel.py) AND keep them in L1 (L1::evict_last
gathers for columns < H, evict_first for the rest).  Times the long / main kernels per H."""
import ctypes
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.join(os.path.dirname(__file__), "..", ".."))
import synth  # noqa: E402
from paper_conf_sc_lu023_b200 import dasp  # noqa: E402
from hot_relabel import time_plan  # noqa: E402


def relabel(A, x, H, order, rows):
    hot = np.sort(order[:H])
    is_hot = np.zeros(A.n, dtype=bool)
    is_hot[hot] = True
    newid = np.empty(A.n, dtype=np.int64)
    newid[hot] = np.arange(H)
    cold = np.nonzero(~is_hot)[0]
    newid[cold] = H + np.arange(len(cold))
    nc = torch.from_numpy(newid[A.col]).cuda()
    key, perm = torch.sort(rows * (1 << 24) + nc)
    col2 = (key & ((1 << 24) - 1)).to(torch.int32).cpu().numpy()
    val2 = A.val[perm.cpu().numpy()]
    inv = np.empty(A.n, dtype=np.int64)
    inv[newid] = np.arange(A.n)
    return synth.CSR(A.m, A.n, A.row_ptr, col2, val2), x[inv]


def main():
    set_hot = dasp.lib().dasp_exp_set_hot
    set_hot.argtypes = [ctypes.c_int32]
    A = synth.generate(synth.config(sys.argv[1] if len(sys.argv) > 1 else "c3"))
    x = synth.vector(101, A.n)
    cnt = np.bincount(A.col, minlength=A.n)
    order = np.argsort(-cnt, kind="stable")
    rows = torch.repeat_interleave(torch.arange(A.m, device="cuda"), torch.from_numpy(np.diff(A.row_ptr)).cuda())
    set_hot(0)
    base, y0 = time_plan(A, x, "f64")
    print(json.dumps({"case": "original, all evict_first", **base}), flush=True)
    for H in (4096, 16384, 65536, 262144):
        B, xb = relabel(A, x, H, order, rows)
        for h in (0, H):
            set_hot(h)
            t, y = time_plan(B, xb, "f64")
            print(json.dumps({"case": f"hot {H} compact, L1 evict_last below {h}", **t,
                              "max_abs_diff": float(np.max(np.abs(y - y0)))}), flush=True)


if __name__ == "__main__":
    main()
