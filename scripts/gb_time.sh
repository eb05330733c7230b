#!/bin/bash
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
cat > /tmp/gbt.py <<'PY'
import time, numpy as np, torch, synth
from paper_conf_sc_lu023_b200 import dasp
for name in ["c3", "c2"]:
    A = synth.generate(synth.config(name))
    rp, col, val = (torch.from_numpy(a).cuda() for a in (A.row_ptr, A.col, A.val))
    for rep in range(3):
        torch.cuda.synchronize(); t = time.perf_counter()
        p = dasp.dasp_plan_create_device(rp, col, val, A.m, A.n, "f64")
        print(name, "device build", p.info["build_ms"], "wall", (time.perf_counter() - t) * 1e3, flush=True)
        del p
    t = time.perf_counter()
    h = dasp.dasp_plan_create(A.row_ptr, A.col, A.val, A.m, A.n, "f64")
    print(name, "host build", h.info["build_ms"], "upload", h.info["upload_ms"], "wall", (time.perf_counter() - t) * 1e3, flush=True)
PY
DASP_GB_TRACE=1 PYTHONPATH=$PWD timeout 600 python /tmp/gbt.py > gpurun_out/gbt.log 2>&1; tail -40 gpurun_out/gbt.log
