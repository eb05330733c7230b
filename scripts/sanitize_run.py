"""Workload for compute-sanitizer (scripts/sanitize.sh): every row class on small matrices, both
compute variants, all three dtypes, beta = 0 and beta != 0, the scatter epilogue, the host-buffer
calls, the device builder and the x-window staging instantiation.  Checks results against the oracle so a silent corruption fails too."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
import synth  # noqa: E402
from paper_conf_sc_lu023_b200 import dasp  # noqa: E402

NP = {"f64": np.float64, "f16": np.float16, "f32": np.float32}


def main():
    cases = {"c1b": synth.generate(synth.config("c1b")),
             "c3s": synth.generate(synth.config("c3", scale=0.004)),
             "c2s": synth.generate(synth.config("c2", scale=16 / 128))}
    for name, A in cases.items():
        x = synth.vector(3, A.n)
        y0 = synth.vector(4, A.m)
        for dt in ("f64", "f16", "f32"):
            val = A.val.astype(NP[dt])
            xv = x.astype(NP[dt])
            plan = dasp.dasp_plan_create(A.row_ptr, A.col, val, A.m, A.n, dt, device=0, panel_rows=700)
            xd = torch.from_numpy(xv).cuda()
            ydt = torch.float64 if dt == "f64" else torch.float32
            for v in (dasp.DASP_VARIANT_MMA, dasp.DASP_VARIANT_CUDACORE):
                for beta in (0.0, -0.5):
                    yd = torch.from_numpy(y0).to(ydt).cuda()
                    dasp.dasp_spmv(plan, xd, yd, 1.5, beta, variant=v)
                    torch.cuda.synchronize()
                    ref, s = oracle.spmv(A.row_ptr, A.col, val.astype(np.float64), xv.astype(np.float64), 1.5, beta,
                                         y0.astype(NP[dt] if dt != "f16" else np.float32).astype(np.float64))
                    assert oracle.tolerance_ok(yd.cpu().numpy().astype(np.float64), ref, s, dt).all(), (name, dt, v, beta)
            dst = [torch.zeros(A.m, dtype=ydt, device="cuda") for _ in range(3)]
            dasp.dasp_spmv_scatter(plan, xd, dst, 1.0, 0.0)
            yh = np.zeros(A.m, dtype=np.float64 if dt == "f64" else np.float32)
            dasp.dasp_spmv_host(plan, xv, yh)
            torch.cuda.synchronize()
            assert all(np.array_equal(d.cpu().numpy(), yh) for d in dst), (name, dt)
            dplan = dasp.dasp_plan_create_device(torch.from_numpy(A.row_ptr).cuda(), torch.from_numpy(A.col).cuda(),
                                                 torch.from_numpy(val).cuda(), A.m, A.n, dt, panel_rows=700)
            for arr in dasp.ARRAYS:
                assert np.array_equal(dasp.dasp_plan_copy_array(dplan, arr), dasp.dasp_plan_copy_array(plan, arr)), arr
            dplan.destroy()
            plan.destroy()
    # x-window staging instantiation (cp.async.bulk + mbarrier): stencil blocks, FP64 / FP32
    A = synth.generate(synth.config("c2", scale=0.25))
    x = synth.vector(5, A.n)
    for dt in ("f64", "f32"):
        val = A.val.astype(NP[dt])
        xv = x.astype(NP[dt])
        st = dasp.dasp_plan_create(A.row_ptr, A.col, val, A.m, A.n, dt, device=0, x_stage=2)
        pl = dasp.dasp_plan_create(A.row_ptr, A.col, val, A.m, A.n, dt, device=0, x_stage=1)
        assert st.info["x_stage_blocks"] > 0
        xd = torch.from_numpy(xv).cuda()
        ydt = torch.float64 if dt == "f64" else torch.float32
        ys, yp = torch.zeros(A.m, dtype=ydt, device="cuda"), torch.zeros(A.m, dtype=ydt, device="cuda")
        dasp.dasp_spmv(st, xd, ys, 1.0, 0.0)
        dasp.dasp_spmv(pl, xd, yp, 1.0, 0.0)
        torch.cuda.synchronize()
        assert torch.equal(ys, yp), dt
        st.destroy()
        pl.destroy()
    torch.cuda.synchronize()
    torch.cuda.empty_cache()   # torch's caching allocator keeps its blocks otherwise (reported as leaks)
    print("sanitize workload ok")


if __name__ == "__main__":
    main()
