"""Row-slab iteration on the GPU (world size 1 here: one GPU per gpurun box): the NCCL path and
the fused scatter path (symmetric memory + dasp_spmv_scatter + device barrier) against K oracle
iterations.  The multi-rank host logic is covered on CPU by tests/test_multigpu.py."""
import socket

import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def pg():
    import torch.distributed as dist
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    torch.cuda.set_device(0)
    dist.init_process_group("nccl", init_method=f"tcp://127.0.0.1:{port}", rank=0, world_size=1,
                            device_id=torch.device("cuda", 0))
    yield dist
    dist.destroy_process_group()


@pytest.mark.parametrize("fused", [False, True])
def test_slab_iteration_world1(pg, fused):
    from paper_conf_sc_lu023_b200.multigpu import SlabSpMV, build_slab
    spec = synth.config("c5", scale=4e-4)
    lens = synth.row_lengths(spec)
    slab = build_slab(lambda r0, nr: synth.generate(spec, r0, nr), lens, 0, 1)
    it = SlabSpMV(slab, 1, 0, "cuda:0", fused=fused)
    x0 = synth.vector(61, spec.n)
    it.set_x(x0)
    alpha = 1.0 / slab.inf_norm
    for _ in range(3):
        it.step(alpha)
    torch.cuda.synchronize()
    got = it.x_global()
    A = synth.generate(spec)
    x = x0
    for _ in range(3):
        x_new, s = oracle.spmv_csr(A, x, alpha=alpha)
        x = x_new
    # each iterate is within tolerance of the oracle applied to the GPU's previous iterate; after
    # three steps of a norm-1 map the accumulated difference stays tiny
    assert np.allclose(got, x, rtol=0, atol=1e-12)


@pytest.mark.parametrize("tdt", ["float64", "float32", "float16"])
def test_gather_halo_kernel_bit_exact(tdt):
    from paper_conf_sc_lu023_b200 import dasp
    rng = np.random.default_rng(3)
    src = torch.from_numpy(rng.standard_normal(100_003).astype(tdt)).cuda()
    for n in (0, 1, 257, 300_001):
        idx = torch.from_numpy(rng.integers(0, src.numel(), n).astype(np.int32)).cuda()
        out = torch.full((n,), -7.0, dtype=src.dtype, device="cuda")
        dasp.dasp_gather_halo(src, idx, out)
        torch.cuda.synchronize()
        assert torch.equal(out.cpu(), src.cpu()[idx.cpu().long()])


def test_gather_halo_bad_args():
    from paper_conf_sc_lu023_b200 import dasp
    L = dasp.lib()
    BAD = dasp.STATUS.index("DASP_ERR_INVALID_ARG")
    assert L.dasp_gather_halo(None, None, 5, None, 8, None) == BAD
    assert L.dasp_gather_halo(None, None, -1, None, 8, None) == BAD
    x = torch.zeros(4, dtype=torch.float64, device="cuda")
    i = torch.zeros(4, dtype=torch.int32, device="cuda")
    assert L.dasp_gather_halo(x.data_ptr(), i.data_ptr(), 4, x.data_ptr(), 3, None) == BAD
    assert L.dasp_gather_halo(None, None, 0, None, 8, None) == 0


@pytest.mark.parametrize("cfg", [("c3", None, 0, 0.004), ("c2", None, 0, 0.25), ("c5", None, 0, 4e-4)])
def test_halo_split_plans_match_oracle(cfg):
    """The f1 halo split on the GPU, one slab at a time: y_p = A_loc x_p (beta 0) then
    y_p += A_rem h with h packed from x by dasp_gather_halo (beta 1) == the oracle rows."""
    from paper_conf_sc_lu023_b200 import dasp
    from paper_conf_sc_lu023_b200.multigpu import slab_bounds, split_halo
    spec = synth.config(*cfg)
    A = synth.generate(spec)
    P = 3
    starts = slab_bounds(np.diff(A.row_ptr), P)
    x = synth.vector(17, spec.n)
    xd = torch.from_numpy(x).cuda()
    for rank in range(P):
        r0, r1 = int(starts[rank]), int(starts[rank + 1])
        rp = A.row_ptr[r0:r1 + 1] - A.row_ptr[r0]
        col = A.col[A.row_ptr[r0]:A.row_ptr[r1]]
        val = A.val[A.row_ptr[r0]:A.row_ptr[r1]]
        sp = split_halo(rp, col, val, starts, rank)
        rows = r1 - r0
        pl = dasp.dasp_plan_create(sp.loc_row_ptr, sp.loc_col, sp.loc_val, rows, rows, "f64")
        y = torch.full((rows,), 123.0, dtype=torch.float64, device="cuda")
        dasp.dasp_spmv(pl, xd[r0:r1].contiguous(), y, 1.0, 0.0)
        if len(sp.halo):
            pr = dasp.dasp_plan_create(sp.rem_row_ptr, sp.rem_col, sp.rem_val, rows, len(sp.halo), "f64")
            h = torch.empty(len(sp.halo), dtype=torch.float64, device="cuda")
            dasp.dasp_gather_halo(xd, torch.from_numpy(sp.halo.astype(np.int32)).cuda(), h)
            dasp.dasp_spmv(pr, h, y, 1.0, 1.0)
        torch.cuda.synchronize()
        y_ref, s = oracle.spmv(rp, col, val, x)
        assert oracle.tolerance_ok(y.cpu().numpy(), y_ref, s).all()


def test_halo_iteration_world1(pg):
    from paper_conf_sc_lu023_b200.multigpu import HaloSlabSpMV, build_slab
    spec = synth.config("c5", scale=4e-4)
    lens = synth.row_lengths(spec)
    slab = build_slab(lambda r0, nr: synth.generate(spec, r0, nr), lens, 0, 1, remap=False)
    it = HaloSlabSpMV(slab, 1, 0, "cuda:0")
    assert it.n_halo == 0 and it.plan_rem is None
    x0 = synth.vector(61, spec.n)
    it.set_x(x0)
    alpha = 1.0 / slab.inf_norm
    for _ in range(3):
        it.step(alpha)
    torch.cuda.synchronize()
    A = synth.generate(spec)
    x = x0
    for _ in range(3):
        x, _ = oracle.spmv_csr(A, x, alpha=alpha)
    assert np.allclose(it.x_global(), x, rtol=0, atol=1e-12)


def test_slab_iteration_world1_f32(pg):
    """The row-slab iteration on an FP32 plan (x and y both float32, R29): three steps against the oracle
    applied to the GPU's own previous iterate, each within the FP32 tolerance."""
    from paper_conf_sc_lu023_b200.multigpu import SlabSpMV, build_slab
    spec = synth.config("c5", scale=4e-4)
    lens = synth.row_lengths(spec)
    slab = build_slab(lambda r0, nr: synth.generate(spec, r0, nr), lens, 0, 1)
    slab.val = slab.val.astype(np.float32)
    it = SlabSpMV(slab, 1, 0, "cuda:0", dtype="f32")
    assert it.x[0].dtype == torch.float32
    x = synth.vector(62, spec.n).astype(np.float32)
    it.set_x(x)
    alpha = 1.0 / slab.inf_norm
    A = synth.generate(spec)
    val = A.val.astype(np.float32).astype(np.float64)
    for _ in range(3):
        it.step(alpha)
        torch.cuda.synchronize()
        got = it.x_global().astype(np.float64)
        ref, s = oracle.spmv(A.row_ptr, A.col, val, x.astype(np.float64), alpha=alpha)
        assert oracle.tolerance_ok(got, ref, s, "f32").all()
        x = got.astype(np.float32)
