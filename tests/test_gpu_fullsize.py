"""Full-size parity: the configurations bench.py times, in the launch configuration it times
(default plan, CUDA-core variant, beta = 0), checked against the CPU oracle on EVERY row
(Alg. 1, defines y for every row).

* C2 (27-point stencil 128^3), C2+ (162^3, 1.13e8 nnz) and C3 (power-law, 2.07e8 nnz) in FP64,
  FP16 and FP32: every row with the OpenMP copy of the oracle loop (oracle.spmv_mt).
* C5 at full size (4.29e9 nnz: 64-bit packed offsets everywhere, above 2^31 elements) in FP64:
  SURVEY.md §8(d)'s sample -- every 1024th row, every long row, and the first and last row of
  every panel -- against the oracle.
"""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_sc_lu023_b200 import dasp  # noqa: E402

NP_VAL = {"f64": np.float64, "f16": np.float16, "f32": np.float32}
_MATS = {}


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    yield
    _MATS.clear()


def matrix(name):
    if name not in _MATS:
        _MATS.clear()                      # one full-size matrix in host memory at a time
        _MATS[name] = synth.generate(synth.config(name))
    return _MATS[name]


def spmv_device(A, val, x, dt):
    plan = dasp.dasp_plan_create(A.row_ptr, A.col, val, A.m, A.n, dt, device=0)
    xd = torch.from_numpy(np.ascontiguousarray(x)).cuda()
    yd = torch.full((A.m,), float("nan"), dtype=torch.float64 if dt == "f64" else torch.float32, device="cuda")
    dasp.dasp_spmv(plan, xd, yd, 1.0, 0.0)
    torch.cuda.synchronize()
    y = yd.cpu().numpy().astype(np.float64)
    info = plan.info
    plan.destroy()
    del xd, yd
    torch.cuda.empty_cache()
    return y, info


@pytest.mark.parametrize("dt", ["f64", "f16", "f32"])
@pytest.mark.parametrize("name", ["c2", "c2big", "c3"])
def test_full_size_every_row(name, dt):
    A = matrix(name)
    val = A.val.astype(NP_VAL[dt])
    x = synth.vector(13, A.n).astype(NP_VAL[dt])
    y, info = spmv_device(A, val, x, dt)
    y_ref, s, _ = oracle.spmv_mt(A.row_ptr, A.col, val.astype(np.float64), x.astype(np.float64))
    ok = oracle.tolerance_ok(y, y_ref, s, dt)
    bad = np.flatnonzero(~ok)
    assert ok.all(), f"{name}/{dt}: {len(bad)} of {A.m} rows off, first {bad[:5]}: {y[bad[:5]]} vs {y_ref[bad[:5]]}"
    if name == "c3":   # every class is on the path that was checked
        assert info["row_long"] > 0 and info["row_medium"] > 0 and info["n_len1"] > 0 and info["n_empty"] == 0


def test_c5_full_size_sampled():
    """C5, 62.5M rows, 4.29e9 nonzeros, FP64, one B200 (the whole packed matrix resident): the rows
    of SURVEY.md §8(d)'s sample against the oracle."""
    _MATS.clear()
    spec = synth.config("c5")
    A = synth.generate(spec)
    assert A.nnz > 2 ** 31
    x = synth.vector(14, A.n)
    plan = dasp.dasp_plan_create(A.row_ptr, A.col, A.val, A.m, A.n, "f64", device=0)
    info = plan.info
    xd = torch.from_numpy(x).cuda()
    yd = torch.full((A.m,), float("nan"), dtype=torch.float64, device="cuda")
    dasp.dasp_spmv(plan, xd, yd, 1.0, 0.0)
    torch.cuda.synchronize()
    y = yd.cpu().numpy()
    plan.destroy()
    del xd, yd
    torch.cuda.empty_cache()
    lens = np.diff(A.row_ptr)
    pr = info["panel_rows"]
    firsts = np.arange(0, A.m, pr)
    lasts = np.minimum(firsts + pr, A.m) - 1
    rows = np.unique(np.concatenate([np.arange(0, A.m, 1024), np.flatnonzero(lens > 256), firsts, lasts]))
    starts, ends = A.row_ptr[rows], A.row_ptr[rows + 1]
    sub_rp = np.zeros(len(rows) + 1, dtype=np.int64)
    np.cumsum(ends - starts, out=sub_rp[1:])
    idx = np.repeat(starts - sub_rp[:-1], ends - starts) + np.arange(sub_rp[-1])
    y_ref, s, _ = oracle.spmv_mt(sub_rp, A.col[idx], A.val[idx], x)
    ok = oracle.tolerance_ok(y[rows], y_ref, s, "f64")
    assert ok.all(), f"{(~ok).sum()} of {len(rows)} sampled rows off"
    assert info["row_long"] > 0 and info["row_medium"] > 0 and info["n_len1"] > 0
    assert len(rows) > 60_000
    del A
