"""f2: the GPU-side builder (dasp_plan_create_device) writes exactly the bytes of the host builder
and of the oracle's literal builder, for every class, both dtypes, several panel sizes and knob
settings; plans built on the device compute the same SpMV."""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_sc_lu023_b200 import dasp  # noqa: E402


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def device_plan(A, dt, **kw):
    val = A.val.astype({"f64": np.float64, "f16": np.float16, "f32": np.float32}[dt])
    return dasp.dasp_plan_create_device(torch.from_numpy(A.row_ptr).cuda(), torch.from_numpy(A.col).cuda(),
                                        torch.from_numpy(np.ascontiguousarray(val)).cuda(), A.m, A.n, dt, **kw)


def cases():
    yield "c1a", synth.generate(synth.config("c1a"))
    yield "c1b", synth.generate(synth.config("c1b"))
    yield "c3s", synth.generate(synth.config("c3", scale=0.004))
    yield "c5s", synth.generate(synth.config("c5", scale=2e-5))
    yield "c6s", synth.generate(synth.config("c6", scale=0.01))
    lens = [0, 1, 2, 3, 4, 5, 9, 17, 31, 33, 64, 255, 256, 257, 300, 1000, 2049, 4, 4, 3, 2, 1, 1, 1, 7, 6]
    yield "lens", synth.from_lengths(lens * 5, n=3000)
    yield "empty", synth.CSR(7, 5, np.zeros(8, dtype=np.int64), np.zeros(0, np.int32), np.zeros(0))


CASES = list(cases())


@pytest.mark.parametrize("dt", ["f64", "f16", "f32"])
@pytest.mark.parametrize("panel", [-1, 97, 1000])
@pytest.mark.parametrize("name,A", CASES, ids=[c[0] for c in CASES])
def test_device_builder_bytes(name, A, dt, panel):
    dplan = device_plan(A, dt, panel_rows=panel)
    info = dplan.info
    ref = oracle.build(A, dt, panel_rows=info["panel_rows"])
    hplan = dasp.dasp_plan_create(A.row_ptr, A.col, A.val, A.m, A.n, dt, device=-1, panel_rows=panel)
    hinfo = hplan.info
    for k in ["n_empty", "n_len1", "n_len2", "n_len3", "n_len4", "row_medium", "row_long", "rowblocks", "n_groups",
              "n_groups_padded", "tiles_13", "tiles_4", "tiles_22", "tiles_single", "nnz_long_new", "nnz_reg_new",
              "nnz_irreg", "nnz_short_new", "nnz_long", "nnz_medium", "nnz_short", "panel_rows", "n_panels",
              "medium_rb_per_warp"]:
        assert info[k] == hinfo[k], k
    for arr in dasp.ARRAYS:
        got = dasp.dasp_plan_copy_array(dplan, arr)
        assert np.array_equal(got, ref.arrays[arr]), arr
        assert np.array_equal(got, dasp.dasp_plan_copy_array(hplan, arr)), arr


@pytest.mark.parametrize("max_len,tau", [(16, 0.75), (1000, 0.5), (256, 1.0)])
def test_device_builder_knobs(max_len, tau):
    A = synth.generate(synth.config("c1b"))
    dplan = device_plan(A, "f64", max_len=max_len, threshold=tau, panel_rows=700)
    ref = oracle.build(A, "f64", panel_rows=700, max_len=max_len, tau=tau)
    for arr in dasp.ARRAYS:
        assert np.array_equal(dasp.dasp_plan_copy_array(dplan, arr), ref.arrays[arr]), arr


@pytest.mark.parametrize("dt", ["f64", "f16"])
def test_device_built_plan_spmv(dt):
    A = synth.generate(synth.config("c3", scale=0.01, val_mode=synth.VAL_INT))
    x = synth.vector(91, A.n, synth.VAL_INT)
    plan = device_plan(A, dt)
    xd = torch.from_numpy(x.astype(np.float64 if dt == "f64" else np.float16)).cuda()
    y = torch.empty(A.m, dtype=torch.float64 if dt == "f64" else torch.float32, device="cuda")
    for v in [dasp.DASP_VARIANT_MMA, dasp.DASP_VARIANT_CUDACORE]:
        dasp.dasp_spmv(plan, xd, y, variant=v)
        torch.cuda.synchronize()
        val = A.val if dt == "f64" else A.val.astype(np.float16).astype(np.float64)
        xv = x if dt == "f64" else x.astype(np.float16).astype(np.float64)
        y_ref, _ = oracle.spmv(A.row_ptr, A.col, val, xv)
        assert np.array_equal(y.cpu().numpy().astype(np.float64), y_ref)


def test_device_builder_rejects_bad_csr():
    A = synth.generate(synth.config("c1a"))
    col = A.col.copy()
    col[3] = A.n + 5
    B = synth.CSR(A.m, A.n, A.row_ptr, col, A.val)
    with pytest.raises(dasp.DaspError) as e:
        device_plan(B, "f64")
    assert e.value.status == 2


def test_device_builder_full_size_matches_host():
    A = synth.generate(synth.config("c3"))
    dplan = device_plan(A, "f64")
    hplan = dasp.dasp_plan_create(A.row_ptr, A.col, A.val, A.m, A.n, "f64", device=-1)
    for arr in dasp.ARRAYS:
        assert np.array_equal(dasp.dasp_plan_copy_array(dplan, arr), dasp.dasp_plan_copy_array(hplan, arr)), arr
    # (the build time itself is reported by bench.py "preprocessing", not asserted here)


def test_device_builder_rejects_short_arrays_before_reading_them():
    """row_ptr[m] larger than the col / val arrays handed over (nnz = their length): INVALID_CSR is
    returned before any kernel reads past them, and the context stays usable."""
    A = synth.generate(synth.config("c1a"))
    rp = torch.from_numpy(A.row_ptr).cuda()
    short = A.nnz - 1000
    col = torch.from_numpy(A.col[:short].copy()).cuda()
    val = torch.from_numpy(A.val[:short].copy()).cuda()
    with pytest.raises(dasp.DaspError) as e:
        dasp.dasp_plan_create_device(rp, col, val, A.m, A.n, "f64")
    assert e.value.status == 2
    torch.cuda.synchronize()                      # no sticky fault
    plan = device_plan(A, "f64")
    assert plan.info["nnz"] == A.nnz
