"""Production builder (libdasp.so, host-only plans) vs the oracle's literal builder: byte for byte
(north_star: "bit-exact for the format builder's indexing and permutation"),
plus the C-ABI surface that needs no GPU.  CPU only."""
import ctypes

import numpy as np
import pytest

import oracle
import synth
from paper_conf_sc_lu023_b200 import dasp
from tests.format_decode import check_roundtrip

COUNT_MAP = {"n0": "n_empty", "n1": "n_len1", "n2": "n_len2", "n3": "n_len3", "n4": "n_len4",
             "row_medium": "row_medium", "row_long": "row_long", "nrb": "rowblocks", "n_groups": "n_groups",
             "n_groups_padded": "n_groups_padded", "t13": "tiles_13", "t4": "tiles_4", "t22": "tiles_22",
             "ts": "tiles_single", "nnz_long_new": "nnz_long_new", "nnz_reg_new": "nnz_reg_new",
             "nnz_irreg": "nnz_irreg", "nnz_short_new": "nnz_short_new", "m": "m", "n": "n", "nnz": "nnz",
             "panel_rows": "panel_rows", "n_panels": "n_panels"}


def host_plan(A, dt, **kw):
    val = {"f64": A.val, "f16": A.val.astype(np.float16), "f32": A.val.astype(np.float32)}[dt]
    return dasp.dasp_plan_create(A.row_ptr, A.col, val, A.m, A.n, dt, device=-1, **kw)


def matrices():
    yield "c1a", synth.generate(synth.config("c1a"))
    yield "c1b", synth.generate(synth.config("c1b"))
    yield "c2s", synth.generate(synth.config("c2", scale=16 / 128))
    yield "c3s", synth.generate(synth.config("c3", scale=0.002))
    yield "c5s", synth.generate(synth.config("c5", scale=2e-5))
    yield "c6s", synth.generate(synth.config("c6", scale=0.01))
    lens = [0, 1, 2, 3, 4, 5, 9, 17, 31, 33, 64, 255, 256, 257, 300, 1000, 2049, 4, 4, 3, 2, 1, 1, 1, 7, 6]
    yield "lens", synth.from_lengths(lens * 5, n=3000)


CASES = list(matrices())


@pytest.mark.parametrize("panel", [0, -1, 1, 97, 1000])
@pytest.mark.parametrize("dt", ["f64", "f16", "f32"])
@pytest.mark.parametrize("name,A", CASES, ids=[c[0] for c in CASES])
def test_builder_bit_exact_vs_oracle(name, A, dt, panel):
    if panel in (1, 97) and A.m > 20000:
        pytest.skip("tiny panels on the small matrices only")
    plan = host_plan(A, dt, panel_rows=panel)
    ref = oracle.build(A, dt, panel_rows=plan.info["panel_rows"])
    info = plan.info
    for k, v in ref.counts.items():
        assert info[COUNT_MAP[k]] == v, k
    for arr in dasp.ARRAYS:
        got = dasp.dasp_plan_copy_array(plan, arr)
        want = ref.arrays[arr]
        assert got.shape == want.shape, arr
        assert np.array_equal(got, want), arr


@pytest.mark.parametrize("dt", ["f64", "f16", "f32"])
@pytest.mark.parametrize("panel", [-1, 333])
def test_builder_roundtrip_via_abi(dt, panel):
    A = synth.generate(synth.config("c1b"))
    plan = host_plan(A, dt, panel_rows=panel)
    info = plan.info
    counts = {k: info[v] for k, v in COUNT_MAP.items()}

    def get(name):
        b = dasp.dasp_plan_copy_array(plan, name)
        if name.endswith("_val"):
            return b.view({"f64": np.float64, "f16": np.float16, "f32": np.float32}[dt])
        if name in ("group_ptr", "rb_ptr", "irr_ptr", "panels"):
            return b.view(np.int64)
        return b.view(np.int32)
    check_roundtrip(A, counts, get, dt)
    assert info["nnz_long"] + info["nnz_medium"] + info["nnz_short"] == A.nnz


def test_builder_threads_deterministic():
    A = synth.generate(synth.config("c3", scale=0.004))
    for panel in [-1, 4096, 50]:    # inner-parallel and one-thread-per-panel paths
        p1, p8 = host_plan(A, "f64", num_threads=1, panel_rows=panel), host_plan(A, "f64", num_threads=8, panel_rows=panel)
        for arr in dasp.ARRAYS:
            assert np.array_equal(dasp.dasp_plan_copy_array(p1, arr), dasp.dasp_plan_copy_array(p8, arr)), arr


def test_exports_every_header_symbol():
    import re
    hdr = open(__file__.replace("tests/test_builder.py", "include/dasp.h")).read()
    declared = set(re.findall(r"\b(dasp_[a-z_]+)\s*\(", hdr))
    assert declared == set(dasp.EXPORTS)
    lib = ctypes.CDLL(dasp.LIB_PATH)
    for s in declared:
        assert getattr(lib, s) is not None


def test_status_strings_and_errors():
    L = dasp.lib()
    assert L.dasp_status_string(2) == b"DASP_ERR_INVALID_CSR"
    A = synth.generate(synth.config("c1a"))
    bad = A.row_ptr.copy()
    bad[5], bad[6] = bad[6], bad[5] - 1            # decreasing row_ptr
    with pytest.raises(dasp.DaspError) as e:
        dasp.dasp_plan_create(bad, A.col, A.val, A.m, A.n, "f64", device=-1)
    assert e.value.status == 2
    col = A.col.copy()
    col[7] = A.n                                    # column out of range
    with pytest.raises(dasp.DaspError) as e:
        dasp.dasp_plan_create(A.row_ptr, col, A.val, A.m, A.n, "f64", device=-1)
    assert e.value.status == 2
    with pytest.raises(dasp.DaspError) as e:
        dasp.dasp_plan_create(A.row_ptr, A.col, A.val, A.m, -1, "f64", device=-1)
    assert e.value.status == 1
    h = ctypes.c_void_p()
    assert L.dasp_plan_create(None, 1, 1, 0, None, None, None, 0, None) == 1
    assert L.dasp_plan_create(ctypes.byref(h), 1, 1, 0, None, None, None, 0, None) == 1
    # spmv on a host-only plan is unsupported, not a crash
    p = dasp.dasp_plan_create(A.row_ptr, A.col, A.val, A.m, A.n, "f64", device=-1)
    assert L.dasp_spmv(p.handle, 16, 32, 1.0, 0.0, None) == 5
    assert L.dasp_spmv(None, 16, 32, 1.0, 0.0, None) == 1


def test_degenerate_plans():
    for m, n in [(0, 0), (5, 3), (3, 0)]:
        rp = np.zeros(m + 1, dtype=np.int64)
        p = dasp.dasp_plan_create(rp, np.zeros(0, np.int32), np.zeros(0), m, n, "f64", device=-1)
        info = p.info
        assert info["n_empty"] == m and info["nnz"] == 0 and info["launches_per_spmv"] == (1 if m else 0)


def test_partition_rows_balanced():
    A = synth.generate(synth.config("c3", scale=0.004))
    for P in [1, 2, 3, 4, 8]:
        s = dasp.dasp_partition_rows(A.row_ptr, P)
        assert s[0] == 0 and s[-1] == A.m and (np.diff(s) >= 0).all()
        for q in range(1, P):   # first row whose start offset reaches q*nnz/P
            target = (A.nnz * q) // P
            assert A.row_ptr[s[q]] >= target and (s[q] == 0 or A.row_ptr[s[q] - 1] < target)


def test_remap_columns_padded_layout():
    A = synth.generate(synth.config("c1b"))
    s = dasp.dasp_partition_rows(A.row_ptr, 3)
    col = A.col.copy()
    S = dasp.dasp_remap_columns(col, s)
    assert S == np.diff(s).max()
    owner = np.searchsorted(s, A.col, side="right") - 1
    assert np.array_equal(col, owner * S + (A.col - s[owner]))


# f3: MAX_LEN ("adjustable") and tau ("customized") as plan options
@pytest.mark.parametrize("dt", ["f64", "f16"])
@pytest.mark.parametrize("max_len,tau", [(16, 0.75), (64, 0.5), (1000, 0.9), (256, 1.0), (4, 0.75)])
def test_builder_knobs_bit_exact(dt, max_len, tau):
    A = synth.generate(synth.config("c1b"))
    plan = host_plan(A, dt, max_len=max_len, threshold=tau, panel_rows=1500)
    info = plan.info
    assert info["max_len"] == max_len and info["threshold"] == tau
    ref = oracle.build(A if dt == "f64" else A.to_fp16(), dt, panel_rows=1500, max_len=max_len, tau=tau)
    for k, v in ref.counts.items():
        assert info[COUNT_MAP[k]] == v, k
    for arr in dasp.ARRAYS:
        assert np.array_equal(dasp.dasp_plan_copy_array(plan, arr), ref.arrays[arr]), arr
    lens = np.diff(A.row_ptr)
    assert info["row_long"] == int((lens > max_len).sum())
    assert info["row_medium"] == int(((lens > 4) & (lens <= max_len)).sum())


def test_knob_closed_forms_on_stencil():
    # 16^3 stencil: MAX_LEN = 20 turns every len-27 row long; tau = 1.0 leaves no regular block
    from tests.test_oracle import stencil_hist
    A = synth.generate(synth.config("c2", scale=16 / 128))
    h = stencil_hist(16)
    info = host_plan(A, "f64", max_len=20).info
    assert info["row_long"] == h[27] and info["row_medium"] == h[18] + h[12] + h[8]
    assert info["nnz_long_new"] == h[27] * 64          # one group of 64 per len-27 row
    info = host_plan(A, "f64", threshold=1.0).info
    assert info["nnz_reg_new"] == 0 and info["nnz_irreg"] == A.nnz
    with pytest.raises(dasp.DaspError):
        host_plan(A, "f64", max_len=3)


@pytest.mark.parametrize("dt", ["f64", "f16", "f32"])
@pytest.mark.parametrize("panel", [-1, 1000])
def test_narrow_mid_split(dt, panel):
    """The launch schedule's narrow / mid row-block counts: per panel, the trailing
    row-blocks whose rows span at most 2K (narrow) / 4K (mid) slots, slots = K*nreg + irregular length
    of the row-block's first row -- recomputed here from the oracle builder's rb_ptr / irr_ptr."""
    rng = np.random.default_rng(3)
    lens = list(rng.choice([0, 1, 3, 5, 6, 7, 8, 9, 12, 16, 20, 27, 31, 40, 100, 300], size=4000))
    A = synth.from_lengths(lens, n=5000)
    plan = host_plan(A, dt, panel_rows=panel)
    info = plan.info
    ref = oracle.build(A, dt, panel_rows=info["panel_rows"])
    K = 8 if dt == "f16" else 4
    rb_ptr, irr_ptr, pan = ref.view("rb_ptr"), ref.view("irr_ptr"), ref.view("panels").reshape(-1, 12)
    narrow = mid = 0
    for p in pan:
        rb0, nrb = int(p[4]), int(p[5])
        slots = [(rb_ptr[rb + 1] - rb_ptr[rb]) // (8 * K) * K + (irr_ptr[8 * rb + 1] - irr_ptr[8 * rb])
                 for rb in range(rb0, rb0 + nrb)]
        n_narrow = n_mid = 0
        while n_narrow < nrb and slots[nrb - 1 - n_narrow] <= 2 * K:
            n_narrow += 1
        while n_narrow + n_mid < nrb and slots[nrb - 1 - n_narrow - n_mid] <= 4 * K:
            n_mid += 1
        narrow += n_narrow
        mid += n_mid
    assert (info["rowblocks_narrow"], info["rowblocks_mid"]) == (narrow, mid)
    assert info["narrow_rb_per_warp"] in (4, 8)


def test_binding_rejects_short_and_mistyped_host_buffers():
    """The ctypes binding checks what the C call trusts: col / val must hold row_ptr[m] entries, and
    host x / y buffers must have the plan's element types and enough elements."""
    A = synth.generate(synth.config("c1a"))
    with pytest.raises(ValueError):
        dasp.dasp_plan_create(A.row_ptr, A.col[:-5], A.val[:-5], A.m, A.n, "f64", device=-1)
    with pytest.raises(ValueError):
        dasp.dasp_plan_create(A.row_ptr, A.col, A.val[:-1], A.m, A.n, "f64", device=-1)
    p = dasp.dasp_plan_create(A.row_ptr, A.col, A.val, A.m, A.n, "f64", device=-1)
    x = np.zeros(A.n)
    y = np.zeros(A.m)
    for bad_x, bad_y in [(x[:-1], y), (x, y[:-1]), (x.astype(np.float32), y), (x, y.astype(np.float32)),
                         (np.zeros((2, A.n))[:, 0], y)]:
        with pytest.raises(ValueError):
            dasp.dasp_spmv_host(p, bad_x, bad_y)
    with pytest.raises(ValueError):
        dasp.dasp_spmv_host_stream(p, np.zeros(2 * A.n - 1), A.n, np.zeros(2 * A.m), A.m, 2)
    with pytest.raises(ValueError):
        dasp.dasp_spmv_host_stream(p, np.zeros(2 * A.n), A.n, np.zeros(2 * A.m - 1), A.m, 2)


def test_x_stage_table_selection():
    """x-window staging is chosen from the plan's own columns: the wide medium blocks of
    a 27-point stencil gather from three dense plane windows (staged); a power-law matrix's blocks
    gather from all of x (never staged); FP16 stencil rows (27 <= 4K = 32 slots) are mid row-blocks,
    not wide ones; x_stage = 1 turns it off; the MMA default variant never stages."""
    st = synth.generate(synth.config("c2", scale=0.25))
    for dt, sx in (("f64", 8), ("f32", 4)):
        val = st.val.astype(np.float64 if dt == "f64" else np.float32)
        info = dasp.dasp_plan_create(st.row_ptr, st.col, val, st.m, st.n, dt, device=-1, x_stage=2).info
        assert info["x_stage_blocks"] > 0
        # tile map (one byte per span tile, 128-B rounded) + staged tiles of 32 columns
        assert info["x_stage_smem"] >= 3 * 32 * sx and (info["x_stage_smem"] - 32 * sx * 96) <= 4096
        off = dasp.dasp_plan_create(st.row_ptr, st.col, val, st.m, st.n, dt, device=-1, x_stage=1).info
        assert off["x_stage_blocks"] == 0 and off["x_stage_smem"] == 0
    mma = dasp.dasp_plan_create(st.row_ptr, st.col, st.val, st.m, st.n, "f64", device=-1,
                                variant=dasp.DASP_VARIANT_MMA, x_stage=2).info
    assert mma["x_stage_blocks"] == 0
    h = dasp.dasp_plan_create(st.row_ptr, st.col, st.val.astype(np.float16), st.m, st.n, "f16", device=-1, x_stage=2).info
    assert h["x_stage_blocks"] == 0 and h["rowblocks_mid"] > 0
    pl = synth.generate(synth.config("c3", scale=0.02))
    assert dasp.dasp_plan_create(pl.row_ptr, pl.col, pl.val, pl.m, pl.n, "f64", device=-1, x_stage=2).info["x_stage_blocks"] == 0
