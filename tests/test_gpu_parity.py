"""GPU parity: libdasp.so kernels (through the C-ABI) vs the CPU oracle on the same seeded inputs.

Bar (BASELINE.json north_star): FP64 |y - y_ref| <= 1e-12 * sum|a_ij x_j| per row; FP16
<= 2e-3 * sum|a_ij x_j| against the FP64 oracle fed the same fp16 values; bit-exact on
small-integer inputs (P5), identity / diagonal / permutation matrices (P2), and for the
device copy of the packed format vs the oracle builder.
"""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_sc_lu023_b200 import dasp  # noqa: E402

VARIANTS = [dasp.DASP_VARIANT_MMA, dasp.DASP_VARIANT_CUDACORE]
DTYPES = ["f64", "f16", "f32"]
NP_VAL = {"f64": np.float64, "f16": np.float16, "f32": np.float32}
VNAME = {dasp.DASP_VARIANT_MMA: "mma", dasp.DASP_VARIANT_CUDACORE: "cudacore"}


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    torch.cuda.init()


def make(A, dt, **kw):
    val = A.val.astype(NP_VAL[dt])
    return dasp.dasp_plan_create(A.row_ptr, A.col, val, A.m, A.n, dt, device=0, **kw)


def run(plan, x_np, dt, alpha=1.0, beta=0.0, y0=None, variant=0):
    xd = torch.from_numpy(np.ascontiguousarray(x_np.astype(NP_VAL[dt]))).cuda()
    ydt = torch.float64 if dt == "f64" else torch.float32
    if y0 is None:
        y = torch.full((plan.m,), float("nan"), dtype=ydt, device="cuda")
    else:
        y = torch.from_numpy(np.ascontiguousarray(y0)).to(ydt).cuda()
    dasp.dasp_spmv(plan, xd, y, alpha, beta, variant=variant)
    torch.cuda.synchronize()
    return y.cpu().numpy().astype(np.float64)


def oracle_ref(A, x, dt, alpha=1.0, beta=0.0, y0=None):
    if dt != "f64":   # the oracle is fed the same stored values (exactly widened to f64)
        val = A.val.astype(NP_VAL[dt]).astype(np.float64)
        x = x.astype(NP_VAL[dt]).astype(np.float64)
        if y0 is not None:
            y0 = y0.astype(np.float32).astype(np.float64)
    else:
        val = A.val
    return oracle.spmv(A.row_ptr, A.col, val, x, alpha, beta, y0)


def cases():
    yield "c1a", lambda vm: synth.generate(synth.config("c1a", val_mode=vm))
    yield "c1b", lambda vm: synth.generate(synth.config("c1b", val_mode=vm))
    yield "c2s", lambda vm: synth.generate(synth.config("c2", scale=24 / 128, val_mode=vm))
    yield "c3s", lambda vm: synth.generate(synth.config("c3", scale=0.01, val_mode=vm))
    yield "c5s", lambda vm: synth.generate(synth.config("c5", scale=4e-4, val_mode=vm))
    yield "c6s", lambda vm: synth.generate(synth.config("c6", scale=0.05, val_mode=vm))
    lens = [0, 1, 2, 3, 4, 5, 9, 17, 31, 33, 64, 255, 256, 257, 300, 1000, 2049, 4, 4, 3, 2, 1, 1, 1, 7, 6]
    yield "lens", lambda vm: synth.from_lengths(lens * 7, n=5000, val_mode=vm)


CASES = list(cases())


@pytest.mark.parametrize("variant", VARIANTS, ids=[VNAME[v] for v in VARIANTS])
@pytest.mark.parametrize("dt", DTYPES)
@pytest.mark.parametrize("name,gen", CASES, ids=[c[0] for c in CASES])
def test_parity_random_values(name, gen, dt, variant):
    A = gen(synth.VAL_UNIFORM)
    x = synth.vector(11, A.n)
    plan = make(A, dt)
    y = run(plan, x, dt, variant=variant)
    y_ref, s = oracle_ref(A, x, dt)
    ok = oracle.tolerance_ok(y, y_ref, s, dt)
    bad = np.flatnonzero(~ok)
    assert ok.all(), f"{len(bad)} rows off, first {bad[:5]}: {y[bad[:5]]} vs {y_ref[bad[:5]]}"


# P5: small-integer values make every summation order exact -> bit-exact in both dtypes,
# which also pins the MMA fragment layout and the diagonal lanes (Fig. 4).
@pytest.mark.parametrize("variant", VARIANTS, ids=[VNAME[v] for v in VARIANTS])
@pytest.mark.parametrize("dt", DTYPES)
@pytest.mark.parametrize("name,gen", CASES, ids=[c[0] for c in CASES])
def test_parity_integer_bit_exact(name, gen, dt, variant):
    A = gen(synth.VAL_INT)
    x = synth.vector(12, A.n, synth.VAL_INT)
    plan = make(A, dt)
    y = run(plan, x, dt, variant=variant)
    y_ref, _ = oracle_ref(A, x, dt)
    assert np.array_equal(y, y_ref)


# R28 panels: every panel size gives the same exact integer results (and parity on reals)
@pytest.mark.parametrize("variant", VARIANTS, ids=[VNAME[v] for v in VARIANTS])
@pytest.mark.parametrize("dt", DTYPES)
@pytest.mark.parametrize("panel", [-1, 1, 97, 1000, 50000])
def test_parity_panels(panel, dt, variant):
    A = synth.generate(synth.config("c3", scale=0.01, val_mode=synth.VAL_INT))
    x = synth.vector(21, A.n, synth.VAL_INT)
    if panel == 1:
        A = synth.generate(synth.config("c1b", val_mode=synth.VAL_INT))
        x = synth.vector(21, A.n, synth.VAL_INT)
    plan = make(A, dt, panel_rows=panel)
    y = run(plan, x, dt, variant=variant)
    y_ref, _ = oracle_ref(A, x, dt)
    assert np.array_equal(y, y_ref)
    y0 = synth.vector(22, A.m, synth.VAL_INT)
    y = run(plan, x, dt, 2.0, -3.0, y0, variant=variant)
    y_ref, _ = oracle_ref(A, x, dt, 2.0, -3.0, y0)
    assert np.array_equal(y, y_ref)


@pytest.mark.parametrize("dt", DTYPES)
def test_identity_diagonal_permutation_exact(dt):
    n = 5003
    rng = np.random.default_rng(3)
    x = rng.uniform(-1, 1, n)
    ar = np.arange(n + 1, dtype=np.int64)
    for val, col in [(np.ones(n), np.arange(n)), (rng.uniform(-4, 4, n), np.arange(n)),
                     (np.ones(n), rng.permutation(n))]:
        A = synth.CSR(n, n, ar, col.astype(np.int32), val)
        for v in VARIANTS:
            y = run(make(A, dt), x, dt, variant=v)
            y_ref, _ = oracle_ref(A, x, dt)
            if dt != "f64":   # one product is exact in the wide type, then rounded to y's fp32
                y_ref = y_ref.astype(np.float32).astype(np.float64)
            assert np.array_equal(y, y_ref)


@pytest.mark.parametrize("dt", DTYPES)
def test_alpha_beta(dt):
    A = synth.generate(synth.config("c1b", val_mode=synth.VAL_INT))
    x = synth.vector(1, A.n, synth.VAL_INT)
    y0 = synth.vector(2, A.m, synth.VAL_INT)
    plan = make(A, dt)
    for alpha, beta in [(2.0, -1.0), (-0.5, 3.0), (1.0, 1.0), (0.0, 2.0), (0.0, 0.0), (3.0, 0.0)]:
        for v in VARIANTS:
            y = run(plan, x, dt, alpha, beta, y0, variant=v)
            y_ref, _ = oracle_ref(A, x, dt, alpha, beta, y0)
            assert np.array_equal(y, y_ref), (alpha, beta, v)
    # beta == 0: y is not read (NaN in y must not propagate)
    y = run(plan, x, dt, 1.0, 0.0, np.full(A.m, np.nan))
    assert np.isfinite(y).all()


# P11: pads carry a sentinel column, so an Inf in x only reaches rows that store that column
@pytest.mark.parametrize("dt", DTYPES)
def test_inf_in_x_only_reaches_referencing_rows(dt):
    A = synth.generate(synth.config("c1b"))
    x = synth.vector(4, A.n)
    plan = make(A, dt)
    base = run(plan, x, dt)
    x2 = x.copy()
    x2[0] = np.inf
    for v in VARIANTS:
        y = run(plan, x2, dt, variant=v)
        touches = np.zeros(A.m, bool)
        rows = np.repeat(np.arange(A.m), np.diff(A.row_ptr))
        touches[rows[A.col == 0]] = True
        assert np.array_equal(y[~touches], run(plan, x, dt, variant=v)[~touches])
        assert not np.isfinite(y[touches]).any() or touches.sum() == 0
    assert np.isfinite(base).all()


@pytest.mark.parametrize("dt", DTYPES)
@pytest.mark.parametrize("panel", [-1, 500])
def test_device_arrays_match_oracle_builder(dt, panel):
    A = synth.generate(synth.config("c1b"))
    plan = make(A, dt, panel_rows=panel)   # keep_host off: copy_array reads back the device buffers
    ref = oracle.build(A, dt, panel_rows=plan.info["panel_rows"])
    for arr in dasp.ARRAYS:
        assert np.array_equal(dasp.dasp_plan_copy_array(plan, arr), ref.arrays[arr]), arr


def test_deterministic_and_variants_agree():
    A = synth.generate(synth.config("c3", scale=0.01))
    x = synth.vector(5, A.n)
    plan = make(A, "f64")
    a = run(plan, x, "f64")
    b = run(plan, x, "f64")
    assert np.array_equal(a, b)
    c = run(plan, x, "f64", variant=dasp.DASP_VARIANT_CUDACORE)
    y_ref, s = oracle_ref(A, x, "f64")
    assert oracle.tolerance_ok(c, y_ref, s).all()


def test_empty_and_degenerate():
    for m, n in [(0, 0), (7, 3), (1, 1)]:
        A = synth.CSR(m, n, np.zeros(m + 1, dtype=np.int64), np.zeros(0, np.int32), np.zeros(0))
        for dt in ["f64", "f16"]:
            plan = make(A, dt)
            if m:
                y = run(plan, np.ones(n), dt, 1.0, 0.0, np.full(m, np.nan))
                assert np.array_equal(y, np.zeros(m))
                y = run(plan, np.ones(n), dt, 1.0, 2.0, np.arange(m, dtype=np.float64))
                assert np.array_equal(y, 2.0 * np.arange(m))


def test_spmv_host_end_to_end():
    A = synth.generate(synth.config("c1b"))
    x = synth.vector(6, A.n)
    plan = make(A, "f64")
    y = np.full(A.m, np.nan)
    dasp.dasp_spmv_host(plan, x, y)
    y_ref, s = oracle.spmv_csr(A, x)
    assert oracle.tolerance_ok(y, y_ref, s).all()
    y0 = synth.vector(7, A.m)
    y = y0.copy()
    dasp.dasp_spmv_host(plan, x, y, 2.0, -1.0)
    y_ref, s = oracle.spmv_csr(A, x, 2.0, -1.0, y0)
    assert oracle.tolerance_ok(y, y_ref, s).all()


NARROW_LENS = {
    "len5-8": list(range(5, 9)),          # FP64/FP32 narrow (one lane per row); FP16 narrow
    "len9-16": list(range(9, 17)),        # FP64/FP32 mid (two lanes per row), nreg up to 4 (full chunk)
    "len13-16": list(range(13, 17)),      # every row-block nreg = 4 in FP64/FP32
    "len17-32": list(range(17, 33)),      # FP16 mid, nreg up to 4; FP64/FP32 wide
    "len29-32": list(range(29, 33)),      # FP16 nreg = 4 (full chunk)
    "mixed": list(range(5, 40)) + [0, 1, 2, 3, 4, 300],
}


@pytest.mark.parametrize("dt", DTYPES)
@pytest.mark.parametrize("name", list(NARROW_LENS))
def test_narrow_medium_paths(dt, name):
    """Narrow / mid medium row-blocks (the CUDA-core variant gives a lane or two lanes to a row)
    vs the oracle, and vs the MMA variant, which runs the same row-blocks on the paper's
    warp-per-row-block path (Alg. 3): real values within tolerance, integers bit-exact."""
    rng = np.random.default_rng(len(name))
    lens = list(rng.choice(NARROW_LENS[name], size=3001))          # ragged: 375 row-blocks + 1 row
    A = synth.from_lengths(lens, n=5000, seed=11)
    x = synth.vector(3, A.n)
    y_ref, s = oracle_ref(A, x, dt)
    plan = make(A, dt)
    for variant in VARIANTS:
        y = run(plan, x, dt, variant=variant)
        assert oracle.tolerance_ok(y, y_ref, s, dt).all(), (VNAME[variant], int((~oracle.tolerance_ok(y, y_ref, s, dt)).sum()))
        y0 = synth.vector(4, A.m)
        y = run(plan, x, dt, 2.0, -0.5, y0, variant=variant)
        y_ref2, s2 = oracle_ref(A, x, dt, 2.0, -0.5, y0)
        assert oracle.tolerance_ok(y, y_ref2, s2, dt).all()
    Ai = synth.from_lengths(lens, n=5000, seed=11, val_mode=synth.VAL_INT)
    xi = synth.vector(5, Ai.n, synth.VAL_INT)
    plan = make(Ai, dt)
    yi_ref, _ = oracle_ref(Ai, xi, dt)
    for variant in VARIANTS:
        assert np.array_equal(run(plan, xi, dt, variant=variant), yi_ref), VNAME[variant]


@pytest.mark.parametrize("dt", DTYPES)
@pytest.mark.parametrize("beta", [0.0, -0.5])
def test_spmv_host_stream_pipelined(dt, beta):
    """dasp_spmv_host_stream: nvec vectors at padded strides through the two-slot H2D/SpMV/D2H
    pipeline; every y_j matches the oracle and equals the one-call-per-vector result bit for bit."""
    A = synth.generate(synth.config("c1b"))
    nvec, ldx, ldy = 5, A.n + 3, A.m + 5
    X = np.zeros((nvec, ldx), dtype=NP_VAL[dt])
    for j in range(nvec):
        X[j, :A.n] = synth.vector(20 + j, A.n).astype(NP_VAL[dt])
    ynp = np.float64 if dt == "f64" else np.float32
    Y0 = np.zeros((nvec, ldy), dtype=ynp)
    for j in range(nvec):
        Y0[j, :A.m] = synth.vector(40 + j, A.m).astype(ynp)
    Xh = torch.from_numpy(X).pin_memory()
    Yh = torch.from_numpy(Y0.copy()).pin_memory()
    plan = make(A, dt)
    dasp.dasp_spmv_host_stream(plan, Xh.data_ptr(), ldx, Yh.data_ptr(), ldy, nvec, 1.5, beta)
    Y = Yh.numpy()
    val64 = A.val.astype(NP_VAL[dt]).astype(np.float64)
    for j in range(nvec):
        y_ref, s = oracle.spmv(A.row_ptr, A.col, val64, X[j, :A.n].astype(np.float64), 1.5, beta,
                               Y0[j, :A.m].astype(np.float64))
        assert oracle.tolerance_ok(Y[j, :A.m].astype(np.float64), y_ref, s, dt).all(), j
        assert np.array_equal(Y[j, A.m:], Y0[j, A.m:])          # stride padding untouched
        y1 = Y0[j, :A.m].copy()
        dasp.dasp_spmv_host(plan, np.ascontiguousarray(X[j, :A.n]), y1, 1.5, beta)
        assert np.array_equal(y1, Y[j, :A.m]), j
    with pytest.raises(dasp.DaspError):
        dasp.dasp_spmv_host_stream(plan, Xh.data_ptr(), A.n - 1, Yh.data_ptr(), ldy, nvec, 1.0, 0.0)


@pytest.mark.parametrize("dt", DTYPES)
def test_spmv_host_large_pinned_vectors(dt):
    """Host vectors >= 1 MiB in page-locked memory at odd strides (misaligned rows for FP16/FP32).
    Every y_j equals the device-resident dasp_spmv result bit for bit and passes the oracle."""
    rng = np.random.default_rng(5)
    n = {"f64": 200_001, "f32": 300_001, "f16": 600_001}[dt]       # x >= 1 MiB; row 1 of X misaligned for f16/f32
    A = synth.from_lengths(list(rng.integers(5, 41, size=3001)), n=n, seed=13)
    nvec, ldx, ldy = 3, n + 1, A.m + 3
    X = np.zeros((nvec, ldx), dtype=NP_VAL[dt])
    for j in range(nvec):
        X[j, :n] = synth.vector(60 + j, n).astype(NP_VAL[dt])
    Xh = torch.from_numpy(X).pin_memory()
    Yh = torch.full((nvec, ldy), float("nan"), dtype=torch.float64 if dt == "f64" else torch.float32).pin_memory()
    plan = make(A, dt)
    dasp.dasp_spmv_host_stream(plan, Xh.data_ptr(), ldx, Yh.data_ptr(), ldy, nvec, 1.0, 0.0)
    for j in range(nvec):
        y_dev = run(plan, X[j, :n], dt)
        assert np.array_equal(Yh.numpy()[j, :A.m].astype(np.float64), y_dev), j
        y_ref, s_ref = oracle_ref(A, X[j, :n].astype(np.float64), dt)
        assert oracle.tolerance_ok(Yh.numpy()[j, :A.m].astype(np.float64), y_ref, s_ref, dt).all(), j
    y1 = torch.full((A.m,), float("nan"), dtype=Yh.dtype).pin_memory()
    dasp.dasp_spmv_host(plan, Xh[0, :n].numpy(), y1.numpy())
    assert np.array_equal(y1.numpy(), Yh.numpy()[0, :A.m])


def test_bad_device_args():
    A = synth.generate(synth.config("c1a"))
    plan = make(A, "f64")
    x = torch.zeros(A.n, dtype=torch.float64, device="cuda")
    with pytest.raises(ValueError):
        dasp.dasp_spmv(plan, x, torch.zeros(A.m, dtype=torch.float32, device="cuda"))
    with pytest.raises(dasp.DaspError):
        dasp.dasp_spmv(plan, x, x, check=False)   # aliasing x == y


# dasp_spmv_scatter: the fused SpMV + all-gather epilogue writes the same values to every
# destination (here several local buffers stand in for the peers' x buffers)
@pytest.mark.parametrize("variant", VARIANTS, ids=[VNAME[v] for v in VARIANTS])
@pytest.mark.parametrize("dt", DTYPES)
def test_scatter_epilogue_writes_every_destination(dt, variant):
    A = synth.generate(synth.config("c1b", val_mode=synth.VAL_INT))
    x = synth.vector(51, A.n, synth.VAL_INT)
    y0 = synth.vector(52, A.m, synth.VAL_INT)
    plan = make(A, dt, variant=variant)
    xd = torch.from_numpy(x.astype(NP_VAL[dt])).cuda()
    ydt = torch.float64 if dt == "f64" else torch.float32
    for alpha, beta in [(1.0, 0.0), (2.0, -1.0), (1.0, 1.0), (0.0, 3.0)]:
        dst = [torch.from_numpy(y0).to(ydt).cuda()] + [torch.full((A.m,), float("nan"), dtype=ydt, device="cuda")
                                                        for _ in range(3)]
        dasp.dasp_spmv_scatter(plan, xd, dst, alpha, beta)
        torch.cuda.synchronize()
        y_ref, _ = oracle_ref(A, x, dt, alpha, beta, y0)
        for d in dst:
            assert np.array_equal(d.cpu().numpy().astype(np.float64), y_ref), (alpha, beta)
    with pytest.raises(dasp.DaspError):
        dasp.dasp_spmv_scatter(plan, xd, [dst[0]] * 9)


# f3 knobs: MAX_LEN and tau move rows between classes and slots between regular / irregular;
# the result must not change (bit-exact on integers)
@pytest.mark.parametrize("dt", DTYPES)
@pytest.mark.parametrize("max_len,tau", [(16, 0.75), (64, 0.5), (1000, 0.9), (256, 1.0), (4, 0.3)])
def test_parity_knobs(dt, max_len, tau):
    A = synth.generate(synth.config("c3", scale=0.004, val_mode=synth.VAL_INT))
    x = synth.vector(71, A.n, synth.VAL_INT)
    y_ref, _ = oracle_ref(A, x, dt)
    for v in VARIANTS:
        plan = make(A, dt, max_len=max_len, threshold=tau)
        assert np.array_equal(run(plan, x, dt, variant=v), y_ref)


@pytest.mark.parametrize("dt", ["f64", "f16", "f32"])
def test_cuda_graph_capture_replay(dt):
    """dasp_spmv enqueues only kernels on the given stream (no host sync, no allocation), so a loop
    of calls can be captured into a CUDA graph; the replayed result is bit-identical to the eager one
    (c1b: long, medium, short rows, empty rows — long phase 2 fused into the main kernel)."""
    A = synth.generate(synth.config("c1b"))
    x = synth.vector(8, A.n)
    plan = make(A, dt)
    eager = run(plan, x, dt)
    xd = torch.from_numpy(x.astype({"f64": np.float64, "f16": np.float16, "f32": np.float32}[dt])).cuda()
    yd = torch.full((A.m,), float("nan"), dtype=torch.float64 if dt == "f64" else torch.float32, device="cuda")
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    g = torch.cuda.CUDAGraph()
    with torch.cuda.stream(s):
        with torch.cuda.graph(g, stream=s):
            for _ in range(3):
                dasp.dasp_spmv(plan, xd, yd, 1.0, 0.0, s, check=False)
    yd.fill_(float("nan"))
    g.replay()
    torch.cuda.synchronize()
    assert np.array_equal(yd.cpu().numpy().astype(np.float64), eager.astype(np.float64))


# P:L91 (CSR): a column index per nonzero, no order implied, so the boundary accepts unsorted
# columns and duplicate (row, col) entries (summed like any other entry; include/dasp.h), and
# rectangular shapes.  Integer values: every summation order gives the same bits.
def _shuffle_rows(A, rng):
    """The same matrix with each row's entries in a random order."""
    rows = np.repeat(np.arange(A.m), np.diff(A.row_ptr))
    perm = np.lexsort((rng.random(A.nnz), rows))
    return synth.CSR(A.m, A.n, A.row_ptr, A.col[perm], A.val[perm])


def _with_duplicates(A, rng, frac=0.3):
    """Every chosen entry repeated 1-3 extra times right after itself (same column, own value):
    rows grow, so rows move between the short / medium / long classes."""
    rep = np.ones(A.nnz, dtype=np.int64)
    pick = rng.random(A.nnz) < frac
    rep[pick] += rng.integers(1, 4, int(pick.sum()))
    rows = np.repeat(np.arange(A.m), np.diff(A.row_ptr))
    lens = np.bincount(rows, weights=rep, minlength=A.m).astype(np.int64)
    rp = np.zeros(A.m + 1, dtype=np.int64)
    np.cumsum(lens, out=rp[1:])
    col = np.repeat(A.col, rep)
    val = np.repeat(A.val, rep)
    val = np.where(rng.random(len(val)) < 0.5, val, -val + 1.0)   # duplicates carry other values
    return synth.CSR(A.m, A.n, rp, col.astype(np.int32), val)


def _rectangular(m, n, rng, lens_choice):
    lens = rng.choice(lens_choice, size=m)
    lens = np.minimum(lens, n)
    rp = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(lens, out=rp[1:])
    col = np.concatenate([rng.choice(n, L, replace=False) for L in lens]).astype(np.int32) if rp[-1] else np.zeros(0, np.int32)
    val = rng.integers(-3, 4, int(rp[-1])).astype(np.float64)
    return synth.CSR(m, n, rp, col, val)


def _irregular_cases():
    rng = np.random.default_rng(77)
    base = synth.generate(synth.config("c1b", val_mode=synth.VAL_INT))
    yield "c1b_unsorted", _shuffle_rows(base, rng)
    yield "c1b_duplicates", _with_duplicates(base, rng)
    yield "c3s_unsorted_dup", _shuffle_rows(_with_duplicates(
        synth.generate(synth.config("c3", scale=0.004, val_mode=synth.VAL_INT)), rng), rng)
    lens = [0, 1, 2, 3, 4, 5, 9, 17, 33, 256, 257, 700]
    yield "tall_6000x700", _rectangular(6000, 700, rng, lens)
    yield "wide_900x20000", _rectangular(900, 20000, rng, lens + [3000])
    yield "one_column", _rectangular(3000, 1, rng, [0, 1])
    yield "dup_single_column", _with_duplicates(_rectangular(2000, 1, rng, [1]), rng, frac=1.0)


IRREGULAR = list(_irregular_cases())


@pytest.mark.parametrize("variant", VARIANTS, ids=[VNAME[v] for v in VARIANTS])
@pytest.mark.parametrize("dt", DTYPES)
@pytest.mark.parametrize("name,A", IRREGULAR, ids=[c[0] for c in IRREGULAR])
def test_unsorted_duplicate_rectangular_bit_exact(name, A, dt, variant):
    x = synth.vector(81, A.n, synth.VAL_INT)
    y0 = synth.vector(82, A.m, synth.VAL_INT)
    for panel in (0, 333):
        plan = make(A, dt, panel_rows=panel)
        y_ref, _ = oracle_ref(A, x, dt)
        assert np.array_equal(run(plan, x, dt, variant=variant), y_ref), name
        y_ref, _ = oracle_ref(A, x, dt, -2.0, 1.0, y0)
        assert np.array_equal(run(plan, x, dt, -2.0, 1.0, y0, variant=variant), y_ref), name
    # the device builder takes the same input and gives the same bytes
    if A.nnz:
        dplan = dasp.dasp_plan_create_device(torch.from_numpy(A.row_ptr).cuda(), torch.from_numpy(A.col).cuda(),
                                             torch.from_numpy(A.val.astype(NP_VAL[dt])).cuda(), A.m, A.n, dt)
        hplan = make(A, dt)
        for arr in dasp.ARRAYS:
            assert np.array_equal(dasp.dasp_plan_copy_array(dplan, arr), dasp.dasp_plan_copy_array(hplan, arr)), arr


# FP16 plans without a wide-medium majority run the 5-block main-kernel instantiation with 2 short
# tiles per warp; every variant must honour the plan's layout (the MMA kernel is compiled for 4)
@pytest.mark.parametrize("name,expect5", [("c2s", True), ("c6s", True), ("c5s", False), ("c1a", True)])
def test_fp16_occupancy5_layout(name, expect5):
    gen = dict(CASES)[name]
    A = gen(synth.VAL_INT)
    x = synth.vector(97, A.n, synth.VAL_INT)
    plan = make(A, "f16")
    assert plan.info["main_blocks_per_sm"] == (5 if expect5 else 4)
    assert plan.info["short_tiles_per_warp"] == (2 if expect5 else 4)
    y_ref, _ = oracle_ref(A, x, "f16")
    for v in VARIANTS:
        assert np.array_equal(run(plan, x, "f16", variant=v), y_ref), (name, VNAME[v])
    mplan = make(A, "f16", variant=dasp.DASP_VARIANT_MMA)           # MMA default: never the 5-block layout
    assert mplan.info["main_blocks_per_sm"] == 4
    for v in VARIANTS:
        assert np.array_equal(run(mplan, x, "f16", variant=v), y_ref), (name, VNAME[v])


# x-window staging (north_star (3) "shared-memory or TMA staging where reuse exists"):
# a staged block gathers the same x values from shared memory, so its y is bitwise the unstaged y
def _band_windows(m, n, windows, width, seed):
    """rows of `windows` clusters of `width` consecutive columns, cluster k at offset k * (n - m) /
    (windows - 1) from the row index (a stencil-like window structure with more windows than runs)"""
    rng = np.random.default_rng(seed)
    step = (n - m - width) // max(1, windows - 1)
    rows = []
    for i in range(m):
        cols = np.concatenate([i + k * step + np.arange(width) for k in range(windows)])
        rows.append(np.unique(np.clip(cols, 0, n - 1)))
    rp = np.zeros(m + 1, dtype=np.int64)
    rp[1:] = np.cumsum([len(r) for r in rows])
    col = np.concatenate(rows).astype(np.int32)
    val = rng.integers(-3, 4, len(col)).astype(np.float64)
    return synth.CSR(m, n, rp, col, val, name="band")


def _stage_cases():
    yield "c2_32", synth.generate(synth.config("c2", scale=0.25, val_mode=synth.VAL_INT))
    yield "c2_64", synth.generate(synth.config("c2", scale=0.5, val_mode=synth.VAL_INT))
    yield "band6", _band_windows(40000, 40000 + 6 * 700 + 33, 6, 5, 3)        # 6 windows -> merged runs
    yield "band3_odd", _band_windows(30001, 30001 + 2 * 900 + 41, 3, 7, 4)    # n not a multiple of 32


STAGE_CASES = list(_stage_cases())


@pytest.mark.parametrize("dt", ["f64", "f32"])
@pytest.mark.parametrize("name,A", STAGE_CASES, ids=[c[0] for c in STAGE_CASES])
def test_x_stage_bitwise_equal_to_unstaged(name, A, dt):
    staged, plain = make(A, dt, x_stage=2), make(A, dt, x_stage=1)
    assert staged.info["x_stage_blocks"] > 0 and staged.info["x_stage_smem"] > 0, name
    assert plain.info["x_stage_blocks"] == 0
    for seed, mode in ((11, synth.VAL_INT), (12, synth.VAL_UNIFORM)):
        x = synth.vector(seed, A.n, mode)
        y0 = synth.vector(seed + 1, A.m, mode)
        for alpha, beta in ((1.0, 0.0), (-0.5, 2.0)):
            ys = run(staged, x, dt, alpha, beta, y0 if beta else None, variant=dasp.DASP_VARIANT_CUDACORE)
            yp = run(plain, x, dt, alpha, beta, y0 if beta else None, variant=dasp.DASP_VARIANT_CUDACORE)
            assert np.array_equal(ys, yp), (name, dt, seed, alpha)
            y_ref, s = oracle_ref(A, x, dt, alpha, beta, y0 if beta else None)
            if mode == synth.VAL_INT:
                assert np.array_equal(ys, y_ref), (name, dt)
            else:
                assert oracle.tolerance_ok(ys, y_ref, s, dt).all(), (name, dt)
        # the MMA variant of a staged plan runs the unstaged kernel: same values
        ym = run(staged, x, dt, variant=dasp.DASP_VARIANT_MMA)
        y_ref, s = oracle_ref(A, x, dt)
        assert oracle.tolerance_ok(ym, y_ref, s, dt).all()


@pytest.mark.parametrize("dt", ["f64", "f32"])
def test_x_stage_misaligned_x_falls_back(dt):
    """x that is not 16-byte aligned (a view at an odd element offset) cannot be the cp.async.bulk
    source: the call runs the unstaged kernel and gives the same y"""
    A = STAGE_CASES[0][1]
    plan = make(A, dt, x_stage=2)
    assert plan.info["x_stage_blocks"] > 0
    x = synth.vector(21, A.n, synth.VAL_INT).astype(NP_VAL[dt])
    buf = torch.zeros(A.n + 1, dtype=torch.float64 if dt == "f64" else torch.float32, device="cuda")
    buf[1:] = torch.from_numpy(x).cuda()
    xv = buf[1:]
    assert xv.data_ptr() % 16 != 0
    ydt = torch.float64 if dt == "f64" else torch.float32
    y1 = torch.empty(A.m, dtype=ydt, device="cuda")
    y2 = torch.empty(A.m, dtype=ydt, device="cuda")
    dasp.dasp_spmv(plan, xv, y1, 1.0, 0.0)
    dasp.dasp_spmv(plan, torch.from_numpy(x).cuda(), y2, 1.0, 0.0)
    torch.cuda.synchronize()
    assert torch.equal(y1, y2)
    y_ref, _ = oracle_ref(A, x.astype(np.float64), dt)
    assert np.array_equal(y1.cpu().numpy().astype(np.float64), y_ref)


# long-row phase 2 of rows with more than 1024 groups runs on the whole warp (kernels.cu
# long_row_sum_warp): huge and ordinary long rows share finish warps; exact on integers, within the
# FP64 / FP16 bars on real values, deterministic
@pytest.mark.parametrize("dt", DTYPES)
def test_huge_long_rows_phase2(dt):
    lens = [300, 2_000_000, 257, 70_000, 10, 3, 8193, 1, 9000, 513, 1025 * 64 + 1, 1024 * 64]
    for vm in (synth.VAL_INT, synth.VAL_UNIFORM):
        A = synth.from_lengths(lens, n=3_000_000, val_mode=vm)
        x = synth.vector(61, A.n, vm)
        plan = make(A, dt)
        y_ref, s = oracle_ref(A, x, dt)
        for v in VARIANTS:
            y = run(plan, x, dt, variant=v)
            if vm == synth.VAL_INT:
                assert np.array_equal(y, y_ref), (dt, VNAME[v])
            else:
                assert oracle.tolerance_ok(y, y_ref, s, dt).all(), (dt, VNAME[v])
                assert np.array_equal(y, run(plan, x, dt, variant=v)), "phase 2 not deterministic"
