"""Pins of the CPU oracle against things other than itself.

CPU only.  Each test names the passage or mathematical fact it relies on.
"""
import numpy as np
import pytest
import scipy.sparse as sp

import oracle
import synth
from tests.format_decode import check_roundtrip


def csr_from_dense(D):
    S = sp.csr_matrix(D)
    S.sort_indices()
    return synth.CSR(D.shape[0], D.shape[1], S.indptr.astype(np.int64), S.indices.astype(np.int32),
                     S.data.astype(np.float64))


def rand_int_dense(rng, m, n, density):
    D = rng.integers(-3, 4, size=(m, n)).astype(np.float64)
    D[rng.random((m, n)) > density] = 0.0
    D[rng.random(m) < 0.2] = 0.0  # empty rows
    return D


# P1: brute-force dense product on tiny matrices, exact with integers (Alg. 1 is y = A x)
@pytest.mark.parametrize("seed", range(6))
def test_p1_dense_bruteforce_exact(seed):
    rng = np.random.default_rng(seed)
    m, n = rng.integers(1, 65, size=2)
    D = rand_int_dense(rng, m, n, rng.uniform(0.05, 0.9))
    x = rng.integers(-3, 4, size=n).astype(np.float64)
    A = csr_from_dense(D)
    y, s = oracle.spmv_csr(A, x)
    want = np.array([sum(D[i, j] * x[j] for j in range(n)) for i in range(m)])  # brute force
    assert np.array_equal(y, want)
    assert np.array_equal(s, np.abs(D * x[None, :]).sum(axis=1))


# P2: identity, diagonal and permutation matrices give exact results (one product per row)
def test_p2_identity_diagonal_permutation():
    rng = np.random.default_rng(11)
    n = 777
    x = rng.uniform(-1, 1, n)
    I = synth.CSR(n, n, np.arange(n + 1, dtype=np.int64), np.arange(n, dtype=np.int32), np.ones(n))
    assert np.array_equal(oracle.spmv_csr(I, x)[0], x)
    d = rng.uniform(-5, 5, n)
    Dg = synth.CSR(n, n, np.arange(n + 1, dtype=np.int64), np.arange(n, dtype=np.int32), d)
    assert np.array_equal(oracle.spmv_csr(Dg, x)[0], d * x)  # a single rounding, same as numpy's
    perm = rng.permutation(n).astype(np.int32)
    P = synth.CSR(n, n, np.arange(n + 1, dtype=np.int64), perm, np.ones(n))
    assert np.array_equal(oracle.spmv_csr(P, x)[0], x[perm])


# P3: A*1 = row sums, against numpy.add.reduceat (independent routine)
@pytest.mark.parametrize("name", ["c1a", "c1b"])
def test_p3_rowsums(name):
    A = synth.generate(synth.config(name, val_mode=synth.VAL_INT))
    y, _ = oracle.spmv_csr(A, np.ones(A.n))
    lens = np.diff(A.row_ptr)
    want = np.zeros(A.m)
    nz = lens > 0
    want[nz] = np.add.reduceat(A.val, A.row_ptr[:-1][nz])
    assert np.array_equal(y, want)
    # real values: within the FP64 tolerance
    A = synth.generate(synth.config(name))
    y, s = oracle.spmv_csr(A, np.ones(A.n))
    want[nz] = np.add.reduceat(A.val, A.row_ptr[:-1][nz])
    want[~nz] = 0
    assert oracle.tolerance_ok(y, want, s).all()


# P4: scipy.sparse CSR product (a textbook library routine), within 1e-13 * s
@pytest.mark.parametrize("name", ["c1a", "c1b", "c6"])
def test_p4_scipy(name):
    A = synth.generate(synth.config(name, scale=0.2 if name == "c6" else 1.0))
    x = synth.vector(5, A.n)
    y, s = oracle.spmv_csr(A, x)
    S = sp.csr_matrix((A.val, A.col, A.row_ptr), shape=(A.m, A.n))
    ref = S @ x
    assert (np.abs(y - ref) <= 1e-13 * s + 0.0).all()


# accurate accumulation: a row whose naive fp64 left-to-right sum is wrong (cancellation)
def test_long_double_accumulation():
    A = synth.CSR(1, 3, np.array([0, 3], dtype=np.int64), np.array([0, 1, 2], dtype=np.int32),
                  np.array([1e16, 1.0, -1e16]))
    y, s = oracle.spmv_csr(A, np.ones(3))
    assert (1e16 + 1.0) - 1e16 == 0.0      # fp64 loses the 1
    assert y[0] == 1.0                      # exact answer
    assert s[0] == 2e16 + 1.0


# P10: alpha/beta (BLAS semantics, R16): linearity and beta == 0 does not read y0
def test_p10_alpha_beta():
    A = synth.generate(synth.config("c1b", val_mode=synth.VAL_INT))
    x = synth.vector(3, A.n, synth.VAL_INT)
    y0 = synth.vector(4, A.m, synth.VAL_INT)
    y1, _ = oracle.spmv_csr(A, x)
    y, s = oracle.spmv_csr(A, x, alpha=-2.0, beta=3.0, y0=y0)
    assert np.array_equal(y, -2.0 * y1 + 3.0 * y0)
    nan_y0 = np.full(A.m, np.nan)
    y, _ = oracle.spmv_csr(A, x, alpha=1.0, beta=0.0, y0=nan_y0)
    assert np.isfinite(y).all()
    y, s = oracle.spmv_csr(A, x, alpha=0.0, beta=2.0, y0=y0)
    assert np.array_equal(y, 2.0 * y0)


def test_tolerance_rule():
    y_ref = np.array([1.0, 0.0, np.nan, np.inf, -np.inf])
    s = np.array([1.0, 0.0, 1.0, 1.0, 1.0])
    assert oracle.tolerance_ok(np.array([1.0 + 5e-13, 0.0, np.nan, np.inf, -np.inf]), y_ref, s).all()
    assert not oracle.tolerance_ok(np.array([1.0 + 5e-12, 0.0, np.nan, np.inf, -np.inf]), y_ref, s)[0]
    assert not oracle.tolerance_ok(np.array([1.0, 1e-300, 0, -np.inf, np.inf]), y_ref, s)[1:].any()


# ---------------------------------------------------------------------------------------------
# format-builder pins
# ---------------------------------------------------------------------------------------------

def stencil_hist(g):
    """closed form: per dimension, g-2 interior points see 3 neighbours and 2 boundary points 2."""
    i, b = g - 2, 2
    return {27: i ** 3, 18: 3 * i * i * b, 12: 3 * i * b * b, 8: b ** 3}


# P9: closed-form stencil counts (classifier + the strict reading R4 of "exceeds")
@pytest.mark.parametrize("g", [16, 128])
def test_p9_stencil_closed_forms(g):
    A = synth.generate(synth.config("c2", scale=g / 128))
    assert A.m == g ** 3 and A.nnz == (3 * g - 2) ** 3
    h = stencil_hist(g)
    lens = np.diff(A.row_ptr)
    assert {int(k): int(v) for k, v in zip(*np.unique(lens, return_counts=True))} == h
    if g == 128:
        assert A.nnz == 55_742_968 and h == {27: 2_000_376, 18: 95_256, 12: 1_512, 8: 8}
    F = oracle.build(A, "f64")
    c = F.counts
    assert c["row_medium"] == A.m and c["row_long"] == 0 and c["n0"] + c["n1"] + c["n2"] + c["n3"] + c["n4"] == 0
    assert c["nrb"] == A.m // 8
    # FP64, K=4: len 27 -> 6 regular blocks + 3 irregular (block 6 holds 24/32, not > 24);
    #            len 18 -> 4 + 2; len 12 -> 3 + 0; len 8 -> 2 + 0.  Zero pads.
    assert c["nnz_reg_new"] == 24 * h[27] + 16 * h[18] + 12 * h[12] + 8 * h[8]
    assert c["nnz_irreg"] == 3 * h[27] + 2 * h[18]
    if g == 128:
        assert (c["nnz_reg_new"], c["nnz_irreg"]) == (49_551_328, 6_191_640)
    if g == 16:
        # FP16, K=8 (m16n8k8, R14): len 27 -> 3 blocks + 3 irregular (block 3: 24/64 <= 48);
        # len 18 -> 2 + 2; len 12 -> block 1 holds 32/64 -> 1 + 4; len 8 -> 1 + 0
        F16 = oracle.build(A.to_fp16(), "f16")
        c16 = F16.counts
        assert c16["nnz_reg_new"] == 24 * h[27] + 16 * h[18] + 8 * h[12] + 8 * h[8]
        assert c16["nnz_irreg"] == 3 * h[27] + 2 * h[18] + 4 * h[12]


# P8: closed-form short piecing counts (R13)
@pytest.mark.parametrize("n1,n2,n3,n4", [(5, 7, 3, 2), (0, 0, 40, 0), (100, 1, 0, 33), (33, 64, 33, 0), (1, 1, 1, 1)])
def test_p8_short_piecing_counts(n1, n2, n3, n4):
    lens = [1] * n1 + [2] * n2 + [3] * n3 + [4] * n4 + [0] * 3
    rng = np.random.default_rng(n1 * 7 + n2)
    lens = list(rng.permutation(lens))
    A = synth.from_lengths(lens, n=64, val_mode=synth.VAL_INT)
    for dt in ["f64", "f16"]:
        F = oracle.build(A if dt == "f64" else A.to_fp16(), dt)
        c = F.counts
        p13 = min(n1, n3)
        n4cat = n4 + (n3 - p13) + n2 % 2
        assert (c["n0"], c["n1"], c["n2"], c["n3"], c["n4"]) == (3, n1, n2, n3, n4)
        assert c["t13"] == -(-p13 // 32) and c["t22"] == -(-(n2 // 2) // 32)
        assert c["t4"] == -(-n4cat // 32) and c["ts"] == -(-(n1 - p13) // 128)
        so = F.view("short_out")
        assert (so >= 0).sum() == n1 + n2 + n3 + n4
        check_roundtrip(A, c, F.view, dt)


# P6: builder round trip on every class and ragged tails, both dtypes
@pytest.mark.parametrize("name", ["c1a", "c1b", "c6s", "lens"])
@pytest.mark.parametrize("dt", ["f64", "f16"])
def test_p6_roundtrip(name, dt):
    if name == "lens":
        lens = [0, 1, 2, 3, 4, 5, 9, 17, 31, 33, 64, 255, 256, 257, 300, 1000, 2049, 4, 4, 3, 2, 1, 1, 1]
        A = synth.from_lengths(lens * 3, n=3000)
    elif name == "c6s":
        A = synth.generate(synth.config("c6", scale=0.01))
    else:
        A = synth.generate(synth.config(name))
    F = oracle.build(A if dt == "f64" else A.to_fp16(), dt)
    check_roundtrip(A, F.counts, F.view, dt)
    c = F.counts
    assert c["n0"] + c["n1"] + c["n2"] + c["n3"] + c["n4"] + c["row_medium"] + c["row_long"] == A.m
    G = 64 if dt == "f64" else 128
    assert c["nnz_long_new"] == sum(-(-L // G) * G for L in np.diff(A.row_ptr) if L > 256)


# R28 panels: the panelized format is the paper's format of each panel, concatenated
@pytest.mark.parametrize("dt", ["f64", "f16"])
@pytest.mark.parametrize("R", [1, 97, 1000, 4096])
def test_panels_roundtrip_and_concatenation(dt, R):
    A = synth.generate(synth.config("c1b"))
    Ad = A if dt == "f64" else A.to_fp16()
    F = oracle.build(Ad, dt, panel_rows=R)
    c = F.counts
    assert c["n_panels"] == -(-A.m // R) and c["panel_rows"] == R
    check_roundtrip(A, c, F.view, dt)
    pn = F.view("panels").reshape(-1, 12)
    # each panel's share equals the global format of that panel's rows alone
    for q in [0, len(pn) // 2, len(pn) - 1]:
        r0, rows = int(pn[q, 0]), int(pn[q, 1])
        sub = synth.CSR(rows, A.n, A.row_ptr[r0:r0 + rows + 1] - A.row_ptr[r0],
                        A.col[A.row_ptr[r0]:A.row_ptr[r0 + rows]], Ad.val[A.row_ptr[r0]:A.row_ptr[r0 + rows]])
        G = oracle.build(sub, dt)
        g = G.counts
        assert int(pn[q, 5]) == g["nrb"]
        assert tuple(int(v) for v in pn[q, 7:11]) == (g["t13"], g["t4"], g["t22"], g["ts"])
        t0, nt = int(pn[q, 6]), g["t13"] + g["t4"] + g["t22"] + g["ts"]
        sv = F.view("short_col")[t0 * 128:(t0 + nt) * 128]
        assert np.array_equal(sv, G.view("short_col"))
        so = F.view("short_out")[int(pn[q, 11]):int(pn[q, 11]) + len(G.view("short_out"))]
        assert np.array_equal(so, np.where(G.view("short_out") >= 0, G.view("short_out") + r0, -1))


def test_medium_sort_is_stable_descending():
    lens = [7, 9, 7, 12, 9, 7, 5, 12, 30, 7]
    A = synth.from_lengths(lens, n=64)
    F = oracle.build(A, "f64")
    mo = F.view("med_out")
    real = [int(r) for r in mo if r >= 0]
    assert real == [8, 3, 7, 1, 4, 0, 2, 5, 9, 6]   # by len desc, ties by original index
    assert list(mo[10:]) == [-1] * 6


def test_empty_and_degenerate():
    A = synth.CSR(5, 3, np.zeros(6, dtype=np.int64), np.zeros(0, np.int32), np.zeros(0))
    y, s = oracle.spmv_csr(A, np.ones(3))
    assert np.array_equal(y, np.zeros(5)) and np.array_equal(s, np.zeros(5))
    F = oracle.build(A, "f64")
    assert F.counts["n0"] == 5 and F.counts["nrb"] == 0 and F.counts["n_groups"] == 0
    A0 = synth.CSR(0, 0, np.zeros(1, dtype=np.int64), np.zeros(0, np.int32), np.zeros(0))
    F0 = oracle.build(A0, "f64")
    assert all(v == 0 for k, v in F0.counts.items() if k not in ("panel_rows", "n_panels"))


def test_oracle_multithreaded_copy_is_bitwise_identical():
    """oracle_spmv_mt runs the same per-row loop with rows split over threads (bench.py's all-core
    oracle timing): every row is computed by one thread in the same order, so y and s are
    bit-identical to the single-thread oracle, with and without alpha/beta."""
    for name, scale in (("c1b", 1.0), ("c3", 0.002)):
        A = synth.generate(synth.config(name, scale=scale))
        x = synth.vector(3, A.n)
        y0 = synth.vector(4, A.m)
        for alpha, beta in ((1.0, 0.0), (-0.5, 2.0)):
            y1, s1 = oracle.spmv(A.row_ptr, A.col, A.val, x, alpha, beta, y0)
            y2, s2, used = oracle.spmv_mt(A.row_ptr, A.col, A.val, x, alpha, beta, y0, threads=4)
            assert used == 4
            assert np.array_equal(y1, y2) and np.array_equal(s1, s2)
