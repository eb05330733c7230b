"""CPU oracle for the DASP SpMV hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product path
(``paper_conf_sc_lu023_b200``) never imports it and shares no code with it.

* :func:`spmv`  — Alg. 1 with alpha/beta, accumulated in double-double
  (``oracle.c`` :: ``oracle_spmv``), returning ``y`` and the tolerance scale
  ``s_i = |alpha| sum_j |a_ij x_j| + |beta y0_i|``.
* :func:`build` — the DASP data structure of §3.2 built literally from the
  FORMAT spec in DESIGN.md §4 (``oracle.c`` :: ``oracle_build``).
* :func:`tolerance_ok` — the acceptance rule of BASELINE.json ``north_star``.

FP16 inputs: the fp16 values are widened to float64 exactly (every binary16 is a
binary64) and the oracle proceeds in long double (north_star: "against an FP64 oracle
fed the same fp16 values").
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")

ARRAYS = ["long_val", "long_col", "group_ptr", "long_out", "rb_ptr", "reg_val", "reg_col", "irr_ptr",
          "irr_val", "irr_col", "med_out", "short_val", "short_col", "short_out", "empty_rows", "panels"]
COUNTS = ["m", "n", "nnz", "n0", "n1", "n2", "n3", "n4", "row_medium", "row_long", "nrb", "n_groups",
          "n_groups_padded", "t13", "t4", "t22", "ts", "nnz_long_new", "nnz_reg_new", "nnz_irreg", "nnz_short_new",
          "panel_rows", "n_panels"]


def build_lib() -> str:
    src = os.path.join(_HERE, "oracle.c")
    if not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fopenmp", "-fPIC", "-shared",
                               "-o", _SO, src, "-lm"])
    return _SO


_lib = None


def _L():
    global _lib
    if _lib is None:
        build_lib()
        lib = ctypes.CDLL(_SO)
        vp, i64, d = ctypes.c_void_p, ctypes.c_int64, ctypes.c_double
        lib.oracle_spmv.argtypes = [i64, vp, vp, vp, vp, d, d, vp, vp, vp]
        lib.oracle_spmv_mt.argtypes = [i64, vp, vp, vp, vp, d, d, vp, vp, vp, ctypes.c_int]
        lib.oracle_spmv_mt.restype = ctypes.c_int
        lib.oracle_build.argtypes = [ctypes.c_int, i64, i64, vp, vp, vp, i64, i64, d]
        lib.oracle_build.restype = vp
        lib.oracle_free.argtypes = [vp]
        lib.oracle_fmt_count.argtypes = [vp, ctypes.c_char_p]
        lib.oracle_fmt_count.restype = i64
        lib.oracle_fmt_array.argtypes = [vp, ctypes.c_char_p, ctypes.POINTER(vp), ctypes.POINTER(i64)]
        _lib = lib
    return _lib


def _p(a):
    return a.ctypes.data if a is not None and a.size else None


def spmv(row_ptr, col, val, x, alpha=1.0, beta=0.0, y0=None):
    """y = alpha*A*x + beta*y0 by Alg. 1 with double-double accumulation; returns (y, s)."""
    row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
    col = np.ascontiguousarray(col, dtype=np.int32)
    val = np.ascontiguousarray(np.asarray(val).astype(np.float64))   # exact for fp16 inputs
    x = np.ascontiguousarray(np.asarray(x).astype(np.float64))
    m = len(row_ptr) - 1
    y = np.empty(max(m, 1))[:m]
    s = np.empty(max(m, 1))[:m]
    if beta != 0.0:
        y0 = np.ascontiguousarray(np.asarray(y0).astype(np.float64))
    else:
        y0 = None
    _L().oracle_spmv(m, _p(row_ptr), _p(col), _p(val), _p(x), float(alpha), float(beta), _p(y0), _p(y), _p(s))
    return y, s


def spmv_mt(row_ptr, col, val, x, alpha=1.0, beta=0.0, y0=None, threads=0):
    """The same as spmv with the rows split over host threads (OpenMP); returns (y, s, threads)."""
    row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
    col = np.ascontiguousarray(col, dtype=np.int32)
    val = np.ascontiguousarray(np.asarray(val).astype(np.float64))
    x = np.ascontiguousarray(np.asarray(x).astype(np.float64))
    m = len(row_ptr) - 1
    y = np.empty(max(m, 1))[:m]
    s = np.empty(max(m, 1))[:m]
    y0 = np.ascontiguousarray(np.asarray(y0).astype(np.float64)) if beta != 0.0 else None
    used = _L().oracle_spmv_mt(m, _p(row_ptr), _p(col), _p(val), _p(x), float(alpha), float(beta), _p(y0), _p(y),
                               _p(s), int(threads))
    return y, s, used


def spmv_csr(A, x, alpha=1.0, beta=0.0, y0=None):
    return spmv(A.row_ptr, A.col, A.val, x, alpha, beta, y0)


def tolerance_ok(y, y_ref, s, dtype="f64"):
    """north_star acceptance per row: |y - y_ref| <= tol * s, with tol 1e-12 (FP64) or 2e-3 (FP16).

    Rows with s == 0 must match exactly; NaN must match NaN; Inf must match sign."""
    y = np.asarray(y, dtype=np.float64)
    # FP32 (R29): f64 arithmetic then one rounding to f32 -> |err| <= 2^-24 |y| + tiny <= 1e-7 s
    tol = {"f64": 1e-12, "f32": 1e-7}.get(dtype, 2e-3)
    nan_ref, nan_y = np.isnan(y_ref), np.isnan(y)
    inf_ref = np.isinf(y_ref)
    fin = ~(nan_ref | inf_ref)
    ok = np.ones(len(y), dtype=bool)
    ok[nan_ref] = nan_y[nan_ref]
    ok[inf_ref] = y[inf_ref] == y_ref[inf_ref]
    with np.errstate(invalid="ignore"):
        ok[fin] = np.abs(y[fin] - y_ref[fin]) <= tol * s[fin]
    return ok


class Format:
    """The oracle builder's arrays (numpy copies) and counts."""

    def __init__(self, A, dtype="f64", panel_rows=0, max_len=256, tau=0.75):
        lib = _L()
        dt = {"f64": 0, "f16": 1, "f32": 2}[dtype]
        val = np.ascontiguousarray(A.val.astype({0: np.float64, 1: np.float16, 2: np.float32}[dt]))
        rp = np.ascontiguousarray(A.row_ptr, dtype=np.int64)
        col = np.ascontiguousarray(A.col, dtype=np.int32)
        h = lib.oracle_build(dt, A.m, A.n, _p(rp), _p(col), _p(val), int(panel_rows), int(max_len), float(tau))
        try:
            self.counts = {c: int(lib.oracle_fmt_count(h, c.encode())) for c in COUNTS}
            self.arrays = {}
            for a in ARRAYS:
                ptr, nb = ctypes.c_void_p(), ctypes.c_int64()
                assert lib.oracle_fmt_array(h, a.encode(), ctypes.byref(ptr), ctypes.byref(nb)) == 0
                buf = (ctypes.c_uint8 * nb.value).from_address(ptr.value) if nb.value else b""
                self.arrays[a] = np.frombuffer(bytes(buf), dtype=np.uint8)
        finally:
            lib.oracle_free(h)
        self.dtype = dtype

    def view(self, name):
        b = self.arrays[name]
        if name.endswith("_val"):
            return b.view({"f64": np.float64, "f16": np.float16, "f32": np.float32}[self.dtype])
        if name in ("group_ptr", "rb_ptr", "irr_ptr", "panels"):
            return b.view(np.int64)
        return b.view(np.int32)


def build(A, dtype="f64", panel_rows=0, max_len=256, tau=0.75) -> Format:
    """panel_rows <= 0: one panel (the paper's global format); else panels of that many rows.
    max_len: MAX_LEN; tau: the regular-block threshold."""
    return Format(A, dtype, panel_rows, max_len, tau)
