"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests and bench.py.

Input generation only: nothing here classifies, packs or multiplies (DESIGN.md §3,
"Input recipe").  The C kernel ``synth.c`` is a counter-based generator keyed by
(seed, row, k) so any row range is reproducible on its own.

Configs (BASELINE.json ``configs``):

* ``c1a``  random CSR 4096x4096, len ~ Poisson(16)                       (configs[0])
* ``c1b``  class-coverage mix: empty/1/2/3/4/U[5,56] + 5 long rows        (configs[0] variant)
* ``c2``   27-point stencil 128^3, 55,742,968 nnz                         (configs[1])
* ``c3``   power-law lengths on [1,1e5], 12.5M rows, ~2e8 nnz             (configs[2])
* ``c5``   mixed-class, mean length ~64, row 1-norm <= 1                  (configs[4])
* ``c6``   short-only rows, len U{1..4}                                   (mc2depi-like)
* ``c7``   long-only rows, len log-uniform [257, 2e4], 40K rows, ~1.8e8 nnz (per-class probe)
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libsynth.so")

SYN_UNIFORM, SYN_MIX, SYN_STENCIL27, SYN_POWERLAW, SYN_MIXED64, SYN_SHORT, SYN_LENLIST = range(7)
VAL_UNIFORM, VAL_INT, VAL_ONES, VAL_SPD = range(4)


class _Params(ctypes.Structure):
    _fields_ = [
        ("m", ctypes.c_int64), ("n", ctypes.c_int64), ("seed", ctypes.c_uint64),
        ("val_mode", ctypes.c_int32), ("nx", ctypes.c_int32), ("ny", ctypes.c_int32), ("nz", ctypes.c_int32),
        ("mean", ctypes.c_double), ("gamma", ctypes.c_double), ("kmax", ctypes.c_int64),
        ("n_forced", ctypes.c_int64), ("local_frac", ctypes.c_double), ("local_w", ctypes.c_int64),
        ("zipf_s", ctypes.c_double), ("lenlist", ctypes.c_void_p),
    ]


def build() -> str:
    """Compile libsynth.so (gcc, OpenMP)."""
    src = os.path.join(_HERE, "synth.c")
    if not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-o", _SO, src, "-lm"])
    return _SO


_lib = None


def _L():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_SO)
        P = ctypes.POINTER(_Params)
        lib.synth_row_lengths.argtypes = [ctypes.c_int, P, ctypes.c_int64, ctypes.c_int64, ctypes.c_void_p]
        lib.synth_fill.argtypes = [ctypes.c_int, P, ctypes.c_int64, ctypes.c_int64, ctypes.c_void_p,
                                   ctypes.c_void_p, ctypes.c_void_p]
        lib.synth_vector.argtypes = [ctypes.c_uint64, ctypes.c_int32, ctypes.c_int64, ctypes.c_int64, ctypes.c_void_p]
        lib.synth_powerlaw_mean.argtypes = [ctypes.c_double, ctypes.c_int64]
        lib.synth_powerlaw_mean.restype = ctypes.c_double
        _lib = lib
    return _lib


@dataclass
class Spec:
    """A synthetic matrix recipe (kind + parameters)."""
    kind: int
    m: int
    n: int
    seed: int = 1
    val_mode: int = VAL_UNIFORM
    nx: int = 0
    ny: int = 0
    nz: int = 0
    mean: float = 16.0
    gamma: float = 1.86
    kmax: int = 100_000
    n_forced: int = 0
    local_frac: float = 0.5
    local_w: int = 4096
    zipf_s: float = 1.1
    lenlist: np.ndarray | None = field(default=None, repr=False)
    name: str = ""

    def _params(self):
        p = _Params(self.m, self.n, self.seed, self.val_mode, self.nx, self.ny, self.nz, self.mean, self.gamma,
                    self.kmax, self.n_forced, self.local_frac, self.local_w, self.zipf_s, None)
        if self.lenlist is not None:
            self._ll = np.ascontiguousarray(self.lenlist, dtype=np.int64)
            p.lenlist = self._ll.ctypes.data
        return p


@dataclass
class CSR:
    m: int
    n: int
    row_ptr: np.ndarray  # int64 [m+1]
    col: np.ndarray      # int32 [nnz]
    val: np.ndarray      # float64 [nnz] (or float16 after .to_fp16())
    name: str = ""

    @property
    def nnz(self) -> int:
        return int(self.row_ptr[-1])

    def to_fp16(self) -> "CSR":
        """Round values to IEEE binary16 (RNE); the oracle is fed these same bits."""
        return CSR(self.m, self.n, self.row_ptr, self.col, self.val.astype(np.float16), self.name + "_fp16")


def row_lengths(spec: Spec, row0: int = 0, nrows: int | None = None) -> np.ndarray:
    nrows = spec.m - row0 if nrows is None else nrows
    out = np.empty(nrows, dtype=np.int64)
    p = spec._params()
    _L().synth_row_lengths(spec.kind, ctypes.byref(p), row0, nrows, out.ctypes.data)
    return out


def generate(spec: Spec, row0: int = 0, nrows: int | None = None) -> CSR:
    """CSR of rows [row0, row0+nrows) of the recipe (global column space)."""
    nrows = spec.m - row0 if nrows is None else nrows
    lens = row_lengths(spec, row0, nrows)
    row_ptr = np.zeros(nrows + 1, dtype=np.int64)
    np.cumsum(lens, out=row_ptr[1:])
    nnz = int(row_ptr[-1])
    col = np.empty(max(nnz, 1), dtype=np.int32)[:nnz]
    val = np.empty(max(nnz, 1), dtype=np.float64)[:nnz]
    p = spec._params()
    rc = _L().synth_fill(spec.kind, ctypes.byref(p), row0, nrows, row_ptr.ctypes.data,
                         col.ctypes.data if nnz else None, val.ctypes.data if nnz else None)
    if rc:
        raise MemoryError("synth_fill failed")
    return CSR(nrows, spec.n, row_ptr, col, val, spec.name)


def vector(seed: int, n: int, mode: int = VAL_UNIFORM, i0: int = 0) -> np.ndarray:
    out = np.empty(max(n, 1), dtype=np.float64)[:n]
    if n:
        _L().synth_vector(seed, mode, i0, n, out.ctypes.data)
    return out


def powerlaw_mean(gamma: float, kmax: int) -> float:
    return float(_L().synth_powerlaw_mean(gamma, kmax))


# ---- the named configs -------------------------------------------------------------------------

def config(name: str, seed: int | None = None, val_mode: int = VAL_UNIFORM, scale: float = 1.0) -> Spec:
    """Named recipes.  ``scale`` shrinks m (and n) for test-sized variants."""
    s = lambda k: int(max(1, round(k * scale)))
    if name == "c1a":
        return Spec(SYN_UNIFORM, 4096, 4096, 1 if seed is None else seed, val_mode, mean=16.0, name=name)
    if name == "c1b":
        return Spec(SYN_MIX, s(4096), s(4096), 1 if seed is None else seed, val_mode, name=name)
    if name == "c2":
        g = s(128) if scale != 1.0 else 128
        return Spec(SYN_STENCIL27, g ** 3, g ** 3, 2 if seed is None else seed, val_mode, nx=g, ny=g, nz=g, name=name)
    if name == "c2big":  # C2+: 162^3 -> 113,379,904 nnz
        return Spec(SYN_STENCIL27, 162 ** 3, 162 ** 3, 2 if seed is None else seed, val_mode, nx=162, ny=162, nz=162,
                    name=name)
    if name == "c3":
        m = s(12_500_000)
        kmax = 100_000 if scale == 1.0 else max(300, min(100_000, m // 4))
        return Spec(SYN_POWERLAW, m, m, 3 if seed is None else seed, val_mode, gamma=1.86, kmax=kmax, n_forced=8,
                    local_frac=0.5, local_w=4096, zipf_s=1.1, name=name)
    if name == "c5":
        m = s(62_500_000)
        return Spec(SYN_MIXED64, m, m, 5 if seed is None else seed, val_mode, local_frac=0.5, local_w=4096,
                    zipf_s=1.1, name=name)
    if name == "c7":  # long rows only: lengths log-uniform on [257, 2e4], columns as c3
        m = s(40_000)
        return Spec(SYN_LENLIST, m, 12_500_000, 7 if seed is None else seed, val_mode,
                    lenlist=_long_lengths(m, 7 if seed is None else seed), local_frac=0.5, local_w=4096,
                    zipf_s=1.1, name=name)
    if name == "c6":
        m = s(525_000)
        return Spec(SYN_SHORT, m, m, 6 if seed is None else seed, val_mode, name=name)
    raise KeyError(name)


def _long_lengths(m, seed):
    rng = np.random.default_rng(seed)
    return np.exp(rng.uniform(np.log(257), np.log(20000), m)).astype(np.int64)


def from_lengths(lens, n: int, seed: int = 7, val_mode: int = VAL_UNIFORM, name: str = "lenlist") -> CSR:
    lens = np.asarray(lens, dtype=np.int64)
    spec = Spec(SYN_LENLIST, len(lens), n, seed, val_mode, lenlist=lens, local_frac=0.0, name=name)
    return generate(spec)
