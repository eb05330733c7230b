"""Thin ctypes binding of libdasp.so (include/dasp.h) — argument marshalling only.

Every step of the hot path runs in the library's sm_100a kernels; this module only turns
numpy arrays (host CSR) and torch CUDA tensors (device x / y, streams) into the plain
pointers of the C-ABI.  The function names are the C names.  There is no CPU fallback:
if libdasp.so is missing or fails to load, importing this module raises.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("DASP_LIB", os.path.join(_HERE, "libdasp.so"))   # override: experiment builds

DASP_R_64F, DASP_R_16F, DASP_R_32F = 0, 1, 2
DASP_VARIANT_DEFAULT, DASP_VARIANT_MMA, DASP_VARIANT_CUDACORE = 0, 1, 2
DASP_K_MAIN, DASP_K_LONG, DASP_K_SCALE, DASP_K_COUNT = 0, 1, 2, 3
KERNEL_NAMES = ["dasp_main_kernel", "dasp_long_kernel", "dasp_scale_kernel"]

ARRAYS = ["long_val", "long_col", "group_ptr", "long_out", "rb_ptr", "reg_val", "reg_col", "irr_ptr",
          "irr_val", "irr_col", "med_out", "short_val", "short_col", "short_out", "empty_rows", "panels"]
STATUS = ["DASP_OK", "DASP_ERR_INVALID_ARG", "DASP_ERR_INVALID_CSR", "DASP_ERR_OUT_OF_MEMORY",
          "DASP_ERR_CUDA", "DASP_ERR_UNSUPPORTED", "DASP_ERR_INTERNAL"]

# every symbol include/dasp.h declares (tests check the library exports all of them)
EXPORTS = ["dasp_options_default", "dasp_plan_create", "dasp_plan_create_device", "dasp_spmv", "dasp_spmv_ex", "dasp_spmv_scatter", "dasp_spmv_host",
           "dasp_spmv_host_stream",
           "dasp_plan_destroy", "dasp_status_string", "dasp_plan_get_info", "dasp_plan_copy_array",
           "dasp_partition_rows", "dasp_remap_columns", "dasp_gather_halo", "dasp_plan_set_timing", "dasp_plan_read_timing",
           "dasp_version"]


class DaspError(RuntimeError):
    def __init__(self, status: int, what: str):
        name = STATUS[status] if 0 <= status < len(STATUS) else f"status {status}"
        super().__init__(f"{what}: {name}")
        self.status = status


class Options(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int32), ("variant", ctypes.c_int32), ("validate", ctypes.c_int32),
                ("keep_host", ctypes.c_int32), ("medium_rb_per_warp", ctypes.c_int32),
                ("num_threads", ctypes.c_int32), ("panel_rows", ctypes.c_int64),
                ("max_len", ctypes.c_int32), ("threshold", ctypes.c_double), ("x_stage", ctypes.c_int32)]


class PlanInfo(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int64) for n in ("m", "n", "nnz")] + \
               [("dtype", ctypes.c_int32), ("device", ctypes.c_int32)] + \
               [(n, ctypes.c_int64) for n in (
                   "n_empty", "n_len1", "n_len2", "n_len3", "n_len4", "row_medium", "row_long", "rowblocks",
                   "n_groups", "n_groups_padded", "tiles_13", "tiles_4", "tiles_22", "tiles_single",
                   "nnz_long_new", "nnz_reg_new", "nnz_irreg", "nnz_short_new", "nnz_long", "nnz_medium",
                   "nnz_short", "device_bytes", "alg_bytes_beta0", "alg_bytes_beta1")] + \
               [("medium_rb_per_warp", ctypes.c_int32), ("launches_per_spmv", ctypes.c_int32),
                ("panel_rows", ctypes.c_int64), ("n_panels", ctypes.c_int64),
                ("max_len", ctypes.c_int64), ("threshold", ctypes.c_double),
                ("build_ms", ctypes.c_double), ("upload_ms", ctypes.c_double),
                ("rowblocks_mid", ctypes.c_int64), ("rowblocks_narrow", ctypes.c_int64), ("narrow_rb_per_warp", ctypes.c_int32),
                ("main_blocks_per_sm", ctypes.c_int32), ("short_tiles_per_warp", ctypes.c_int32),
                ("x_stage_blocks", ctypes.c_int64), ("x_stage_smem", ctypes.c_int32)]

    def as_dict(self):
        return {name: getattr(self, name) for name, _ in self._fields_}


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: run `make` (or __graft_entry__.build()) first; "
                          "there is no CPU fallback")
    lib = ctypes.CDLL(LIB_PATH)
    vp, i64, i32, d = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32, ctypes.c_double
    sig = {
        "dasp_options_default": ([ctypes.POINTER(Options)], None),
        "dasp_plan_create": ([ctypes.POINTER(vp), i64, i64, i64, vp, vp, vp, ctypes.c_int, ctypes.POINTER(Options)],
                             ctypes.c_int),
        "dasp_plan_create_device": ([ctypes.POINTER(vp), i64, i64, i64, vp, vp, vp, ctypes.c_int,
                                     ctypes.POINTER(Options), vp], ctypes.c_int),
        "dasp_spmv": ([vp, vp, vp, d, d, vp], ctypes.c_int),
        "dasp_spmv_ex": ([vp, vp, vp, d, d, vp, i32], ctypes.c_int),
        "dasp_spmv_host": ([vp, vp, vp, d, d, vp], ctypes.c_int),
        "dasp_spmv_host_stream": ([vp, vp, i64, vp, i64, i64, d, d, vp], ctypes.c_int),
        "dasp_spmv_scatter": ([vp, vp, ctypes.POINTER(vp), i32, d, d, vp], ctypes.c_int),
        "dasp_plan_destroy": ([vp], ctypes.c_int),
        "dasp_status_string": ([ctypes.c_int], ctypes.c_char_p),
        "dasp_plan_get_info": ([vp, ctypes.POINTER(PlanInfo)], ctypes.c_int),
        "dasp_plan_copy_array": ([vp, i32, vp, ctypes.POINTER(i64)], ctypes.c_int),
        "dasp_partition_rows": ([vp, i64, i32, vp], ctypes.c_int),
        "dasp_remap_columns": ([vp, i64, vp, i32, ctypes.POINTER(i64)], ctypes.c_int),
        "dasp_gather_halo": ([vp, vp, i64, vp, i32, vp], ctypes.c_int),
        "dasp_plan_set_timing": ([vp, i32], ctypes.c_int),
        "dasp_plan_read_timing": ([vp, vp, vp], ctypes.c_int),
        "dasp_version": ([], ctypes.c_char_p),
    }
    for name, (args, res) in sig.items():
        f = getattr(lib, name)
        f.argtypes = args
        f.restype = res
    return lib


_lib = _load()


def lib():
    return _lib


def _check(st: int, what: str):
    if st != 0:
        raise DaspError(st, what)


def _ptr(a) -> int | None:
    """Device/host pointer of a torch tensor, numpy array or raw int."""
    if a is None:
        return None
    if isinstance(a, int):
        return a
    if isinstance(a, np.ndarray):
        return a.ctypes.data if a.size else None
    return a.data_ptr() if a.numel() else None


def _stream_ptr(stream) -> int | None:
    if stream is None:
        return None
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


def dasp_version() -> str:
    return _lib.dasp_version().decode()


class Plan:
    """Owns a dasp_plan_t.  Create with :func:`dasp_plan_create`."""

    def __init__(self, handle, dtype, m, n):
        self.handle = handle
        self.dtype = dtype
        self.m, self.n = m, n

    def __del__(self):
        if getattr(self, "handle", None) and _lib is not None:   # _lib is None at interpreter exit
            _lib.dasp_plan_destroy(self.handle)
            self.handle = None

    def destroy(self):
        if self.handle:
            _check(_lib.dasp_plan_destroy(self.handle), "dasp_plan_destroy")
            self.handle = None

    @property
    def info(self) -> dict:
        return dasp_plan_get_info(self)


def dasp_plan_create(row_ptr, col_idx, val, m: int, n: int, dtype: str = "f64", device: int = 0,
                     variant: int = DASP_VARIANT_CUDACORE, validate: bool = True, keep_host: bool = False,
                     medium_rb_per_warp: int = 0, num_threads: int = 0, panel_rows: int = 0,
                     max_len: int = 256, threshold: float = 0.75, x_stage: int = 0) -> Plan:
    """Build the DASP format of a host CSR matrix and upload it (device=-1: host-only plan).

    row_ptr int64[m+1], col_idx int32[nnz], val float64[nnz] (dtype "f64") or float16[nnz]
    (dtype "f16"; passed as binary16 bits) or float32[nnz] (dtype "f32").  panel_rows: 0 automatic,
    -1 one global panel.  x_stage: shared-memory x-window staging, 0 automatic, 1 off, 2 on."""
    row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
    col_idx = np.ascontiguousarray(col_idx, dtype=np.int32)
    if dtype == "f64":
        val = np.ascontiguousarray(val, dtype=np.float64)
        dt = DASP_R_64F
    elif dtype == "f16":
        val = np.ascontiguousarray(val, dtype=np.float16)
        dt = DASP_R_16F
    elif dtype == "f32":
        val = np.ascontiguousarray(val, dtype=np.float32)
        dt = DASP_R_32F
    else:
        raise ValueError(dtype)
    if len(row_ptr) != m + 1:
        raise ValueError("row_ptr must have m+1 entries")
    nnz = int(row_ptr[-1]) if m >= 0 else 0
    # the C call trusts nnz: both arrays must hold it (a short array would be read past its end)
    if len(col_idx) != len(val) or len(col_idx) < nnz:
        raise ValueError(f"col_idx ({len(col_idx)}) and val ({len(val)}) must both hold row_ptr[m] = {nnz} entries")
    opts = Options()
    _lib.dasp_options_default(ctypes.byref(opts))
    opts.device, opts.variant, opts.validate = device, variant, int(validate)
    opts.keep_host, opts.medium_rb_per_warp, opts.num_threads = int(keep_host), medium_rb_per_warp, num_threads
    opts.panel_rows = panel_rows
    opts.max_len, opts.threshold = int(max_len), float(threshold)
    opts.x_stage = int(x_stage)
    h = ctypes.c_void_p()
    st = _lib.dasp_plan_create(ctypes.byref(h), m, n, nnz, _ptr(row_ptr), _ptr(col_idx), _ptr(val), dt,
                               ctypes.byref(opts))
    _check(st, "dasp_plan_create")
    return Plan(h, dtype, m, n)


def dasp_plan_create_device(row_ptr, col_idx, val, m: int, n: int, dtype: str = "f64", device: int = 0,
                            variant: int = DASP_VARIANT_CUDACORE, validate: bool = True, medium_rb_per_warp: int = 0,
                            panel_rows: int = 0, max_len: int = 256, threshold: float = 0.75,
                            stream=None) -> Plan:
    """Build the plan on the GPU from a device CSR (torch CUDA tensors: int64 row_ptr, int32
    col_idx, float64 / float16 val) -- SURVEY.md §8(f) f2."""
    import torch
    want = {"f64": torch.float64, "f16": torch.float16, "f32": torch.float32}[dtype]
    for t, dt_ in ((row_ptr, torch.int64), (col_idx, torch.int32), (val, want)):
        if not isinstance(t, torch.Tensor) or not t.is_cuda or t.dtype != dt_ or not t.is_contiguous():
            raise ValueError("dasp_plan_create_device needs contiguous CUDA tensors (int64, int32, value dtype)")
    if row_ptr.numel() != m + 1:
        raise ValueError("row_ptr must have m+1 entries")
    if val.numel() != col_idx.numel():
        raise ValueError("col_idx and val must have the same length")
    opts = Options()
    _lib.dasp_options_default(ctypes.byref(opts))
    opts.device, opts.variant, opts.validate = device, variant, int(validate)
    opts.medium_rb_per_warp, opts.panel_rows = medium_rb_per_warp, panel_rows
    opts.max_len, opts.threshold = int(max_len), float(threshold)
    h = ctypes.c_void_p()
    st = _lib.dasp_plan_create_device(ctypes.byref(h), m, n, int(col_idx.numel()), _ptr(row_ptr), _ptr(col_idx),
                                      _ptr(val), {"f64": DASP_R_64F, "f16": DASP_R_16F, "f32": DASP_R_32F}[dtype],
                                      ctypes.byref(opts),
                                      _stream_ptr(stream))
    _check(st, "dasp_plan_create_device")
    return Plan(h, dtype, m, n)


def _xy_dtypes(dtype):
    """(x, y) torch dtypes of a plan dtype."""
    import torch
    return {"f64": (torch.float64, torch.float64), "f16": (torch.float16, torch.float32),
            "f32": (torch.float32, torch.float32)}[dtype]


def _xy_np(dtype):
    """(x, y) numpy dtypes of a plan dtype."""
    return {"f64": (np.float64, np.float64), "f16": (np.float16, np.float32), "f32": (np.float32, np.float32)}[dtype]


def _check_host(a, need, want, name):
    """A host buffer passed by pointer to the C call: a numpy array or a CPU torch tensor of the
    plan's element type, contiguous, with at least `need` elements (the library reads / writes
    exactly that many).  Raw integer pointers are the caller's responsibility."""
    if isinstance(a, int):
        return
    if isinstance(a, np.ndarray):
        ok = a.dtype == np.dtype(want) and a.flags.c_contiguous and a.size >= need
        got = f"{a.dtype}[{a.size}]"
    else:
        import torch
        tw = {np.float64: torch.float64, np.float32: torch.float32, np.float16: torch.float16}[want]
        ok = (isinstance(a, torch.Tensor) and not a.is_cuda and a.dtype == tw and a.is_contiguous()
              and a.numel() >= need)
        got = f"{getattr(a, 'dtype', type(a))}[{a.numel() if isinstance(a, torch.Tensor) else '?'}]"
    if not ok:
        raise ValueError(f"{name}: need a contiguous host {np.dtype(want).name} buffer of >= {need} elements, got {got}")


def _default_stream(plan, stream):
    """stream=None means torch's current stream on the plan's device (not the legacy NULL stream,
    which torch's pool streams do not synchronise with)."""
    if stream is not None:
        return stream
    if not hasattr(plan, "_dev"):
        plan._dev = plan.info["device"]
    if plan._dev < 0:                     # host-only plan: the library reports UNSUPPORTED
        return None
    import torch
    return torch.cuda.current_stream(plan._dev)


def _check_vec(t, length, want_dtype, name, plan_device):
    import torch
    if not isinstance(t, torch.Tensor):
        raise TypeError(f"{name} must be a torch CUDA tensor")
    if not t.is_cuda or t.device.index != plan_device:
        raise ValueError(f"{name} must live on cuda:{plan_device}")
    if t.dtype != want_dtype or not t.is_contiguous() or t.numel() < length:
        raise ValueError(f"{name}: need contiguous {want_dtype} with >= {length} elements")


def dasp_spmv(plan: Plan, x, y, alpha: float = 1.0, beta: float = 0.0, stream=None,
              variant: int = DASP_VARIANT_DEFAULT, check: bool = True):
    """y = alpha*A*x + beta*y on the plan's device (x, y torch CUDA tensors; enqueue only on
    `stream`, default torch's current stream)."""
    if check:
        dev = plan.info["device"] if not hasattr(plan, "_dev") else plan._dev
        plan._dev = dev
        xd, yd = _xy_dtypes(plan.dtype)
        _check_vec(x, plan.n, xd, "x", dev)
        _check_vec(y, plan.m, yd, "y", dev)
    stream = _default_stream(plan, stream)
    st = _lib.dasp_spmv_ex(plan.handle, _ptr(x), _ptr(y), float(alpha), float(beta), _stream_ptr(stream), variant)
    _check(st, "dasp_spmv")


def dasp_spmv_scatter(plan: Plan, x, dsts, alpha: float = 1.0, beta: float = 0.0, stream=None):
    """y = alpha*A*x + beta*y written to every pointer of `dsts` (dsts[0] is this GPU's y; the rest
    are raw device pointers or tensors, e.g. peer x buffers mapped over NVLink)."""
    stream = _default_stream(plan, stream)
    ptrs = (ctypes.c_void_p * len(dsts))(*[_ptr(d) for d in dsts])
    st = _lib.dasp_spmv_scatter(plan.handle, _ptr(x), ptrs, len(dsts), float(alpha), float(beta), _stream_ptr(stream))
    _check(st, "dasp_spmv_scatter")


def dasp_spmv_host(plan: Plan, x: np.ndarray, y: np.ndarray, alpha: float = 1.0, beta: float = 0.0, stream=None):
    """End-to-end call with host buffers (copies inside; synchronises)."""
    xt, yt = _xy_np(plan.dtype)
    if alpha != 0.0 and plan.n > 0:
        _check_host(x, plan.n, xt, "x")
    _check_host(y, plan.m, yt, "y")
    stream = _default_stream(plan, stream)
    st = _lib.dasp_spmv_host(plan.handle, _ptr(x), _ptr(y), float(alpha), float(beta), _stream_ptr(stream))
    _check(st, "dasp_spmv_host")


def dasp_spmv_host_stream(plan: Plan, x, ldx: int, y, ldy: int, nvec: int, alpha: float = 1.0, beta: float = 0.0,
                          stream=None):
    """nvec end-to-end SpMVs with host buffers (vectors at strides ldx / ldy elements), H2D / SpMV / D2H
    pipelined over two device slots; synchronises."""
    if nvec < 0 or ldx < 0 or ldy < 0:
        raise ValueError("nvec, ldx and ldy must be >= 0")
    xt, yt = _xy_np(plan.dtype)
    if nvec > 0:
        if alpha != 0.0 and plan.n > 0:
            _check_host(x, (nvec - 1) * ldx + plan.n, xt, "x")
        _check_host(y, (nvec - 1) * ldy + plan.m, yt, "y")
    stream = _default_stream(plan, stream)
    st = _lib.dasp_spmv_host_stream(plan.handle, _ptr(x), int(ldx), _ptr(y), int(ldy), int(nvec), float(alpha),
                                    float(beta), _stream_ptr(stream))
    _check(st, "dasp_spmv_host_stream")


def dasp_plan_destroy(plan: Plan):
    plan.destroy()


def dasp_plan_get_info(plan: Plan) -> dict:
    info = PlanInfo()
    _check(_lib.dasp_plan_get_info(plan.handle, ctypes.byref(info)), "dasp_plan_get_info")
    return info.as_dict()


def dasp_plan_copy_array(plan: Plan, name: str) -> np.ndarray:
    """Packed array `name` (see ARRAYS) as raw bytes (uint8)."""
    idx = ARRAYS.index(name)
    nb = ctypes.c_int64(0)
    _check(_lib.dasp_plan_copy_array(plan.handle, idx, None, ctypes.byref(nb)), "dasp_plan_copy_array")
    out = np.empty(max(nb.value, 1), dtype=np.uint8)[:nb.value]
    if nb.value:
        _check(_lib.dasp_plan_copy_array(plan.handle, idx, out.ctypes.data, ctypes.byref(nb)), "dasp_plan_copy_array")
    return out


def dasp_partition_rows(row_ptr: np.ndarray, nparts: int) -> np.ndarray:
    row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
    starts = np.zeros(nparts + 1, dtype=np.int64)
    _check(_lib.dasp_partition_rows(row_ptr.ctypes.data, len(row_ptr) - 1, nparts, starts.ctypes.data),
           "dasp_partition_rows")
    return starts


def dasp_remap_columns(col: np.ndarray, starts: np.ndarray) -> int:
    """In-place remap of int32 columns into the padded all-gather layout; returns the stride S."""
    assert col.dtype == np.int32 and col.flags.c_contiguous
    starts = np.ascontiguousarray(starts, dtype=np.int64)
    S = ctypes.c_int64(0)
    _check(_lib.dasp_remap_columns(_ptr(col), len(col), starts.ctypes.data, len(starts) - 1, ctypes.byref(S)),
           "dasp_remap_columns")
    return int(S.value)


def dasp_gather_halo(src, idx, dst, stream=None):
    """dst[k] = src[idx[k]] on the device (the halo pack of the sparse x exchange).  src / dst are
    CUDA tensors of the same element size (2, 4 or 8 bytes), idx an int32 CUDA tensor."""
    n = idx.numel()
    if dst.numel() < n or src.element_size() != dst.element_size():
        raise ValueError("dasp_gather_halo: dst too small or element sizes differ")
    _check(_lib.dasp_gather_halo(_ptr(src), _ptr(idx), n, _ptr(dst), src.element_size(), _stream_ptr(stream)),
           "dasp_gather_halo")


def dasp_plan_set_timing(plan: Plan, capacity: int):
    _check(_lib.dasp_plan_set_timing(plan.handle, capacity), "dasp_plan_set_timing")


def dasp_plan_read_timing(plan: Plan):
    """Returns {kernel_name: (total_ms, launches)} of the timed dasp_spmv calls."""
    ms = np.zeros(DASP_K_COUNT, dtype=np.float64)
    n = np.zeros(DASP_K_COUNT, dtype=np.int64)
    _check(_lib.dasp_plan_read_timing(plan.handle, ms.ctypes.data, n.ctypes.data), "dasp_plan_read_timing")
    return {KERNEL_NAMES[k]: (float(ms[k]), int(n[k])) for k in range(DASP_K_COUNT)}
