"""Row-slab multi-GPU mode (BASELINE.json north_star (4)).

Each rank owns a contiguous, nnz-balanced slab of rows (``dasp_partition_rows``), builds
the DASP plan of its slab only (per-row generation, so no rank holds the full CSR), with
columns remapped (``dasp_remap_columns``) into a padded x layout of P chunks of S =
max_p rows_p entries.  One iteration of iterated SpMV is

    dasp_spmv(slab, x_cur)  -> written straight into x_next[p*S : p*S + rows_p]
    all_gather_into_tensor(x_next, x_next[p*S : (p+1)*S])      (NCCL over NVLink / NVSwitch)

so the collective is the only data exchange and runs in place on the padded buffer.
Rows are independent, so the slab SpMV needs nothing from other ranks but x.
torch.distributed is the plumbing (process group, NCCL all-gather); the SpMV is libdasp.

The local SpMV is pluggable (``local_spmv``) so the partition / remap / all-gather logic
is testable on CPU with the gloo backend (tests/test_multigpu.py).

``fused=True`` replaces the all-gather by the SpMV epilogue itself: both x buffers live in
torch symmetric memory (every rank maps every peer's buffers over NVLink), and
``dasp_spmv_scatter`` stores each y value of this rank's slab into ALL ranks' next x buffer
(P posted NVLink stores per row, overlapped with the rest of the SpMV), followed by one
device-side barrier across ranks.  No NCCL call is left on the data path.
"""
from __future__ import annotations

import numpy as np

from . import dasp


def slab_bounds(row_lengths: np.ndarray, nparts: int) -> np.ndarray:
    """nnz-balanced contiguous row slabs from the global row lengths (via the C-ABI)."""
    rp = np.zeros(len(row_lengths) + 1, dtype=np.int64)
    np.cumsum(row_lengths, out=rp[1:])
    return dasp.dasp_partition_rows(rp, nparts)


class Slab:
    """One rank's slab: host CSR (columns remapped to the padded layout) and its row range."""

    def __init__(self, row_ptr, col, val, row0, rows, starts, S, inf_norm):
        self.row_ptr, self.col, self.val = row_ptr, col, val
        self.row0, self.rows = row0, rows
        self.starts, self.S = starts, S
        self.inf_norm = inf_norm          # max_i sum_j |a_ij| over the whole matrix (for scaling)

    @property
    def nnz(self):
        return int(self.row_ptr[-1])


def build_slab(generate_rows, row_lengths: np.ndarray, rank: int, world: int, reduce_max=None,
               need_norm: bool = True) -> Slab:
    """generate_rows(row0, nrows) -> CSR of those rows (global columns).  reduce_max(v) -> max over ranks.
    need_norm=False skips the infinity norm (only the iteration needs it)."""
    starts = slab_bounds(row_lengths, world)
    r0, r1 = int(starts[rank]), int(starts[rank + 1])
    A = generate_rows(r0, r1 - r0)
    if world == 1:                      # one slab: no remap (also valid for rectangular matrices)
        col, S = np.ascontiguousarray(A.col, dtype=np.int32), A.n
    else:
        col = np.ascontiguousarray(A.col, dtype=np.int32).copy()
        S = dasp.dasp_remap_columns(col, starts)
    inf_norm = 1.0
    if need_norm:
        absval = np.abs(A.val.astype(np.float64))
        lens = np.diff(A.row_ptr)
        rs = np.zeros(len(lens))
        nz = lens > 0
        if nz.any():
            rs[nz] = np.add.reduceat(absval, A.row_ptr[:-1][nz])
        local = float(rs.max()) if len(rs) else 0.0
        inf_norm = reduce_max(local) if reduce_max else local
    return Slab(A.row_ptr, col, A.val, r0, r1 - r0, starts, S, inf_norm)


def scatter_destinations(peer_base, rank, world, buf_index, n_pad, S, elem_bytes):
    """Device addresses that receive this rank's y slab: its own next-x slab first (the one
    dasp_spmv_scatter treats as y), then the same slab in every peer's next x.  peer_base[q] is
    rank q's symmetric buffer [x0 | x1] as mapped into this process."""
    off = (buf_index * n_pad + rank * S) * elem_bytes
    return [peer_base[rank] + off] + [peer_base[q] + off for q in range(world) if q != rank]


class SlabSpMV:
    """Iterated SpMV over P ranks: x_{k+1} = alpha * A x_k, x all-gathered every step.

    x buffers are torch tensors of length P*S (padded layout).  ``local_spmv(x, y_view,
    alpha)`` computes the slab rows; the default calls libdasp on this rank's GPU."""

    def __init__(self, slab: Slab, world: int, rank: int, device, dtype="f64", group=None, local_spmv=None,
                 variant=dasp.DASP_VARIANT_DEFAULT, fused=False):
        import torch
        self.slab, self.world, self.rank, self.group = slab, world, rank, group
        self.device = torch.device(device)
        self.dtype = dtype
        self.fused = fused
        tdt = torch.float64
        n_pad = world * slab.S
        self.n_pad = n_pad
        if fused:
            import torch.distributed as dist
            import torch.distributed._symmetric_memory as symm_mem
            buf = symm_mem.empty(2 * n_pad, dtype=tdt, device=self.device)
            buf.zero_()
            self.hdl = symm_mem.rendezvous(buf, group if group is not None else dist.group.WORLD)
            self.peer_base = [int(b) for b in self.hdl.buffer_ptrs]
            self.x = [buf[:n_pad], buf[n_pad:]]
        else:
            self.x = [torch.zeros(n_pad, dtype=tdt, device=self.device) for _ in range(2)]
        self.cur = 0
        if local_spmv is None:
            if self.device.type != "cuda":
                raise RuntimeError("the libdasp slab SpMV needs a CUDA device (no CPU fallback)")
            self.plan = dasp.dasp_plan_create(slab.row_ptr, slab.col, slab.val, slab.rows, n_pad, dtype,
                                              device=self.device.index or 0)

            def _local(x, y, alpha):
                dasp.dasp_spmv(self.plan, x, y, alpha, 0.0, torch.cuda.current_stream(self.device),
                               variant=variant, check=False)
            self.local_spmv = _local
        else:
            self.plan = None
            self.local_spmv = local_spmv

    def set_x(self, x_global: np.ndarray):
        """Load the global x (length n) into the padded layout of the current buffer."""
        import torch
        st, S = self.slab.starts, self.slab.S
        buf = np.zeros(self.world * S)
        for q in range(self.world):
            buf[q * S: q * S + st[q + 1] - st[q]] = x_global[st[q]:st[q + 1]]
        self.x[self.cur].copy_(torch.from_numpy(buf))

    def my_view(self, buf):
        p, S = self.rank, self.slab.S
        return buf[p * S: p * S + self.slab.rows]

    def spmv(self, alpha=1.0):
        """Slab SpMV only: x_next[slab] = alpha * A_slab x_cur."""
        nxt = self.x[1 - self.cur]
        self.local_spmv(self.x[self.cur], self.my_view(nxt), alpha)
        return nxt

    def exchange(self):
        """In-place all-gather of the padded next buffer, then swap (the one collective)."""
        import torch.distributed as dist
        nxt = self.x[1 - self.cur]
        if self.world > 1:
            p, S = self.rank, self.slab.S
            dist.all_gather_into_tensor(nxt, nxt[p * S:(p + 1) * S], group=self.group)
        self.cur = 1 - self.cur

    def step(self, alpha=1.0):
        if self.fused:
            return self.fused_step(alpha)
        self.spmv(alpha)
        self.exchange()

    def fused_step(self, alpha=1.0):
        """One iteration with the all-gather fused into the SpMV epilogue (see module doc)."""
        import torch
        nb = 1 - self.cur
        dsts = scatter_destinations(self.peer_base, self.rank, self.world, nb, self.n_pad, self.slab.S, 8)
        dasp.dasp_spmv_scatter(self.plan, self.x[self.cur], dsts, alpha, 0.0, torch.cuda.current_stream(self.device))
        self.hdl.barrier(channel=0)          # every rank's stores have landed before x is read
        self.cur = nb

    def x_global(self) -> np.ndarray:
        st, S = self.slab.starts, self.slab.S
        b = self.x[self.cur].cpu().numpy()
        return np.concatenate([b[q * S: q * S + st[q + 1] - st[q]] for q in range(self.world)])
