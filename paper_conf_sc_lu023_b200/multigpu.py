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

``HaloSlabSpMV`` shrinks and hides the exchange instead: each slab is split
by column owner into a LOCAL sub-matrix (columns inside the slab, indexed 0..rows_p-1, so it
reads this rank's x slab directly) and a REMOTE sub-matrix whose columns are renumbered
0..R-1 over the sorted set of remote columns it references (its halo).  One step is

    side stream:  dasp_gather_halo(x_p -> send)  ;  all_to_all_single(recv <- send)   (NCCL)
    main stream:  dasp_spmv(local, x_p -> y_p, alpha, 0)        (overlaps the exchange)
                  wait(side) ; dasp_spmv(remote, recv -> y_p, alpha, 1)

so only referenced x values move (a stencil slab exchanges two planes instead of all of x) and
the local part computes while they move.  x_p is the slab alone (no padded global x).
"""
from __future__ import annotations

import numpy as np

from . import dasp

# iterated SpMV feeds y back as the next x, so x and y must share one element type: FP64 (the
# north-star mode) or FP32 (R29).  FP16 plans take binary16 x but write FP32 y (R15), which would
# need a cast inside the loop; they are not part of the multi-GPU mode.
_ITER_DTYPES = {"f64": ("float64", 8), "f32": ("float32", 4)}


def _iter_dtype(dtype):
    if dtype not in _ITER_DTYPES:
        raise ValueError(f"row-slab iteration needs x and y of one type (f64 or f32), not {dtype!r}")
    import torch
    name, size = _ITER_DTYPES[dtype]
    return getattr(torch, name), size


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
               need_norm: bool = True, remap: bool = True) -> Slab:
    """generate_rows(row0, nrows) -> CSR of those rows (global columns).  reduce_max(v) -> max over ranks.
    need_norm=False skips the infinity norm (only the iteration needs it); remap=False keeps
    global columns (the halo mode splits them itself)."""
    starts = slab_bounds(row_lengths, world)
    r0, r1 = int(starts[rank]), int(starts[rank + 1])
    A = generate_rows(r0, r1 - r0)
    if world == 1 or not remap:         # one slab: no remap (also valid for rectangular matrices)
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
    slab = Slab(A.row_ptr, col, A.val, r0, r1 - r0, starts, S, inf_norm)
    slab.remapped = world > 1 and remap
    return slab


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
        tdt, self.elem_bytes = _iter_dtype(dtype)
        self._checked = False
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
                               variant=variant, check=not self._checked)   # full checks on the first call
                self._checked = True
            self.local_spmv = _local
        else:
            self.plan = None
            self.local_spmv = local_spmv

    def set_x(self, x_global: np.ndarray):
        """Load the global x (length n) into the padded layout of the current buffer."""
        import torch
        st, S = self.slab.starts, self.slab.S
        buf = np.zeros(self.world * S, dtype=_ITER_DTYPES[self.dtype][0])
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
        dsts = scatter_destinations(self.peer_base, self.rank, self.world, nb, self.n_pad, self.slab.S, self.elem_bytes)
        dasp.dasp_spmv_scatter(self.plan, self.x[self.cur], dsts, alpha, 0.0, torch.cuda.current_stream(self.device))
        self.hdl.barrier(channel=0)          # every rank's stores have landed before x is read
        self.cur = nb

    def x_global(self) -> np.ndarray:
        st, S = self.slab.starts, self.slab.S
        b = self.x[self.cur].cpu().numpy()
        return np.concatenate([b[q * S: q * S + st[q + 1] - st[q]] for q in range(self.world)])


# ------------------------------------------------------------------------------------------
# sparse halo exchange (f1)
# ------------------------------------------------------------------------------------------
class HaloSplit:
    """A slab split by column owner.  loc_*: CSR over local columns (c - starts[rank]);
    rem_*: CSR over halo positions; halo: the sorted global columns the slab references outside
    itself; recv_counts[q]: how many of them rank q owns (halo is grouped by owner because it is
    sorted and owners are contiguous column ranges)."""

    def __init__(self, loc, rem, halo, recv_counts):
        (self.loc_row_ptr, self.loc_col, self.loc_val) = loc
        (self.rem_row_ptr, self.rem_col, self.rem_val) = rem
        self.halo = halo
        self.recv_counts = recv_counts


def split_halo(row_ptr, col, val, starts, rank) -> HaloSplit:
    """Split a slab CSR (global columns, square matrix partitioned like its rows) into its local
    and remote sub-matrices; the per-row order of the nonzeros is kept in both."""
    starts = np.asarray(starts, dtype=np.int64)
    n = int(starts[-1])
    r0, r1 = int(starts[rank]), int(starts[rank + 1])
    rows = len(row_ptr) - 1
    c = np.asarray(col, dtype=np.int64)
    if len(c) and (c.min() < 0 or c.max() >= n):
        raise ValueError("split_halo: column out of range")
    own = (c >= r0) & (c < r1)
    row_of = np.repeat(np.arange(rows, dtype=np.int64), np.diff(row_ptr))

    def sub(mask, newcol):
        rp = np.zeros(rows + 1, dtype=np.int64)
        np.cumsum(np.bincount(row_of[mask], minlength=rows), out=rp[1:])
        return rp, np.ascontiguousarray(newcol, dtype=np.int32), np.ascontiguousarray(val[mask])

    loc = sub(own, c[own] - r0)
    rc = c[~own]
    mark = np.zeros(n, dtype=bool)
    mark[rc] = True
    halo = np.flatnonzero(mark).astype(np.int64)
    pos = np.cumsum(mark, dtype=np.int64) - 1
    rem = sub(~own, pos[rc])
    recv_counts = (np.searchsorted(halo, starts[1:]) - np.searchsorted(halo, starts[:-1])).astype(np.int64)
    return HaloSplit(loc, rem, halo, recv_counts)


def exchange_lists(split: HaloSplit, starts, rank, world, group=None, device="cpu"):
    """Setup-time exchange of the halo requests: returns (send_idx int32 local positions, grouped
    by destination rank, send_counts[q]).  One all_to_all of counts and one of indices."""
    import torch
    import torch.distributed as dist
    dev = torch.device(device)
    rc = torch.from_numpy(split.recv_counts.copy()).to(dev)
    sc = torch.empty_like(rc)
    dist.all_to_all_single(sc, rc, group=group)
    send_counts = sc.cpu().numpy().astype(np.int64)
    req = torch.from_numpy(split.halo.copy()).to(dev)
    got = torch.empty(int(send_counts.sum()), dtype=torch.int64, device=dev)
    dist.all_to_all_single(got, req, output_split_sizes=send_counts.tolist(),
                           input_split_sizes=split.recv_counts.tolist(), group=group)
    send_idx = got.cpu().numpy() - int(np.asarray(starts)[rank])
    rows = int(np.asarray(starts)[rank + 1] - np.asarray(starts)[rank])
    if len(send_idx) and (send_idx.min() < 0 or send_idx.max() >= rows):
        raise RuntimeError("exchange_lists: a peer requested a column this rank does not own")
    return send_idx.astype(np.int32), send_counts


class HaloSlabSpMV:
    """Iterated SpMV x_{k+1} = alpha*A*x_k with the sparse halo exchange overlapped with the
    local part (module doc).  ``spmv_local(x, y, alpha)``, ``spmv_remote(h, y, alpha)`` (y +=)
    and ``pack(x, idx, out)`` are pluggable for the CPU tests; the defaults are libdasp calls."""

    def __init__(self, slab: Slab, world: int, rank: int, device, dtype="f64", group=None,
                 variant=dasp.DASP_VARIANT_DEFAULT, spmv_local=None, spmv_remote=None, pack=None):
        import torch
        if getattr(slab, "remapped", False):
            raise ValueError("HaloSlabSpMV needs a slab with global columns (build_slab(remap=False))")
        self.slab, self.world, self.rank, self.group = slab, world, rank, group
        self.device = torch.device(device)
        self.dtype = dtype
        tdt, self.elem_bytes = _iter_dtype(dtype)
        self.split = split_halo(slab.row_ptr, slab.col, slab.val, slab.starts, rank)
        if world > 1:
            send_idx, self.send_counts = exchange_lists(self.split, slab.starts, rank, world, group,
                                                        self.device if self.device.type == "cuda" else "cpu")
        else:
            send_idx, self.send_counts = np.zeros(0, np.int32), np.zeros(1, np.int64)
        self.x = [torch.zeros(slab.rows, dtype=tdt, device=self.device) for _ in range(2)]
        self.cur = 0
        self.send_idx = torch.from_numpy(send_idx).to(self.device)
        self.send = torch.zeros(len(send_idx), dtype=tdt, device=self.device)
        self.recv = torch.zeros(len(self.split.halo), dtype=tdt, device=self.device)
        self.n_halo = len(self.split.halo)
        self.plan = self.plan_rem = None
        sp = self.split
        if spmv_local is None:
            if self.device.type != "cuda":
                raise RuntimeError("the libdasp slab SpMV needs a CUDA device (no CPU fallback)")
            dev = self.device.index or 0
            self.plan = dasp.dasp_plan_create(sp.loc_row_ptr, sp.loc_col, sp.loc_val, slab.rows, slab.rows, dtype,
                                              device=dev)
            if self.n_halo:
                self.plan_rem = dasp.dasp_plan_create(sp.rem_row_ptr, sp.rem_col, sp.rem_val, slab.rows, self.n_halo,
                                                      dtype, device=dev)

            def _loc(x, y, alpha):
                dasp.dasp_spmv(self.plan, x, y, alpha, 0.0, torch.cuda.current_stream(self.device), variant=variant,
                               check=False)

            def _rem(h, y, alpha):
                dasp.dasp_spmv(self.plan_rem, h, y, alpha, 1.0, torch.cuda.current_stream(self.device),
                               variant=variant, check=False)

            def _pack(x, idx, out):
                dasp.dasp_gather_halo(x, idx, out, torch.cuda.current_stream(self.device))
            spmv_local, spmv_remote, pack = _loc, _rem, _pack
            self.side = torch.cuda.Stream(self.device)
        else:
            self.side = None
        self.spmv_local, self.spmv_remote, self.pack = spmv_local, spmv_remote, pack

    @property
    def halo_bytes(self) -> int:
        """x bytes this rank receives per step (an all-gather would receive (n - rows)*8)."""
        return self.n_halo * self.elem_bytes

    def set_x(self, x_global: np.ndarray):
        import torch
        r0 = self.slab.row0
        self.x[self.cur].copy_(torch.from_numpy(np.ascontiguousarray(x_global[r0:r0 + self.slab.rows],
                                                                     dtype=_ITER_DTYPES[self.dtype][0])))

    def my_x(self):
        return self.x[self.cur]

    def _exchange(self):
        import torch.distributed as dist
        if self.world > 1:
            self.pack(self.x[self.cur], self.send_idx, self.send)
            dist.all_to_all_single(self.recv, self.send, output_split_sizes=self.split.recv_counts.tolist(),
                                   input_split_sizes=self.send_counts.tolist(), group=self.group)

    def step(self, alpha=1.0):
        import torch
        nxt = self.x[1 - self.cur]
        if self.side is not None:
            main = torch.cuda.current_stream(self.device)
            self.side.wait_stream(main)            # x_cur is final; the last remote SpMV read recv
            with torch.cuda.stream(self.side):
                self._exchange()
            self.spmv_local(self.x[self.cur], nxt, alpha)
            main.wait_stream(self.side)
        else:
            self._exchange()
            self.spmv_local(self.x[self.cur], nxt, alpha)
        if self.n_halo:
            self.spmv_remote(self.recv, nxt, alpha)
        self.cur = 1 - self.cur

    def x_global(self) -> np.ndarray:
        """The whole current x on every rank (test / readback helper, one all_gather)."""
        import torch
        import torch.distributed as dist
        st = self.slab.starts
        if self.world == 1:
            return self.x[self.cur].cpu().numpy().copy()
        S = int(max(np.diff(st)))
        buf = torch.zeros(S, dtype=self.x[0].dtype, device=self.device)
        buf[:self.slab.rows] = self.x[self.cur]
        parts = [torch.empty_like(buf) for _ in range(self.world)]
        dist.all_gather(parts, buf, group=self.group)
        return np.concatenate([parts[q].cpu().numpy()[: st[q + 1] - st[q]] for q in range(self.world)])
