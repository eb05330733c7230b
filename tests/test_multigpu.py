"""Row-slab multi-GPU mode on CPU: world_size-2 gloo process group, the same partition /
column-remap / in-place all-gather code as the NCCL path, with the local slab SpMV supplied
by the oracle (test infrastructure).  Pins P12 of SURVEY.md §8(c): K iterations of the
slab-parallel iteration == K oracle iterations on the whole matrix."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synth
from paper_conf_sc_lu023_b200.multigpu import SlabSpMV, build_slab, slab_bounds


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _oracle_local(slab):
    def f(x, y, alpha):
        yy, _ = oracle.spmv(slab.row_ptr, slab.col, slab.val, x.numpy(), alpha=alpha)
        y.copy_(torch.from_numpy(yy))
    return f


def _worker(rank, world, port, cfg, iters, out):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    spec = synth.config(*cfg)
    lens = synth.row_lengths(spec)

    def red(v):
        t = torch.tensor([v], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())
    slab = build_slab(lambda r0, nr: synth.generate(spec, r0, nr), lens, rank, world, red)
    it = SlabSpMV(slab, world, rank, "cpu", local_spmv=_oracle_local(slab))
    x0 = synth.vector(9, spec.n)
    it.set_x(x0)
    alpha = 1.0 / slab.inf_norm
    for _ in range(iters):
        it.step(alpha)
    if rank == 0:
        np.save(out, it.x_global())
        np.save(out + ".norm.npy", np.array([slab.inf_norm]))
    dist.destroy_process_group()


@pytest.mark.parametrize("cfg,world", [(("c1b",), 2), (("c5", None, 0, 2e-5), 2), (("c3", None, 0, 0.002), 3)])
def test_slab_iteration_matches_oracle(tmp_path, cfg, world):
    iters = 3
    out = str(tmp_path / "x.npy")
    mp.spawn(_worker, args=(world, _free_port(), cfg, iters, out), nprocs=world, join=True)
    got = np.load(out)
    inf_norm = float(np.load(out + ".norm.npy")[0])
    spec = synth.config(*cfg)
    A = synth.generate(spec)
    lens = np.diff(A.row_ptr)
    assert inf_norm == pytest.approx(max(np.add.reduceat(np.abs(A.val), A.row_ptr[:-1][lens > 0])), rel=1e-12)
    x = synth.vector(9, spec.n)
    for _ in range(iters):
        x, _ = oracle.spmv_csr(A, x, alpha=1.0 / inf_norm)
    # same products, same per-row order (the oracle is the local SpMV): the slab split changes nothing
    assert np.array_equal(got, x)


def test_slab_bounds_cover_and_balance():
    spec = synth.config("c3", scale=0.004)
    lens = synth.row_lengths(spec)
    for P in [2, 4, 8]:
        s = slab_bounds(lens, P)
        per = np.add.reduceat(lens, s[:-1]) if len(lens) else []
        assert s[0] == 0 and s[-1] == len(lens)
        assert max(per) <= lens.sum() / P + lens.max()   # balanced up to one row


def test_scatter_destinations_layout():
    from paper_conf_sc_lu023_b200.multigpu import scatter_destinations
    bases = [1000, 5000, 9000, 13000]
    d = scatter_destinations(bases, rank=2, world=4, buf_index=1, n_pad=40, S=10, elem_bytes=8)
    off = (40 + 2 * 10) * 8
    assert d == [9000 + off, 1000 + off, 5000 + off, 13000 + off]
    assert scatter_destinations([7], 0, 1, 0, 5, 5, 8) == [7]


# ---- sparse halo exchange ----
def test_split_halo_reassembles_rows():
    """The local and remote sub-matrices hold exactly the slab's nonzeros (per-row order kept),
    the halo is the sorted set of referenced remote columns grouped by owner, and
    A_slab x == A_loc x_p + A_rem x[halo] (oracle, within the FP64 tolerance)."""
    from paper_conf_sc_lu023_b200.multigpu import split_halo
    spec = synth.config("c3", scale=0.002)
    A = synth.generate(spec)
    lens = np.diff(A.row_ptr)
    starts = slab_bounds(lens, 3)
    x = synth.vector(5, spec.n)
    for rank in range(3):
        r0, r1 = int(starts[rank]), int(starts[rank + 1])
        rp = A.row_ptr[r0:r1 + 1] - A.row_ptr[r0]
        col = A.col[A.row_ptr[r0]:A.row_ptr[r1]]
        val = A.val[A.row_ptr[r0]:A.row_ptr[r1]]
        sp = split_halo(rp, col, val, starts, rank)
        assert np.array_equal(np.diff(sp.loc_row_ptr) + np.diff(sp.rem_row_ptr), np.diff(rp))
        assert np.all(np.diff(sp.halo) > 0)
        assert not np.any((sp.halo >= r0) & (sp.halo < r1))
        assert sp.recv_counts[rank] == 0 and sp.recv_counts.sum() == len(sp.halo)
        assert np.array_equal(np.unique(col[(col < r0) | (col >= r1)]), sp.halo)
        for i in range(r1 - r0):                          # row i's nonzeros, order preserved
            c = col[rp[i]:rp[i + 1]]
            lc = sp.loc_col[sp.loc_row_ptr[i]:sp.loc_row_ptr[i + 1]] + r0
            rc = sp.halo[sp.rem_col[sp.rem_row_ptr[i]:sp.rem_row_ptr[i + 1]]]
            own = (c >= r0) & (c < r1)
            assert np.array_equal(c[own], lc) and np.array_equal(c[~own], rc)
        y_ref, s = oracle.spmv(rp, col, val, x)
        yl, _ = oracle.spmv(sp.loc_row_ptr, sp.loc_col, sp.loc_val, x[r0:r1])
        y, _ = oracle.spmv(sp.rem_row_ptr, sp.rem_col, sp.rem_val, x[sp.halo], beta=1.0, y0=yl)
        assert oracle.tolerance_ok(y, y_ref, s).all()


def test_split_halo_stencil_volume():
    """A 27-point stencil slab references only the neighbouring planes: the halo is far smaller
    than the all-gathered remainder of x."""
    from paper_conf_sc_lu023_b200.multigpu import split_halo
    spec = synth.config("c2", scale=0.25)            # 32^3
    A = synth.generate(spec)
    starts = slab_bounds(np.diff(A.row_ptr), 4)
    r0, r1 = int(starts[1]), int(starts[2])
    rp = A.row_ptr[r0:r1 + 1] - A.row_ptr[r0]
    sp = split_halo(rp, A.col[A.row_ptr[r0]:A.row_ptr[r1]], A.val[A.row_ptr[r0]:A.row_ptr[r1]], starts, 1)
    nx = round(spec.m ** (1 / 3))
    assert len(sp.halo) <= 2 * (nx * nx + nx + 1) * 2     # at most two planes (+ edge) per side
    assert len(sp.halo) < (spec.n - (r1 - r0)) / 4


def _halo_worker(rank, world, port, cfg, iters, out):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_sc_lu023_b200.multigpu import HaloSlabSpMV
    spec = synth.config(*cfg)
    lens = synth.row_lengths(spec)

    def red(v):
        t = torch.tensor([v], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())
    slab = build_slab(lambda r0, nr: synth.generate(spec, r0, nr), lens, rank, world, red, remap=False)
    holder = {}

    def loc(x, y, alpha):
        sp = holder["it"].split
        yy, _ = oracle.spmv(sp.loc_row_ptr, sp.loc_col, sp.loc_val, x.numpy(), alpha=alpha)
        y.copy_(torch.from_numpy(yy))

    def rem(h, y, alpha):
        sp = holder["it"].split
        yy, _ = oracle.spmv(sp.rem_row_ptr, sp.rem_col, sp.rem_val, h.numpy(), alpha=alpha, beta=1.0, y0=y.numpy())
        y.copy_(torch.from_numpy(yy))

    def pack(x, idx, outb):
        outb.copy_(x[idx.long()])
    it = HaloSlabSpMV(slab, world, rank, "cpu", spmv_local=loc, spmv_remote=rem, pack=pack)
    holder["it"] = it
    it.set_x(synth.vector(9, spec.n))
    for _ in range(iters):
        it.step(1.0 / slab.inf_norm)
    xg = it.x_global()
    if rank == 0:
        np.save(out, xg)
        np.save(out + ".norm.npy", np.array([slab.inf_norm]))
    dist.destroy_process_group()


@pytest.mark.parametrize("cfg,world", [(("c1b",), 2), (("c2", None, 0, 0.25), 3), (("c3", None, 0, 0.002), 3)])
def test_halo_iteration_matches_oracle(tmp_path, cfg, world):
    """Halo mode over gloo: K iterations == K oracle iterations on the whole matrix, up to the one
    extra rounding of adding the local and remote partial sums (|err| <= 2^-52 per step, norm-1 map)."""
    iters = 3
    out = str(tmp_path / "x.npy")
    mp.spawn(_halo_worker, args=(world, _free_port(), cfg, iters, out), nprocs=world, join=True)
    got = np.load(out)
    inf_norm = float(np.load(out + ".norm.npy")[0])
    spec = synth.config(*cfg)
    A = synth.generate(spec)
    x = synth.vector(9, spec.n)
    for _ in range(iters):
        x, _ = oracle.spmv_csr(A, x, alpha=1.0 / inf_norm)
    assert np.allclose(got, x, rtol=0, atol=1e-13 * max(1.0, np.abs(x).max()))


def test_slab_iteration_dtypes():
    """The iteration feeds y back as x: x and y buffers take the plan's one element type (f64 / f32);
    FP16 plans (binary16 x, f32 y) are rejected instead of reading float64 storage as halves."""
    spec = synth.config("c1b")
    lens = synth.row_lengths(spec)
    slab = build_slab(lambda r0, nr: synth.generate(spec, r0, nr), lens, 0, 1)
    for dt, tdt in (("f64", torch.float64), ("f32", torch.float32)):
        it = SlabSpMV(slab, 1, 0, "cpu", dtype=dt, local_spmv=lambda x, y, a: y.copy_(x[:len(y)] * a))
        assert it.x[0].dtype == tdt and it.elem_bytes == tdt.itemsize
        it.set_x(synth.vector(3, spec.n))
        it.step(0.5)
        assert it.x_global().dtype == (np.float64 if dt == "f64" else np.float32)
    with pytest.raises(ValueError):
        SlabSpMV(slab, 1, 0, "cpu", dtype="f16", local_spmv=lambda x, y, a: None)
