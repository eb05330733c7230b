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
