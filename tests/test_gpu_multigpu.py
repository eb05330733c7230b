"""Row-slab iteration on the GPU (world size 1 here: one GPU per gpurun box): the NCCL path and
the fused scatter path (symmetric memory + dasp_spmv_scatter + device barrier) against K oracle
iterations.  The multi-rank host logic is covered on CPU by tests/test_multigpu.py."""
import socket

import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def pg():
    import torch.distributed as dist
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    torch.cuda.set_device(0)
    dist.init_process_group("nccl", init_method=f"tcp://127.0.0.1:{port}", rank=0, world_size=1,
                            device_id=torch.device("cuda", 0))
    yield dist
    dist.destroy_process_group()


@pytest.mark.parametrize("fused", [False, True])
def test_slab_iteration_world1(pg, fused):
    from paper_conf_sc_lu023_b200.multigpu import SlabSpMV, build_slab
    spec = synth.config("c5", scale=4e-4)
    lens = synth.row_lengths(spec)
    slab = build_slab(lambda r0, nr: synth.generate(spec, r0, nr), lens, 0, 1)
    it = SlabSpMV(slab, 1, 0, "cuda:0", fused=fused)
    x0 = synth.vector(61, spec.n)
    it.set_x(x0)
    alpha = 1.0 / slab.inf_norm
    for _ in range(3):
        it.step(alpha)
    torch.cuda.synchronize()
    got = it.x_global()
    A = synth.generate(spec)
    x = x0
    for _ in range(3):
        x_new, s = oracle.spmv_csr(A, x, alpha=alpha)
        x = x_new
    # each iterate is within tolerance of the oracle applied to the GPU's previous iterate; after
    # three steps of a norm-1 map the accumulated difference stays tiny
    assert np.allclose(got, x, rtol=0, atol=1e-12)
