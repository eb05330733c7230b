"""GPU fuzz parity: seeded random CSR matrices mixing every row class (empty, short 1-4, medium 5-256,
long, an occasional row of 10^4-10^5 nonzeros), rectangular shapes, banded and scattered columns,
unsorted columns and duplicate entries, random panel sizes, both compute variants, all dtypes and the
x-window staging path -- on small integer values, so every y must equal the CPU oracle bit for bit
("fuzz recipe").  P:L77-93 (Alg. 1) defines y for every row whatever the class mix."""
import os

import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_sc_lu023_b200 import dasp  # noqa: E402

NP_VAL = {"f64": np.float64, "f16": np.float16, "f32": np.float32}
N_SEEDS = int(os.environ.get("DASP_FUZZ_SEEDS", "32"))   # a longer one-off run: DASP_FUZZ_SEEDS=256


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def random_csr(seed):
    rng = np.random.default_rng(1000 + seed)
    m = int(rng.integers(1, 40_000))
    n = int(max(1, m * rng.choice([0.25, 1.0, 1.0, 3.0]) + rng.integers(0, 50)))
    p = rng.dirichlet([1.0, 2.0, 3.0, 0.3]) * (1 - 0.1)                 # short, medium, ..., long
    cls = rng.choice(5, size=m, p=np.append(p, 0.1)[[4, 0, 1, 2, 3]] / 1.0)   # 0 empty 1 short 2 medium 3 med-wide 4 long
    lens = np.zeros(m, dtype=np.int64)
    lens[cls == 1] = rng.integers(1, 5, (cls == 1).sum())
    lens[cls == 2] = rng.integers(5, 33, (cls == 2).sum())
    lens[cls == 3] = rng.integers(33, 257, (cls == 3).sum())
    lens[cls == 4] = rng.integers(257, 3000, (cls == 4).sum())
    if seed % 3 == 0 and m > 4:
        lens[rng.integers(0, m)] = int(rng.integers(10_000, 100_000))  # a huge long row
    lens = np.minimum(lens, n if seed % 5 else 10 * n)               # duplicates may exceed n
    band = rng.random() < 0.5
    rows = []
    for i in range(m):
        L = int(lens[i])
        if L == 0:
            rows.append(np.zeros(0, np.int64))
            continue
        if band:
            centre = int(i * n / m)
            c = centre + rng.integers(-64, 65, L)
        else:
            c = rng.integers(0, n, L)
        c = np.clip(c, 0, n - 1)
        if seed % 5 != 0:                      # distinct columns, sorted or not
            c = np.unique(c)
            if seed % 2:
                rng.shuffle(c)
        rows.append(c)
    rp = np.zeros(m + 1, dtype=np.int64)
    rp[1:] = np.cumsum([len(r) for r in rows])
    col = np.concatenate(rows).astype(np.int32) if rp[-1] else np.zeros(0, np.int32)
    val = rng.integers(-3, 4, len(col)).astype(np.float64)
    return synth.CSR(m, n, rp, col, val, name=f"fuzz{seed}"), rng


@pytest.mark.parametrize("dt", ["f64", "f16", "f32"])
@pytest.mark.parametrize("seed", range(N_SEEDS))
def test_fuzz_bit_exact(seed, dt):
    A, rng = random_csr(seed)
    x = rng.integers(-3, 4, A.n).astype(np.float64)
    y0 = rng.integers(-3, 4, A.m).astype(np.float64)
    panel = int(rng.choice([0, 333, 4096, -1]))
    val = A.val.astype(NP_VAL[dt])
    xd = torch.from_numpy(x.astype(NP_VAL[dt])).cuda()
    ydt = torch.float64 if dt == "f64" else torch.float32
    stages = (1, 2) if dt != "f16" else (1,)
    for xs in stages:
        plan = dasp.dasp_plan_create(A.row_ptr, A.col, val, A.m, A.n, dt, device=0, panel_rows=panel, x_stage=xs)
        for alpha, beta in ((1.0, 0.0), (-2.0, 1.0)):
            ref, _ = oracle.spmv(A.row_ptr, A.col, A.val, x, alpha, beta, y0 if beta else None)
            for v in (dasp.DASP_VARIANT_MMA, dasp.DASP_VARIANT_CUDACORE):
                y = torch.from_numpy(y0).to(ydt).cuda()
                dasp.dasp_spmv(plan, xd, y, alpha, beta, variant=v)
                torch.cuda.synchronize()
                got = y.cpu().numpy().astype(np.float64)
                bad = np.nonzero(got != ref)[0]
                assert bad.size == 0, (A.name, dt, xs, v, alpha, bad[:5], got[bad[:5]], ref[bad[:5]])
        plan.destroy()


@pytest.mark.parametrize("dt", ["f64", "f16"])
@pytest.mark.parametrize("seed", range(0, 32, 4))
def test_fuzz_device_builder_bytes(seed, dt):
    """the GPU-side builder gives the host builder's bytes on the same fuzz matrices"""
    A, rng = random_csr(seed)
    panel = int(rng.choice([0, 333, 4096, -1]))
    val = A.val.astype(NP_VAL[dt])
    h = dasp.dasp_plan_create(A.row_ptr, A.col, val, A.m, A.n, dt, device=0, panel_rows=panel)
    d = dasp.dasp_plan_create_device(torch.from_numpy(A.row_ptr).cuda(), torch.from_numpy(A.col).cuda(),
                                     torch.from_numpy(val).cuda(), A.m, A.n, dt, panel_rows=panel)
    for arr in dasp.ARRAYS:
        assert np.array_equal(dasp.dasp_plan_copy_array(d, arr), dasp.dasp_plan_copy_array(h, arr)), (A.name, arr)
