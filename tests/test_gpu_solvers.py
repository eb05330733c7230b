"""f4: a solver consuming the plan -- CG on the SPD 27-point stencil, residual checked by the oracle."""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


def test_cg_on_spd_stencil():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sc_lu023_b200 import dasp, solvers
    A = synth.generate(synth.config("c2", scale=24 / 128, val_mode=synth.VAL_SPD))
    plan = dasp.dasp_plan_create(A.row_ptr, A.col, A.val, A.m, A.n, "f64")
    b_np = synth.vector(81, A.m)
    b = torch.from_numpy(b_np).cuda()
    res = solvers.conjugate_gradient(plan, b, tol=1e-10, maxiter=500)
    assert res.converged
    x = res.x.cpu().numpy()
    Ax, s = oracle.spmv_csr(A, x)
    assert np.linalg.norm(Ax - b_np) <= 1e-9 * np.linalg.norm(b_np)
    lam, _ = solvers.power_iteration(plan, torch.ones(A.n, dtype=torch.float64, device="cuda"), iters=50)
    assert 0 < lam <= 2 * 27.5                          # Gershgorin bound of the SPD stencil
