"""Consumers of a DASP plan: iterative methods that amortise the
preprocessing (P:L420 -- "acceptable if more SpMV kernel calls are needed in an iterative
solver").  The SpMV is libdasp; the vector updates are plain torch ops (plumbing).
"""
from __future__ import annotations

from dataclasses import dataclass

from . import dasp


@dataclass
class SolveResult:
    x: object
    iterations: int
    residual_norm: float
    converged: bool


def conjugate_gradient(plan: dasp.Plan, b, x0=None, tol: float = 1e-10, maxiter: int = 1000, stream=None):
    """CG for SPD A (FP64 plan): x minimising ||b - A x||, stopping at ||r|| <= tol * ||b||."""
    import torch
    if plan.dtype != "f64":
        raise ValueError("CG needs an FP64 plan")
    x = torch.zeros_like(b) if x0 is None else x0.clone()
    r = b.clone()
    if x0 is not None:                                   # r = b - A x0
        dasp.dasp_spmv(plan, x, r, -1.0, 1.0, stream)
    p = r.clone()
    Ap = torch.empty_like(b)
    rr = torch.dot(r, r)
    bnorm = torch.linalg.vector_norm(b)
    it = 0
    for it in range(1, maxiter + 1):
        dasp.dasp_spmv(plan, p, Ap, 1.0, 0.0, stream)
        alpha = rr / torch.dot(p, Ap)
        x.add_(p, alpha=alpha)
        r.sub_(Ap, alpha=alpha)
        rr_new = torch.dot(r, r)
        if it % 10 == 0 or it == maxiter:
            if float(torch.sqrt(rr_new)) <= tol * float(bnorm):
                rr = rr_new
                break
        p.mul_(rr_new / rr).add_(r)
        rr = rr_new
    res = float(torch.sqrt(rr))
    return SolveResult(x, it, res, res <= tol * float(bnorm))


def power_iteration(plan: dasp.Plan, x0, iters: int = 100, stream=None):
    """Dominant eigenvalue estimate by x <- A x / ||A x|| (any square plan, FP64)."""
    import torch
    x = x0 / torch.linalg.vector_norm(x0)
    y = torch.empty_like(x)
    lam = 0.0
    for _ in range(iters):
        dasp.dasp_spmv(plan, x, y, 1.0, 0.0, stream)
        lam = float(torch.dot(x, y))
        x = y / torch.linalg.vector_norm(y)
    return lam, x
