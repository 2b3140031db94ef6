"""CPU oracle for the CG workload -- TEST INFRASTRUCTURE ONLY (same rules as oracle/__init__.py:
only tests/, __graft_entry__.smoke() and benchmark baselines may import it).

Conjugate Gradient as the paper's §VI-D evaluates it (each iteration one SpMV that
needs the whole x -- gathered with AllGatherv -- and two dot products that need an AllReduce),
written as the textbook algorithm (Hestenes & Stiefel 1952; Saad, Iterative Methods, Alg. 6.18),
in float64, step by step in this order:

    r0 = b - A x0 ;  p0 = r0 ;  rr0 = r0.r0
    for k = 0, 1, ...:
        q     = A p_k                  (SpMV)
        alpha = rr_k / (p_k . q)       (dot product 1)
        x     = x + alpha p_k
        r     = r - alpha q
        rr_k+1 = r . r                 (dot product 2)
        beta  = rr_k+1 / rr_k
        p_k+1 = r + beta p_k

The matrix-vector product and the dot products are library primitives (scipy CSR @, numpy
dot).  Returns the iterate and the history of rr after every iteration.
Pins: tests/test_oracle_cg.py (eigenvector right-hand side -> exact in one step, agreement with
a direct solve after N steps, A-conjugacy of the search directions, true vs recursive residual).
"""
from __future__ import annotations

import numpy as np


def cg(A, b: np.ndarray, iters: int, x0: np.ndarray | None = None, return_dirs: bool = False):
    b = np.asarray(b, dtype=np.float64)
    x = np.zeros_like(b) if x0 is None else np.array(x0, dtype=np.float64)
    r = b - A @ x
    p = r.copy()
    rr = float(np.dot(r, r))
    hist = []
    dirs = [p.copy()] if return_dirs else None
    for _ in range(iters):
        q = A @ p
        alpha = rr / float(np.dot(p, q))
        x = x + alpha * p
        r = r - alpha * q
        rr_new = float(np.dot(r, r))
        beta = rr_new / rr
        rr = rr_new
        hist.append(rr)
        p = r + beta * p
        if return_dirs:
            dirs.append(p.copy())
    if return_dirs:
        return x, np.array(hist), r, dirs
    return x, np.array(hist)
