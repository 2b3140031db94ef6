"""Pins for the CG oracle (oracle/cg.py) and its input generator (inputs/cg_gen.py).  CPU only."""
import math

import numpy as np
import pytest

from inputs import cg_gen
from oracle import cg as ocg


def _eigvec(nx, ny, nz, kx, ky, kz):
    """Separable sine mode: an eigenvector of both the 7- and the 27-point Dirichlet matrices
    (they are polynomials in the 1-D second-difference tridiagonal operators)."""
    ix, iy, iz = np.arange(1, nx + 1), np.arange(1, ny + 1), np.arange(1, nz + 1)
    sx, sy, sz = (np.sin(np.pi * k * i / (n + 1)) for k, i, n in ((kx, ix, nx), (ky, iy, ny), (kz, iz, nz)))
    return (sz[:, None, None] * sy[None, :, None] * sx[None, None, :]).ravel()


def _eigval(stencil, nx, ny, nz, kx, ky, kz):
    c = [math.cos(math.pi * k / (n + 1)) for k, n in ((kx, nx), (ky, ny), (kz, nz))]
    if stencil == 7:
        return 6 - 2 * sum(c)
    return 27 - math.prod(1 + 2 * ci for ci in c)


@pytest.mark.parametrize("stencil", [7, 27])
def test_matrix_structure_and_symmetry(stencil):
    A = cg_gen.matrix_scipy(5, 4, 3, stencil)
    assert A.shape == (60, 60)
    assert (A != A.T).nnz == 0
    d = A.diagonal()
    assert np.all(d == cg_gen.diag_value(stencil))
    # an interior point of a 5x4x3 grid has all stencil neighbours
    g = 2 + 5 * (1 + 4 * 1)
    assert A[g].nnz == stencil
    assert A[0].nnz == (8 if stencil == 27 else 4)  # corner
    w = np.linalg.eigvalsh(A.toarray())
    assert w.min() > 0  # SPD


@pytest.mark.parametrize("stencil", [7, 27])
def test_eigenvector_rhs_converges_in_one_step(stencil):
    """b = v (eigenvector, eigenvalue lam): p0 = r0 = v, alpha = 1/lam, x1 = v/lam exactly."""
    nx, ny, nz = 9, 7, 5
    A = cg_gen.matrix_scipy(nx, ny, nz, stencil)
    v = _eigvec(nx, ny, nz, 2, 3, 1)
    lam = _eigval(stencil, nx, ny, nz, 2, 3, 1)
    assert np.allclose(A @ v, lam * v, rtol=0, atol=1e-12)
    x, hist = ocg.cg(A, v, 1)
    assert np.allclose(x, v / lam, rtol=0, atol=1e-14)
    assert hist[0] < 1e-24 * np.dot(v, v)


@pytest.mark.parametrize("stencil", [7, 27])
def test_matches_direct_solve(stencil):
    """CG terminates in at most N steps in exact arithmetic; in fp64 it reaches the direct
    solution of a small well-conditioned system well before that."""
    A = cg_gen.matrix_scipy(6, 5, 4, stencil)
    b = cg_gen.rhs(A.shape[0])
    x, hist = ocg.cg(A, b, 60)
    xs = np.linalg.solve(A.toarray(), b)
    assert np.allclose(x, xs, rtol=1e-10, atol=1e-12)
    assert hist[-1] < 1e-20 * np.dot(b, b)


def test_search_directions_are_A_conjugate_and_residual_consistent():
    A = cg_gen.matrix_scipy(7, 6, 5, 27)
    b = cg_gen.rhs(A.shape[0], seed=5)
    x, hist, r, dirs = ocg.cg(A, b, 8, return_dirs=True)
    P = np.array(dirs[:8])
    G = P @ (A @ P.T)
    off = G - np.diag(np.diag(G))
    assert np.abs(off).max() < 1e-9 * np.abs(np.diag(G)).max()
    # recursive residual equals the true residual b - A x
    assert np.allclose(r, b - A @ x, rtol=0, atol=1e-12)
    assert math.isclose(hist[-1], float(r @ r), rel_tol=1e-12)


def test_rhs_generator():
    b = cg_gen.rhs(1000, seed=7)
    assert b.dtype == np.float64 and b.min() >= 0 and b.max() < 1
    assert np.all(b * 2.0 ** 53 == np.floor(b * 2.0 ** 53))
    assert np.array_equal(cg_gen.rhs(10, seed=7, g0=990), b[990:])
