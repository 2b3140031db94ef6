"""Seeded synthetic inputs for the CG workload (§VI-D).

No arithmetic of the method lives here -- only the problem definition both sides start from:

* Matrix: the 3-D 27-point (or 7-point) stencil matrix on an nx x ny x nz grid with Dirichlet
  boundaries, N = nx*ny*nz unknowns, global row g = x + nx*(y + ny*z) (x fastest).
  27-point: A[g][g] = 26, A[g][h] = -1 for every other grid point h of the 3x3x3 neighbourhood
  inside the grid.  7-point: A[g][g] = 6, -1 for the 6 face neighbours.  Both are symmetric,
  irreducibly diagonally dominant M-matrices, hence SPD.  They stand in for the paper's
  SuiteSparse 3-D FEM matrices (Serena 1.39 M rows, Queen_4147 4.1 M rows), which need
  datasets: a 112^3 27-point grid has Serena's row count, 160^3 Queen_4147's.
* Right-hand side: b[g] = (splitmix64(seed ^ g) >> 11) * 2^-53, a 53-bit value in [0, 1).
* Start vector x0 = 0; rows split equally over the ranks ("without accounting for the
  number of nonzeros").
"""
from __future__ import annotations

import numpy as np

from .gen import splitmix64

DEFAULT_SEED = 0xC6


def rhs(n: int, seed: int = DEFAULT_SEED, g0: int = 0) -> np.ndarray:
    g = np.arange(g0, g0 + n, dtype=np.uint64)
    h = splitmix64(np.uint64(seed) ^ g)
    return (h >> np.uint64(11)).astype(np.float64) * 2.0 ** -53


def stencil_offsets(stencil: int):
    if stencil == 27:
        return [(dx, dy, dz) for dz in (-1, 0, 1) for dy in (-1, 0, 1) for dx in (-1, 0, 1)]
    if stencil == 7:
        return [(0, 0, -1), (0, -1, 0), (-1, 0, 0), (0, 0, 0), (1, 0, 0), (0, 1, 0), (0, 0, 1)]
    raise ValueError("stencil must be 7 or 27")


def diag_value(stencil: int) -> float:
    return 26.0 if stencil == 27 else 6.0


def matrix_scipy(nx: int, ny: int, nz: int, stencil: int = 27):
    """The matrix as scipy.sparse CSR (columns sorted), built from the definition above."""
    import scipy.sparse as sp
    N = nx * ny * nz
    idx = np.arange(N)
    x, y, z = idx % nx, (idx // nx) % ny, idx // (nx * ny)
    rows, cols, vals = [], [], []
    for dx, dy, dz in stencil_offsets(stencil):
        xx, yy, zz = x + dx, y + dy, z + dz
        ok = (xx >= 0) & (xx < nx) & (yy >= 0) & (yy < ny) & (zz >= 0) & (zz < nz)
        rows.append(idx[ok])
        cols.append((xx + nx * (yy + ny * zz))[ok])
        v = diag_value(stencil) if (dx, dy, dz) == (0, 0, 0) else -1.0
        vals.append(np.full(ok.sum(), v))
    A = sp.csr_matrix((np.concatenate(vals), (np.concatenate(rows), np.concatenate(cols))), shape=(N, N))
    A.sort_indices()
    return A
