"""Seeded synthetic inputs for the Jacobi hot path (shared by the oracle tests and the CUDA path).

This module holds NO arithmetic of the method (no stencil, no norm): it only builds the
initial global field that both sides start from.  The recipe (DESIGN.md "Input recipe",
SURVEY.md §8(c) readings G2/G5/G6) is:

* Global array ``(NY+2) x NX`` float32, row-major, x contiguous.  Rows ``1..NY`` are the
  computed rows (global computed-row index ``gy = row - 1``); rows ``0`` and ``NY+1`` are the
  y-halo / y-boundary rows; columns ``0`` and ``NX-1`` are fixed (Dirichlet) columns.
  The paper's workload is a 2^14 x 2^14 fp32 grid, 5-point star, split equally along y
  (§VI-C); it does not state the initial field or boundary data (G5, G6).
* Interior (rows 1..NY, columns 1..NX-2): ``u = (splitmix64(seed ^ (gy*NX + x)) >> 40) * 2^-24``,
  a 24-bit value in [0, 1), exactly representable in fp32.  ``zero_init`` sets it to 0.
* ``topology="ring"`` (y periodic, every listing posts to top and bottom unconditionally,
  P:43-46): column 0 = ``(float)sin(2*pi*gy/NY)`` computed in double,
  column NX-1 = 0; halo row 0 = row NY and halo row NY+1 = row 1 (wrap).
* ``topology="dirichlet"`` (validation, the sin-sinh problem): row 0 = ``(float)sin(pi*x/(NX-1))``,
  row NY+1 = 0, columns 0 and NX-1 = 0.

``splitmix64`` is the public-domain counter-based mixer (Steele, Lea, Flood 2014); the CUDA
path implements the same counter-based generator independently (device-side init) and the
tests check the two agree bit-for-bit at iteration 0.
"""
from __future__ import annotations

import math

import numpy as np

DEFAULT_SEED = 0x5EED
TOPOLOGIES = ("ring", "dirichlet")

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)


def splitmix64(x: np.ndarray) -> np.ndarray:
    """Vectorised splitmix64 finaliser on uint64 (wrapping arithmetic)."""
    z = x.astype(np.uint64, copy=True)
    with np.errstate(over="ignore"):
        z += np.uint64(0x9E3779B97F4A7C15)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        z = z ^ (z >> np.uint64(31))
    return z


def interior_rows(nx: int, gy0: int, rows: int, seed: int = DEFAULT_SEED) -> np.ndarray:
    """Random interior values of computed rows ``gy0 .. gy0+rows-1`` (all NX columns)."""
    gy = np.arange(gy0, gy0 + rows, dtype=np.uint64)[:, None]
    x = np.arange(nx, dtype=np.uint64)[None, :]
    with np.errstate(over="ignore"):
        ctr = gy * np.uint64(nx) + x
    h = splitmix64(np.uint64(seed) ^ ctr)
    return ((h >> np.uint64(40)).astype(np.float64) * 2.0 ** -24).astype(np.float32)


def ring_left_column(ny: int) -> np.ndarray:
    """Column 0 of the ring problem for computed rows gy = 0..NY-1 (double sin, rounded once)."""
    return np.array([math.sin(2.0 * math.pi * gy / ny) for gy in range(ny)], dtype=np.float64).astype(np.float32)


def dirichlet_top_row(nx: int) -> np.ndarray:
    """Row 0 of the dirichlet-y (sin-sinh) problem."""
    return np.array([math.sin(math.pi * x / (nx - 1)) for x in range(nx)], dtype=np.float64).astype(np.float32)


def global_field(nx: int, ny: int, topology: str = "ring", seed: int = DEFAULT_SEED,
                 zero_init: bool = False, chunk_rows: int = 1024) -> np.ndarray:
    """The full ``(NY+2) x NX`` float32 initial array (see module docstring)."""
    if topology not in TOPOLOGIES:
        raise ValueError(f"topology must be one of {TOPOLOGIES}")
    if nx < 3 or ny < 1:
        raise ValueError("need nx >= 3 and ny >= 1")
    g = np.zeros((ny + 2, nx), dtype=np.float32)
    if not zero_init:
        for gy0 in range(0, ny, chunk_rows):
            rows = min(chunk_rows, ny - gy0)
            g[1 + gy0:1 + gy0 + rows, :] = interior_rows(nx, gy0, rows, seed)
    if topology == "ring":
        g[1:ny + 1, 0] = ring_left_column(ny)
        g[1:ny + 1, nx - 1] = 0.0
        g[0, :] = g[ny, :]
        g[ny + 1, :] = g[1, :]
    else:
        g[1:ny + 1, 0] = 0.0
        g[1:ny + 1, nx - 1] = 0.0
        g[0, :] = dirichlet_top_row(nx)
        g[ny + 1, :] = 0.0
    return g


def rank_slab(g: np.ndarray, rank: int, size: int, topology: str = "ring") -> np.ndarray:
    """Rank ``rank``'s ``(n+2) x NX`` slab of the global array (rows r*n .. r*n+n+1).

    Equal y-split; NY % size must be 0 (reading G4).  In ring topology the global
    halo rows 0 and NY+1 already hold the wrapped rows, so slicing is enough.
    """
    ny = g.shape[0] - 2
    if ny % size:
        raise ValueError("NY must be divisible by the number of ranks")
    n = ny // size
    return np.ascontiguousarray(g[rank * n: rank * n + n + 2, :])


def rows_field(nx: int, ny: int, gys, topology: str = "ring", seed: int = DEFAULT_SEED,
               zero_init: bool = False) -> np.ndarray:
    """Rows of the global initial field by computed-row index gy (-1 = the top boundary/halo row,
    NY = the bottom one; ring indices wrap), without materialising the global array."""
    out = np.zeros((len(gys), nx), dtype=np.float32)
    for j, gy in enumerate(gys):
        if topology == "ring":
            gyw = gy % ny
            if not zero_init:
                out[j] = interior_rows(nx, gyw, 1, seed)[0]
            out[j, 0] = np.float32(math.sin(2.0 * math.pi * gyw / ny))
            out[j, nx - 1] = 0.0
        elif gy < 0:
            out[j] = dirichlet_top_row(nx)
        elif gy >= ny:
            out[j] = 0.0
        else:
            if not zero_init:
                out[j] = interior_rows(nx, gy, 1, seed)[0]
            out[j, 0] = 0.0
            out[j, nx - 1] = 0.0
    return out


def slab_field(nx: int, ny: int, rank: int, size: int, topology: str = "ring",
               seed: int = DEFAULT_SEED, zero_init: bool = False) -> np.ndarray:
    """Rank slab generated directly (without materialising the global array)."""
    n = ny // size
    if ny % size:
        raise ValueError("NY must be divisible by the number of ranks")
    s = np.zeros((n + 2, nx), dtype=np.float32)
    rows = [(rank * n + j - 1) for j in range(n + 2)]  # computed-row index for slab row j
    for j, gy in enumerate(rows):
        if topology == "ring":
            gyw = gy % ny
            if not zero_init:
                s[j] = interior_rows(nx, gyw, 1, seed)[0]
            s[j, 0] = np.float32(math.sin(2.0 * math.pi * gyw / ny))
            s[j, nx - 1] = 0.0
        else:
            if gy < 0:
                s[j] = dirichlet_top_row(nx)
            elif gy >= ny:
                s[j] = 0.0
            else:
                if not zero_init:
                    s[j] = interior_rows(nx, gy, 1, seed)[0]
                s[j, 0] = 0.0
                s[j, nx - 1] = 0.0
    return s
