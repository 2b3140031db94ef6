"""Multi-core host baseline (OpenMP C) of the Jacobi hot path for bench.py's ``cpu_parallel``
object: the same global-grid loop as the oracle on all host cores, bit-identical grid.  Not the
product (the product is libuniconn_b200.so) and not the parity oracle (oracle/ stays the plain
single-threaded checker)."""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "jacobi_omp.c")
_LIB = os.path.join(_HERE, "libjacobi_omp.so")
CFLAGS = ["-O3", "-march=native", "-std=c11", "-fopenmp", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared"]
_lib = None


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, _SRC, "-o", tmp])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        lib.omp_jacobi_run.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p,
                                       ctypes.c_int, ctypes.c_int, ctypes.c_void_p]
        lib.omp_jacobi_run.restype = ctypes.c_int
        lib.omp_threads.restype = ctypes.c_int
        _lib = lib
    return _lib


def threads() -> int:
    return _load().omp_threads()


def jacobi_run(g: np.ndarray, iters: int, topology: str = "ring", norm_every: int = 0, inplace: bool = False):
    """Like oracle.jacobi_run (returns (final array, sums of squares)); inplace=True runs on g
    itself (float32, C-contiguous) to keep copies out of a timed region."""
    a = g if inplace else np.array(g, dtype=np.float32, copy=True, order="C")
    assert a.dtype == np.float32 and a.flags.c_contiguous
    ny, nx = a.shape[0] - 2, a.shape[1]
    tmp = np.empty_like(a)
    m = (iters + norm_every - 1) // norm_every if norm_every > 0 else 0
    sums = np.zeros(max(m, 1), np.float64)
    rc = _load().omp_jacobi_run(nx, ny, 1 if topology == "ring" else 0, a.ctypes.data, tmp.ctypes.data, iters,
                                norm_every, sums.ctypes.data)
    if rc != 0:
        raise RuntimeError(f"omp_jacobi_run rc={rc}")
    return a, sums[:m]
