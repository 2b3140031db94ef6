"""CPU parity oracle for the Jacobi hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product path
(``paper_conf_cluster_sagbilieinu25_b200``) never imports it and shares no code with it.

``oracle/jacobi_oracle.c`` is a plain single-threaded C Jacobi over the global grid
(see its header for the PAPER.md passages it follows).  It is compiled with
``-O2 -ffp-contract=off -fno-fast-math`` so that fp32 ``0.25f*((l+r)+(t+b))`` is evaluated
exactly as written (no FMA, no FTZ).

Every function here has a pin in ``tests/test_oracle.py``; nothing is "parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "jacobi_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
CFLAGS = ["-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared"]

_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (idempotent)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, _SRC, "-o", tmp])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    with _lock:
        if _lib is None:
            lib = ctypes.CDLL(build())
            lib.oracle_jacobi_run.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                              ctypes.c_void_p, ctypes.c_int, ctypes.c_int,
                                              ctypes.c_void_p]
            lib.oracle_jacobi_run.restype = ctypes.c_int
            lib.oracle_num_norms.argtypes = [ctypes.c_int, ctypes.c_int]
            lib.oracle_num_norms.restype = ctypes.c_int
            _lib = lib
    return _lib


def jacobi_run(g: np.ndarray, iters: int, topology: str = "ring", norm_every: int = 0):
    """Run ``iters`` iterations on a copy of the ``(NY+2) x NX`` float32 global array.

    Returns ``(final_global_array, sums_of_squares)`` where ``sums_of_squares[m]`` is
    sum over all updated points of d^2 (d = new - old, fp32; squared and summed in double,
    sequentially) at iteration ``k = m * norm_every``.  ``norm = sqrt(sum)``.
    """
    if topology not in ("ring", "dirichlet"):
        raise ValueError("topology must be 'ring' or 'dirichlet'")
    a = np.array(g, dtype=np.float32, copy=True, order="C")
    if a.ndim != 2:
        raise ValueError("expected a 2-D (NY+2) x NX array")
    ny, nx = a.shape[0] - 2, a.shape[1]
    lib = _load()
    m = lib.oracle_num_norms(iters, norm_every)
    sums = np.zeros(max(m, 1), dtype=np.float64)
    rc = lib.oracle_jacobi_run(nx, ny, 1 if topology == "ring" else 0, a.ctypes.data, iters,
                               norm_every, sums.ctypes.data if norm_every > 0 else None)
    if rc != 0:
        raise RuntimeError(f"oracle_jacobi_run failed rc={rc}")
    return a, sums[:m]
