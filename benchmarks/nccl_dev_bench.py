#!/usr/bin/env python
"""In-box "native" comparator: the paper's Listing-3 structure (PAPER.md P:52-74,
dedicated boundary blocks that compute the first/last rows, put them into the neighbours' halos
and synchronise; one iteration per launch) on NCCL 2.28's device API -- LSA peer pointers of a
symmetric window + an LSA barrier -- timed at the bench workload beside the product kernel.

    python benchmarks/nccl_dev_bench.py [--nx 16384] [--ny 16384] [--iters 100] [--reps 5]

One process = one rank (P = 1 here: top = bottom = itself in ring topology; NCCL allows one rank
per GPU, so P > 1 needs one GPU per rank).  Prints one JSON line: GLUPS, ms per iteration, and the
fraction of the measured copy bandwidth at 8 B per point (the one-iteration roofline).
"""
from __future__ import annotations

import argparse
import ctypes
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "benchmarks", "native", "libuc_nccl_dev.so")


def load():
    if not os.path.exists(LIB):
        raise ImportError(f"{LIB} not built (python -c 'import __graft_entry__ as g; g.build()')")
    lib = ctypes.CDLL(LIB)
    vp = ctypes.c_void_p
    lib.ucn_unique_id.argtypes = [vp]
    lib.ucn_create.argtypes = [ctypes.c_int, ctypes.c_int, vp, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                               ctypes.POINTER(vp)]
    lib.ucn_copy_in.argtypes = [vp, vp]
    lib.ucn_copy_out.argtypes = [vp, vp]
    lib.ucn_run.argtypes = [vp, ctypes.c_int, vp]
    lib.ucn_destroy.argtypes = [vp]
    lib.ucn_last_error.restype = ctypes.c_char_p
    return lib


class NcclDevJacobi:
    """One rank of the comparator: (n+2) x nx slabs in an NCCL symmetric window."""

    def __init__(self, lib, rank, nranks, uid: bytes, nx, n, top, bottom):
        self.lib, self.nx, self.n = lib, nx, n
        self.h = ctypes.c_void_p()
        buf = ctypes.create_string_buffer(uid, 128)
        self._check(lib.ucn_create(rank, nranks, buf, nx, n, top, bottom, ctypes.byref(self.h)), "ucn_create")

    def _check(self, rc, what):
        if rc != 0:
            raise RuntimeError(f"{what}: {self.lib.ucn_last_error().decode()}")

    def copy_in(self, slab: np.ndarray):
        a = np.ascontiguousarray(slab, dtype=np.float32)
        assert a.shape == (self.n + 2, self.nx)
        self._check(self.lib.ucn_copy_in(self.h, a.ctypes.data), "ucn_copy_in")

    def copy_out(self) -> np.ndarray:
        a = np.empty((self.n + 2, self.nx), np.float32)
        self._check(self.lib.ucn_copy_out(self.h, a.ctypes.data), "ucn_copy_out")
        return a

    def run(self, iters, stream=None):
        self._check(self.lib.ucn_run(self.h, iters, stream), "ucn_run")

    def destroy(self):
        if self.h:
            self._check(self.lib.ucn_destroy(self.h), "ucn_destroy")
            self.h = ctypes.c_void_p()


def unique_id(lib) -> bytes:
    b = ctypes.create_string_buffer(128)
    if lib.ucn_unique_id(b) != 0:
        raise RuntimeError(lib.ucn_last_error().decode())
    return b.raw


def single_rank(nx, ny, topology):
    """P = 1 solver: ring = self-neighbour, dirichlet = fixed halo rows."""
    lib = load()
    nb = 0 if topology == "ring" else -1
    return NcclDevJacobi(lib, 0, 1, unique_id(lib), nx, ny, nb, nb)


def main():
    import torch

    sys.path.insert(0, ROOT)
    from inputs import gen

    ap = argparse.ArgumentParser()
    ap.add_argument("--nx", type=int, default=16384)
    ap.add_argument("--ny", type=int, default=16384)
    ap.add_argument("--iters", type=int, default=100)
    ap.add_argument("--reps", type=int, default=5)
    a = ap.parse_args()
    torch.cuda.set_device(0)
    J = single_rank(a.nx, a.ny, "ring")
    J.copy_in(gen.global_field(a.nx, a.ny, "ring"))
    st = torch.cuda.Stream()
    J.run(10, st.cuda_stream)
    times = []
    for _ in range(a.reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        J.run(a.iters, st.cuda_stream)
        e1.record(st)
        torch.cuda.synchronize()
        times.append(e0.elapsed_time(e1))
    times = sorted(times)[1:-1] if len(times) > 2 else times  # drop the lowest and highest
    ms = sum(times) / len(times)
    pts = a.ny * (a.nx - 2) * a.iters
    peak = None
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            peak = float(json.load(f)["hbm_gbs"])
    gbs = 8.0 * a.ny * a.nx * a.iters / (ms / 1e3) / 1e9
    print(json.dumps({"comparator": "nccl_device_api_listing3", "nccl": torch.cuda.nccl.version(),
                      "workload": f"jacobi2d_{a.nx}x{a.ny}_P1_ring", "iters": a.iters, "reps": a.reps,
                      "glups": round(pts / (ms / 1e3) / 1e9, 2), "ms_per_iteration": round(ms / a.iters, 5),
                      "gbs_at_8B_per_point": round(gbs, 1),
                      "frac_of_copy_peak": None if peak is None else round(gbs / peak, 4)}))
    J.destroy()


if __name__ == "__main__":
    main()
