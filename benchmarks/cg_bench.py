#!/usr/bin/env python
"""CG workload benchmark (§VI-D).

    python benchmarks/cg_bench.py [--grid 160] [--stencil 27] [--iters 100] [--steps 5] [--mode device]
    torchrun --nproc-per-node N --master-addr 127.0.0.1 benchmarks/cg_bench.py ...

Default problem: the 160^3 27-point matrix (4.1 M rows, 110 M nonzeros: Queen_4147's row count,
P:432); --grid 112 gives Serena's.  A step = `iters` CG iterations (one CUDA graph); reported:
iterations/s (the paper reports CG run time for 10K iterations, Fig. 6) and the achieved HBM
bandwidth of an iteration against the measured copy peak, with the algorithmic bytes per
iteration (float64 values, int32 columns, int64 row pointers):
  SpMV  8(n+1) + 12 nnz + 8 n (q) + 8 N (p, each element at least once)
  update 6 x 8 n (x, r read+write; p, q read), p-update 3 x 8 n (r, p read; p write)
cpu_baseline: the oracle (scipy CSR SpMV + numpy dots, one core) on the same matrix.
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--grid", type=int, default=160)
    ap.add_argument("--stencil", type=int, default=27)
    ap.add_argument("--iters", type=int, default=100)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--mode", default="device", choices=["device", "host", "partial"])
    ap.add_argument("--cpu-iters", type=int, default=5)
    ap.add_argument("--lanes", type=int, default=0, help="SpMV lanes per row (4, 8, 16, 32)")
    ap.add_argument("--rows-in-flight", type=int, default=0, help="SpMV rows per lane group (1, 2, 4)")
    a = ap.parse_args()
    import numpy as np
    import torch
    import torch.distributed as dist

    import paper_conf_cluster_sagbilieinu25_b200 as U
    rank, world, local = (int(os.environ.get(v, d)) for v, d in (("RANK", 0), ("WORLD_SIZE", 1), ("LOCAL_RANK", 0)))
    if world > 1:
        dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(local)
    env = U.Env(rank, world, local, U.torch_allgather() if world > 1 else None)
    comm = U.Comm(env, *U.ring_neighbours(rank, world))
    st = torch.cuda.Stream()
    mode = {"device": U.UC_MODE_DEVICE, "host": U.UC_MODE_HOST, "partial": U.UC_MODE_PARTIAL}[a.mode]
    co = U.Coord(comm, mode, st.cuda_stream)
    g = a.grid
    t0 = time.time()
    cg = U.CG(comm, g, g, g, a.stencil)
    if a.lanes or a.rows_in_flight:
        cg.set_launch(a.lanes, a.rows_in_flight)
    setup_s = time.time() - t0
    hist = np.zeros(a.iters)
    for _ in range(a.warmup):
        cg.run(co, a.iters, True, hist)
    co.sync()
    if world > 1:
        dist.barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    for _ in range(a.steps):
        cg.run(co, a.iters, True, hist)
    e1.record(st)
    co.sync()
    ms = e0.elapsed_time(e1)
    if world > 1:
        t = torch.tensor([ms], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    it_s = a.steps * a.iters / (ms / 1e3)
    n, N, nnz = cg.n_local, cg.N, cg.nnz_local
    bytes_it = 8 * (n + 1) + 12 * nnz + 8 * n + 8 * N + 6 * 8 * n + 3 * 8 * n
    ms_it = ms / (a.steps * a.iters)
    gbs = bytes_it / (ms_it / 1e3) / 1e9
    peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"] \
        if os.path.exists(os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6650.0
    comm.barrier()
    cg.destroy()
    co.destroy()
    comm.destroy()
    env.finalize()
    cpu = None
    if rank == 0 and world == 1 and a.cpu_iters > 0:
        from inputs import cg_gen
        from oracle import cg as ocg
        A = cg_gen.matrix_scipy(g, g, g, a.stencil)
        b = cg_gen.rhs(A.shape[0])
        t = time.perf_counter()
        ocg.cg(A, b, a.cpu_iters)
        dt = time.perf_counter() - t
        cpu = {"value": round(a.cpu_iters / dt, 3), "unit": "CG iterations/s", "cores": 1, "kind": "oracle",
               "sample": f"{a.cpu_iters} iterations of the same {g}^3 {a.stencil}-point system (scipy CSR, 1 core)"}
    if rank == 0:
        print(json.dumps({
            "metric": "CG iterations/s (paper §VI-D workload, synthetic 3-D stencil SPD matrix)",
            "value": round(it_s, 1), "unit": "iterations/s", "n_gpus": world, "steps": a.steps, "warmup": a.warmup,
            "ms_per_iteration": round(ms_it, 5), "higher_is_better": True, "dtype": "f64", "data": "synthetic",
            "config": {"workload": f"cg_{g}^3_{a.stencil}pt_{a.mode}", "rows": N, "nnz_per_rank": nnz,
                       "iters_per_step": a.iters, "setup_s": round(setup_s, 1)},
            "roofline": {"bound": "hbm", "achieved": round(gbs, 1), "peak": peak, "unit": "GB/s",
                         "frac": round(gbs / peak, 4), "alg_bytes_per_iteration": bytes_it,
                         "note": "whole iteration (3 kernels + exchanges) vs copy peak"},
            "cpu_baseline": cpu, "final_rr": float(hist[-1])}))
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
