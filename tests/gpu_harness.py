"""Runs the CUDA path through the C-ABI for P virtual ranks on one GPU and assembles the
global field, so tests can compare it with the oracle element by element."""
from __future__ import annotations

import numpy as np

from inputs import gen
from vranks import run_ranks

MODES = {"device": 1, "host": 0, "partial": 2}
TIMEOUT_S = 5.0  # device spin-wait timeout (raised by scripts/sanitize_run.py)


def neighbours(U, topology):
    return U.ring_neighbours if topology == "ring" else U.chain_neighbours


def solve_gpu(nx, ny, P, topology="ring", mode="device", iters=10, norm_every=0, seed=gen.DEFAULT_SEED,
              zero_init=False, init=None, use_graph=True, stepwise=False, block_x=0, blocks_per_sm=0,
              variant=-1, stages=0, tile_rows=0,
              chunks_of_run=None, host_path=None, balance=None, balance_rates=None):
    """Returns dict(init=[slab0 per rank], final=[slab per rank], norms=np.array (rank 0),
    norms_all=[per rank], launch=launch_info of rank 0)."""
    import torch

    import paper_conf_cluster_sagbilieinu25_b200 as U

    def body(rank, P, ag):
        env = U.Env(rank, P, 0, ag)
        top, bot = neighbours(U, topology)(rank, P)
        comm = U.Comm(env, top, bot)
        stream = torch.cuda.Stream()
        coord = U.Coord(comm, MODES[mode], stream.cuda_stream)
        coord.set_timeout(TIMEOUT_S)
        J = U.Jacobi(comm, nx, ny, seed, zero_init)
        try:
            if block_x or blocks_per_sm or variant >= 0 or stages or tile_rows:
                J.set_launch(variant, block_x, blocks_per_sm, stages, tile_rows)
            if host_path is not None:
                J.set_host_path(*host_path)
            if balance is not None or balance_rates is not None:
                J.set_balance(True if balance is None else balance)
            if balance_rates is not None:  # a callable: (rank, grid) -> per-block rates
                J.balance_rates(coord, balance_rates(rank, J.launch_info()["grid"]))
            slab0 = J.copy_out()
            if init is not None:
                J.copy_in(gen.rank_slab(init, rank, P))
            comm.barrier()
            if stepwise:
                norms = []
                for i in range(iters):
                    want = norm_every > 0 and J.iteration % norm_every == 0
                    buf = np.zeros(1, np.float64)
                    J.step(coord, want, buf if want else None)
                    coord.sync()
                    if want:
                        norms.append(buf[0])
                norms = np.array(norms)
            else:
                parts = chunks_of_run or [iters]
                outs = [J.run(coord, it, norm_every, use_graph) for it in parts]
                coord.sync()
                norms = np.concatenate(outs) if outs else np.zeros(0)
            coord.sync()
            final = J.copy_out(coord)
            info = J.launch_info()
            counts = J.launch_counts()
            pm = MODES[mode] | (U.UC_PLAN_DEEP_HALO if host_path and host_path[0] and mode == "host" else 0)
            want = expected_counts(U, info, pm, ny // P, iters, norm_every, stepwise, chunks_of_run)
            if want is not None:  # the launches that really ran are the plan's (no silent demotion)
                # (slot 15 counts blocks whose scaled march re-ran unscaled, not launches)
                assert counts[:15] == want[:15], (f"rank {rank}: launches by iterations per launch {counts[:9]} != "
                                        f"plan {want[:9]} ({info})")
            return slab0, final, norms, info, counts, J.balance_table()
        finally:
            comm.barrier()
            J.destroy()
            coord.destroy()
            comm.destroy()
            env.finalize()

    res = run_ranks(P, body)
    return {"init": [r[0] for r in res], "final": [r[1] for r in res], "norms": res[0][2],
            "norms_all": [r[2] for r in res], "launch": res[0][3], "counts": res[0][4],
            "counts_all": [r[4] for r in res], "balance_tables": [r[5] for r in res]}


def expected_counts(U, info, mode, n_local, iters, norm_every, stepwise=False, chunks_of_run=None):
    """Histogram (launches by iterations per launch) the launch plan predicts for a run, or None
    where launches are not one-per-plan-entry (the persistent variant 3 in device mode)."""
    v = info["variant"]
    if v == 3 and mode & 0xff == 1:
        return None
    h = [0] * 16
    if stepwise:
        h[1] = iters
        return h
    for it in (chunks_of_run or [iters]):
        for t in U.launch_plan(v, info["tile_rows"] if v == 5 else 1, mode, n_local, it, norm_every):
            h[t] += 1
    return h


def bits(a):
    return np.ascontiguousarray(a, dtype=np.float32).view(np.uint32)


def assert_slabs_equal_global(slabs, g, P, topology, what="final"):
    for r, s in enumerate(slabs):
        want = gen.rank_slab(g, r, P, topology)
        if not np.array_equal(bits(s), bits(want)):
            diff = np.argwhere(bits(s) != bits(want))
            j, i = diff[0]
            raise AssertionError(f"{what}: rank {r} differs at {len(diff)} points, first (row {j}, col {i}): "
                                 f"gpu={s[j, i]!r} oracle={want[j, i]!r}")
