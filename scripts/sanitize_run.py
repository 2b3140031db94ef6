"""Small end-to-end runs of every kernel variant and launch mode, for compute-sanitizer:

    compute-sanitizer --tool memcheck|racecheck|synccheck|initcheck python scripts/sanitize_run.py

Checks each result against the oracle as well (bit-exact grid).  Sizes are tiny because the
tools slow kernels down by orders of magnitude; spin-wait timeouts are raised accordingly.
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import numpy as np  # noqa: E402

import oracle  # noqa: E402
from gpu_harness import assert_slabs_equal_global, solve_gpu  # noqa: E402
from inputs import gen  # noqa: E402

import gpu_harness  # noqa: E402


def main():
    cases = [
        dict(P=1, mode="device", variant=1), dict(P=1, mode="device", variant=0), dict(P=1, mode="device", variant=2),
        dict(P=1, mode="device", variant=3), dict(P=1, mode="host", variant=1), dict(P=1, mode="partial", variant=1),
        dict(P=2, mode="device", variant=1), dict(P=2, mode="device", variant=3),
        dict(P=1, mode="device", variant=4), dict(P=2, mode="device", variant=4),
        dict(P=1, mode="device", variant=5, T=4, ne=4), dict(P=2, mode="device", variant=5, T=4, ne=4),
        dict(P=2, mode="device", variant=5, T=3, ne=3), dict(P=1, mode="device", variant=5, T=2, ne=2),
        dict(P=1, mode="host", variant=5, T=4), dict(P=1, mode="partial", variant=5, T=4),
    ]
    # the shipped default, jacobi_t_kernel<6, 2> (two ghost lanes, five h-row levels), at P = 1
    # (self-exchange), P = 2 (top == bottom) and P = 3 (distinct peers); ne = 6 keeps every launch
    # at T = 6 (a norm cadence below T demotes launches)
    t6 = [dict(P=1, mode="device", variant=5, T=6, ne=6, iters=13), dict(P=2, mode="device", variant=5, T=6, ne=0, iters=12),
          dict(P=3, mode="device", variant=5, T=6, ne=6, iters=12),
          dict(P=1, mode="device", variant=5, T=8, ne=8, iters=17), dict(P=2, mode="device", variant=5, T=8, ne=0, iters=16),
          dict(P=3, mode="device", variant=5, T=8, ne=8, iters=16)]
    # round 2: the pair-frame march and the scaled march run in warps without a fixed column, so
    # rows wide enough for interior warps (nx = 1028: 257 float4 columns, 2 strips); norm-free
    # launches (scaled) and a forced balanced-chunk table
    t6 += [dict(P=1, mode="device", variant=5, T=8, ne=0, iters=16, nx=1028, ny=64),
           dict(P=2, mode="device", variant=5, T=8, ne=0, iters=24, nx=1028, ny=64, balance=True),
           dict(P=3, mode="device", variant=5, T=6, ne=0, iters=12, nx=1028, ny=64)]
    if os.environ.get("UC_SANITIZE_T6_ONLY"):
        cases = t6
    else:
        cases += t6
    if len(sys.argv) > 1:
        cases = cases[: int(sys.argv[1])]
    for c in cases:
        P = c["P"]
        nx, ny = c.get("nx", 132), c.get("ny", 24)
        iters = c.get("iters", 9)
        ne = c.get("ne", 2)
        extra = {}
        if c.get("balance"):
            extra["balance_rates"] = lambda rank, grid: [1.0 + 0.5 * ((b * 7 + rank) % 5) for b in range(grid)]
        res = solve_gpu(nx, ny * P, P, "ring", c["mode"], iters, ne if c["mode"] != "partial" or P == 1 else 0,
                        variant=c["variant"], tile_rows=c.get("T", 0), use_graph=False, **extra)
        want, _ = oracle.jacobi_run(gen.global_field(nx, ny * P, "ring"), iters, "ring")
        assert_slabs_equal_global(res["final"], want, P, "ring")
        if c["variant"] == 5 and c.get("T", 0) in (6, 8):
            import paper_conf_cluster_sagbilieinu25_b200 as U
            plan = U.launch_plan(5, c["T"], 1, ny, iters, ne)  # ny = rows per rank
            assert plan[0] == c["T"], plan
        print("ok", c, flush=True)
    print("SANITIZE_RUN_DONE")


if __name__ == "__main__":
    gpu_harness.TIMEOUT_S = 300.0
    main()
