"""Full-size parity at the north-star configuration: 8 ranks x 16384^2 per rank (BASELINE.json
configs[3], weak scaling; 16384 x 131072 global), device mode, ring, the launch configuration
bench.py times -- as 8 virtual ranks on one GPU (16 GB of slabs).

The oracle cannot sweep 2.1 G points per iteration in a test, so it computes SAMPLED rows one
window at a time: after k iterations a point depends only on initial values within k rows, so
the oracle run on a window of rows [y0-k-1, y1+k+1] with its two edge rows held fixed (the
oracle's dirichlet-y mode) reproduces rows [y0, y1] exactly.  Sampled: every rank boundary
(where the NVLink halo exchange acts), the ring wrap-around, and the middle of each rank.
"""
import numpy as np
import pytest

import oracle
from gpu_harness import bits
from inputs import gen
from vranks import run_ranks

pytestmark = pytest.mark.gpu


def window_oracle(nx, ny, y0, y1, k, topology="ring"):
    """Oracle values of computed rows y0..y1 (global indices, ring-wrapped) after k iterations."""
    gys = list(range(y0 - k - 1, y1 + k + 2))
    w = gen.rows_field(nx, ny, gys, topology)
    out, _ = oracle.jacobi_run(w, k, "dirichlet")
    return out[k + 1:k + 1 + (y1 - y0 + 1)]


@pytest.mark.parametrize("variant,k,ne", [(5, 12, 6), (5, 4, 4), (4, 4, 4), (1, 4, 4)])
def test_weak_scaling_8x16384sq_sampled_rows(variant, k, ne):
    """variant 5 at k = 12, norm every 6: two launches of the shipped jacobi_t_kernel<6, 2> with 8
    distinct ranks; k = 4: one T = 4 launch."""
    import torch

    import paper_conf_cluster_sagbilieinu25_b200 as U
    P, nx, n = 8, 16384, 16384
    ny = P * n
    edge = 6  # owned rows sampled at each end of a slab, plus both halo rows

    def body(rank, P, ag):
        env = U.Env(rank, P, 0, ag)
        comm = U.Comm(env, *U.ring_neighbours(rank, P))
        st = torch.cuda.Stream()
        co = U.Coord(comm, U.UC_MODE_DEVICE, st.cuda_stream)
        co.set_timeout(30.0)
        J = U.Jacobi(comm, nx, ny)
        if variant != 5:
            J.set_launch(variant)
        try:
            comm.barrier()
            J.run(co, k, ne, use_graph=True)
            co.sync()
            counts = J.launch_counts()
            co.sync()
            top = J.copy_rows(co, 0, edge + 1)                  # halo row 0 + owned rows 1..edge
            bot = J.copy_rows(co, n + 1 - edge, edge + 1)       # owned rows n-edge+1..n + halo n+1
            mid = J.copy_rows(co, n // 2, 3)
            info = J.launch_info()
            return top, bot, mid, info, counts
        finally:
            comm.barrier()
            J.destroy()
            co.destroy()
            comm.destroy()
            env.finalize()

    res = run_ranks(P, body)
    assert res[0][3]["variant"] == variant
    if variant == 5:
        for r in range(P):
            c = res[r][4]
            assert (c[6], sum(c[:15])) == ((2, 2) if k == 12 else (0, 1)), c
    for r in range(P):
        top, bot, mid, _, _ = res[r]
        g0 = r * n  # global computed row of slab row 1
        # slab row j <-> global computed row g0 + j - 1 (ring-wrapped for the halo rows)
        want_top = window_oracle(nx, ny, g0 - 1, g0 + edge - 1, k)
        want_bot = window_oracle(nx, ny, g0 + n - edge, g0 + n, k)
        want_mid = window_oracle(nx, ny, g0 + n // 2 - 1, g0 + n // 2 + 1, k)
        for got, want, what in ((top, want_top, "top"), (bot, want_bot, "bottom"), (mid, want_mid, "middle")):
            if not np.array_equal(bits(got), bits(want)):
                d = np.argwhere(bits(got) != bits(want))
                raise AssertionError(f"rank {r} {what}: {len(d)} points differ, first {d[0]}")
