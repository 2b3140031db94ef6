"""Object lifetimes and ordering of the asynchronous copies (round-1 advisor findings).

* A coordinator's cached graphs die with it: a solver that ran graphs on coordinator A, then A is
  destroyed and B created (possibly on the same stream handle), must not replay A's graph (it
  points at A's freed error word) -- B's runs stay exact and B reports its own timeouts.
* uc_jacobi_copy_in_async is collective and ordered against the neighbours' puts: after a device
  mode run at P = 2, copy_in_async of new data followed by a run gives the oracle's result for
  the new data, on every rank (no neighbour put lands on top of the copied halo rows).
"""
import numpy as np
import pytest

from gpu_harness import assert_slabs_equal_global
from inputs import gen
from test_gpu_jacobi import _oracle
from vranks import run_ranks

pytestmark = pytest.mark.gpu


def test_graphs_do_not_outlive_their_coordinator():
    import torch

    import paper_conf_cluster_sagbilieinu25_b200 as U
    nx, ny = 1028, 48
    env = U.Env(0, 1, 0)
    comm = U.Comm(env, 0, 0)
    st = torch.cuda.Stream()
    J = U.Jacobi(comm, nx, ny)
    total = 0
    for rep in range(3):  # same stream handle every time: only the coordinator differs
        co = U.Coord(comm, U.UC_MODE_DEVICE, st.cuda_stream)
        co.set_timeout(5.0 + rep)  # a new timeout must never replay a graph built with the old one
        J.run(co, 18, 6, use_graph=True)
        co.sync()
        total += 18
        co.destroy()
    co = U.Coord(comm, U.UC_MODE_DEVICE, st.cuda_stream)
    out = J.copy_out(co)
    counts = J.launch_counts()
    J.destroy()
    co.destroy()
    comm.destroy()
    env.finalize()
    _, want, _ = _oracle(nx, ny, "ring", total, 0)
    assert_slabs_equal_global([out], want, 1, "ring")
    assert counts[6] == 9, counts


@pytest.mark.parametrize("P", [2, 3])
def test_copy_in_async_is_ordered_against_neighbour_puts(P):
    import torch

    import paper_conf_cluster_sagbilieinu25_b200 as U
    nx, n = 1028, 24
    ny = n * P
    rng = np.random.default_rng(P)
    init = rng.random((ny + 2, nx), dtype=np.float32)
    init[0], init[-1] = init[ny], init[1]

    def body(rank, P, ag):
        env = U.Env(rank, P, 0, ag)
        comm = U.Comm(env, *U.ring_neighbours(rank, P))
        st = torch.cuda.Stream()
        co = U.Coord(comm, U.UC_MODE_DEVICE, st.cuda_stream)
        co.set_timeout(10.0)
        J = U.Jacobi(comm, nx, ny)
        host = torch.empty((n + 2) * nx, dtype=torch.float32, pin_memory=True)
        host.numpy()[:] = gen.rank_slab(init, rank, P).ravel()
        outs = []
        try:
            for _ in range(3):
                J.run(co, 13, 0, use_graph=True)   # leaves puts in flight towards the neighbours
                J.copy_in_async(co, host.data_ptr())  # no sync in between: stream-ordered only
                J.run(co, 12, 6, use_graph=True)
                res = torch.empty((n + 2) * nx, dtype=torch.float32, pin_memory=True)
                J.copy_out_async(co, res.data_ptr())
                co.sync()
                outs.append(res.numpy().reshape(n + 2, nx).copy())
            return outs
        finally:
            comm.barrier()
            J.destroy()
            co.destroy()
            comm.destroy()
            env.finalize()

    res = run_ranks(P, body)
    _, want, _ = _oracle(nx, ny, "ring", 12, 6, init=init)
    for i in range(3):
        assert_slabs_equal_global([r[i] for r in res], want, P, "ring", f"repeat {i}")
