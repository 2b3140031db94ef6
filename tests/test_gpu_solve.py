"""CPU-free convergence loop (uc_jacobi_solve): the device decides when to stop.

The run must stop after the same period as the oracle's first norm below the tolerance (norms
taken on each period's first iteration, k % norm_every == 0), with the grid bit-exact after that
many iterations -- at one rank and across virtual ranks (every rank stops after the same period
because every rank holds the same norms)."""
import numpy as np
import pytest

import oracle
from gpu_harness import assert_slabs_equal_global
from inputs import gen
from vranks import run_ranks

pytestmark = pytest.mark.gpu


def _expected(nx, ny, topology, ne, tol, max_iters):
    g = gen.global_field(nx, ny, topology)
    _, sums = oracle.jacobi_run(g, max_iters, topology, ne)
    norms = np.sqrt(sums)
    below = np.nonzero(norms < tol)[0]
    periods = int(below[0]) + 1 if below.size else max_iters // ne
    want, _ = oracle.jacobi_run(g, periods * ne, topology, ne)
    return periods * ne, want, norms[periods - 1]


def _solve(nx, ny, P, topology, ne, tol, max_iters, k0=0):
    import torch

    import paper_conf_cluster_sagbilieinu25_b200 as U

    def body(rank, P, ag):
        env = U.Env(rank, P, 0, ag)
        nb = U.ring_neighbours if topology == "ring" else U.chain_neighbours
        comm = U.Comm(env, *nb(rank, P))
        st = torch.cuda.Stream()
        co = U.Coord(comm, U.UC_MODE_DEVICE, st.cuda_stream)
        co.set_timeout(10.0)
        J = U.Jacobi(comm, nx, ny)
        try:
            if k0:
                J.run(co, k0, ne)
                co.sync()
            it, nrm = J.solve(co, max_iters, ne, tol)
            out = J.copy_out(co)
            return it, nrm, out, J.iteration
        finally:
            comm.barrier()
            J.destroy()
            co.destroy()
            comm.destroy()
            env.finalize()

    return run_ranks(P, body)


@pytest.mark.parametrize("P,topology", [(1, "ring"), (1, "dirichlet"), (3, "ring"), (2, "dirichlet")])
@pytest.mark.parametrize("ne,tol", [(10, 0.3), (12, 0.05), (6, 1e-9)])
def test_solve_stops_where_the_oracle_does(P, topology, ne, tol):
    nx, ny, max_iters = 260, 48 * P, 240
    want_it, want, want_norm = _expected(nx, ny, topology, ne, tol, max_iters)
    res = _solve(nx, ny, P, topology, ne, tol, max_iters)
    for it, nrm, _, k in res:
        assert it == want_it and k == want_it, (it, want_it)
        assert abs(nrm - want_norm) <= 1e-5 * want_norm, (nrm, want_norm)
    assert_slabs_equal_global([r[2] for r in res], want, P, topology)


def test_solve_after_a_run_and_max_iters_cap():
    """Starts at k0 = 24 (a multiple of norm_every); tol = 0 never converges: max_iters caps."""
    nx, ny, ne = 260, 64, 8
    res = _solve(nx, ny, 2, "ring", ne, 0.0, 64, k0=24)
    g = gen.global_field(nx, ny, "ring")
    want, _ = oracle.jacobi_run(g, 24 + 64, "ring", ne)
    for it, _, _, k in res:
        assert it == 64 and k == 88
    assert_slabs_equal_global([r[2] for r in res], want, 2, "ring")
