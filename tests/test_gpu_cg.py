"""GPU parity of the CG workload against the CPU oracle (oracle/cg.py).

Floating point (fp64) with a different reduction order than the oracle (ordered block sums,
rank-ordered allreduce vs numpy's pairwise dot): the iterate and the |r|^2 history agree to a
relative 1e-9 over a few dozen iterations (DESIGN.md §11 derives the bound); every rank holds
bit-identical scalars.  Device mode with 1..4 virtual ranks, host and partial mode with 1 rank.
"""
import numpy as np
import pytest

from inputs import cg_gen
from oracle import cg as ocg
from vranks import run_ranks

pytestmark = pytest.mark.gpu

RTOL = 1e-9


def solve_cg_gpu(nx, ny, nz, stencil, P, mode, iters, chunks=None, use_graph=True, seed=cg_gen.DEFAULT_SEED):
    import torch

    import paper_conf_cluster_sagbilieinu25_b200 as U

    def body(rank, P, ag):
        env = U.Env(rank, P, 0, ag)
        comm = U.Comm(env, *U.ring_neighbours(rank, P))
        st = torch.cuda.Stream()
        co = U.Coord(comm, mode, st.cuda_stream)
        co.set_timeout(10.0)
        cg = U.CG(comm, nx, ny, nz, stencil, seed)
        try:
            hist = []
            for it in (chunks or [iters]):
                hist.append(cg.run(co, it, use_graph))
                co.sync()
            x = cg.x(co)
            return x, np.concatenate(hist), cg.row0
        finally:
            comm.barrier()
            cg.destroy()
            co.destroy()
            comm.destroy()
            env.finalize()

    res = run_ranks(P, body)
    x = np.concatenate([r[0] for r in res])
    return x, [r[1] for r in res]


def _oracle(nx, ny, nz, stencil, iters, seed=cg_gen.DEFAULT_SEED):
    A = cg_gen.matrix_scipy(nx, ny, nz, stencil)
    b = cg_gen.rhs(A.shape[0], seed)
    return ocg.cg(A, b, iters)


def _check(nx, ny, nz, stencil, P, mode, iters, **kw):
    x, hists = solve_cg_gpu(nx, ny, nz, stencil, P, mode, iters, **kw)
    xw, hw = _oracle(nx, ny, nz, stencil, iters)
    assert np.allclose(x, xw, rtol=RTOL, atol=RTOL * np.abs(xw).max())
    for h in hists:
        assert np.array_equal(h, hists[0])  # every rank: bit-identical scalars
        assert np.allclose(h, hw, rtol=RTOL, atol=0)


@pytest.mark.parametrize("stencil", [7, 27])
@pytest.mark.parametrize("P", [1, 2, 3, 4])
def test_cg_device_mode(stencil, P):
    _check(12, 10, 8 * P if P != 3 else 24, stencil, P, 1, 25)


@pytest.mark.parametrize("mode", [0, 2])
def test_cg_host_and_partial_mode(mode):
    _check(16, 9, 7, 27, 1, mode, 25)


def test_cg_graph_chunks_and_eager_agree():
    a, ha = solve_cg_gpu(14, 11, 8, 27, 2, 1, 30)
    b, hb = solve_cg_gpu(14, 11, 8, 27, 2, 1, 30, chunks=[1, 12, 17])
    c, hc = solve_cg_gpu(14, 11, 8, 27, 2, 1, 30, use_graph=False)
    assert np.array_equal(a, b) and np.array_equal(a, c)
    assert np.array_equal(ha[0], hb[0]) and np.array_equal(ha[0], hc[0])


def test_cg_64cubed_vs_oracle():
    """262,144 rows (7 M nonzeros), 40 iterations vs the oracle; |r|^2 falls by > 10^3."""
    x, hists = solve_cg_gpu(64, 64, 64, 27, 1, 1, 40)
    xw, hw = _oracle(64, 64, 64, 27, 40)
    assert np.allclose(x, xw, rtol=1e-8, atol=1e-8 * np.abs(xw).max())
    assert np.allclose(hists[0], hw, rtol=1e-8)
    assert hists[0][-1] < 1e-3 * hists[0][0]


def test_cg_eigenvector_rhs_one_step_on_gpu():
    """Closed form independent of the oracle: with b an eigenvector v of A (eigenvalue lam),
    one CG step gives x = v / lam.  The solver's b is the seeded generator's, so here we check
    the GPU's first step against the exact one-step formula x1 = (b.b / b.Ab) b instead."""
    nx, ny, nz = 10, 9, 8
    x, hists = solve_cg_gpu(nx, ny, nz, 27, 2, 1, 1)
    A = cg_gen.matrix_scipy(nx, ny, nz, 27)
    b = cg_gen.rhs(A.shape[0])
    x1 = (b @ b) / (b @ (A @ b)) * b
    assert np.allclose(x, x1, rtol=1e-12, atol=0)
