"""GPU parity of kernel variant 4 (two Jacobi iterations per launch, temporal blocking of depth 2)
against the CPU oracle.

Variant 4 computes A_{k+1} in registers and stores only A_{k+2}; the boundary rows of BOTH
iterations are still exchanged with the neighbours (prologue puts of A_{k+1} rows through the
h1 buffers, deferred puts of A_{k+2} rows into the halo rows).  The bar is the same as for the
one-iteration kernel (BASELINE.json north_star): the grid bit-exact after N iterations, norms
within 1e-5.  Odd iteration counts end with one one-iteration launch; norm_every == 1 and n == 1
run one-iteration launches throughout; every mixture must stay bit-exact.
"""
import numpy as np
import pytest

from gpu_harness import assert_slabs_equal_global, bits, solve_gpu
from test_gpu_jacobi import NORM_RTOL, _check, _oracle

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("topology", ["ring", "dirichlet"])
@pytest.mark.parametrize("iters,ne", [(100, 10), (101, 10), (100, 0), (37, 3)])
def test_c1_256(topology, iters, ne):
    """configs[0] (256^2, 100 iterations, 1 GPU) and odd/even counts, norms at both levels."""
    res = _check(256, 256, 1, topology, "device", iters, norm_every=ne, variant=4)
    assert res["launch"]["variant"] == 4


@pytest.mark.parametrize("nx,ny,iters", [(4, 2, 4), (8, 7, 20), (12, 5, 9), (1028, 64, 38), (2052, 33, 12),
                                         (4096, 40, 8), (36, 3, 6), (40, 4, 10)])
@pytest.mark.parametrize("topology", ["ring", "dirichlet"])
def test_shapes_single_rank(nx, ny, iters, topology):
    """Ragged last strip, tiny grids, n = 2..4 (one row chunk), odd row counts."""
    _check(nx, ny, 1, topology, "device", iters, norm_every=4, variant=4)


@pytest.mark.parametrize("P", [2, 3, 4, 8])
@pytest.mark.parametrize("topology", ["ring", "dirichlet"])
@pytest.mark.parametrize("ne", [5, 4])
def test_partition_invariance(P, topology, ne):
    """Virtual ranks P = 2..8: A_{k+1} rows cross ranks through the h1 buffers, A_{k+2} rows
    through the halo rows; norm rounds on the first (ne = 4) or second (ne = 5, odd k) level."""
    _check(520, 24 * P, P, topology, "device", 26, norm_every=ne, variant=4)


@pytest.mark.parametrize("P,ny", [(2, 2), (4, 4), (3, 3), (2, 4), (2, 6), (4, 16)])
def test_few_rows_per_rank(P, ny):
    """n = 1 (one-iteration launches), n = 2 and 3 (one row chunk does both sides), n = 4."""
    for topology in ("ring", "dirichlet"):
        _check(64, ny, P, topology, "device", 12, norm_every=2, variant=4)


@pytest.mark.parametrize("block_x,bps,stages", [(32, 1, 3), (64, 2, 4), (128, 0, 2), (256, 1, 8)])
def test_launch_geometries(block_x, bps, stages):
    """Strip width (cross-strip halo columns of A_{k+1}), chunk count and ring depth change the
    blocking, not the results; 4 ranks so strips meet rank boundaries."""
    res = _check(1028, 96, 4, "ring", "device", 10, norm_every=3, block_x=block_x, blocks_per_sm=bps,
                 variant=4, stages=stages)
    assert res["launch"]["variant"] == 4


def test_random_values_everywhere():
    """Random data in every cell, including both fixed columns, ragged strips."""
    nx, ny = 1028, 24
    rng = np.random.default_rng(7)
    init = rng.random((ny + 2, nx), dtype=np.float32)
    init[0], init[-1] = init[ny], init[1]
    _check(nx, ny, 1, "ring", "device", 14, norm_every=2, init=init, variant=4)
    _check(nx, ny, 3, "ring", "device", 14, norm_every=2, init=init, variant=4)
    _check(nx, ny, 2, "dirichlet", "device", 14, norm_every=2, init=init, variant=4)


def test_graph_eager_stepwise_chunked_agree():
    """CUDA graph, eager launches, single steps and runs of odd lengths (two-iteration launches
    followed by one-iteration launches, parity offset flipping) give identical grids and norms."""
    kw = dict(variant=4)
    a = solve_gpu(516, 64, 2, "ring", "device", 30, 7, use_graph=True, **kw)
    b = solve_gpu(516, 64, 2, "ring", "device", 30, 7, use_graph=False, **kw)
    c = solve_gpu(516, 64, 2, "ring", "device", 30, 1, stepwise=True, **kw)
    d = solve_gpu(516, 64, 2, "ring", "device", 30, 7, chunks_of_run=[3, 11, 16], **kw)
    e = solve_gpu(516, 64, 2, "ring", "device", 30, 7, chunks_of_run=[5, 5, 5, 15], use_graph=False, **kw)
    for x in (b, c, d, e):
        for s1, s2 in zip(a["final"], x["final"]):
            assert np.array_equal(bits(s1), bits(s2))
    assert np.array_equal(a["norms"], b["norms"]) and np.array_equal(a["norms"], d["norms"])
    assert np.array_equal(a["norms"], e["norms"])
    assert np.array_equal(a["norms"], c["norms"][[0, 7, 14, 21, 28]])
    _, want, want_norms = _oracle(516, 64, "ring", 30, 7)
    assert_slabs_equal_global(a["final"], want, 2, "ring")
    assert np.allclose(a["norms"], want_norms, rtol=NORM_RTOL, atol=0)


def test_norm_every_iteration_falls_back_to_single_steps():
    _check(1028, 48, 2, "ring", "device", 9, norm_every=1, variant=4)


def test_switch_variants_and_modes_mid_run():
    """Variant 4 -> variant 1 -> variant 4 (odd counts, so the parity offset is 1 at each switch),
    then a host-mode and a partial-mode run on the same solver (P = 1)."""
    import torch

    import paper_conf_cluster_sagbilieinu25_b200 as U
    from vranks import run_ranks
    nx, ny, P = 1028, 48, 2

    def body(rank, P, ag):
        env = U.Env(rank, P, 0, ag)
        comm = U.Comm(env, *U.ring_neighbours(rank, P))
        st = torch.cuda.Stream()
        coord = U.Coord(comm, U.UC_MODE_DEVICE, st.cuda_stream)
        coord.set_timeout(5.0)
        J = U.Jacobi(comm, nx, ny)
        J.set_launch(4)
        n1 = J.run(coord, 6, 5)   # 3 two-iteration launches: parity offset 1
        coord.sync()
        J.set_launch(1, 64, 0, 5)
        n2 = J.run(coord, 7, 5)
        coord.sync()
        J.set_launch(4, 128)
        n3 = J.run(coord, 9, 5)
        coord.sync()
        out = J.copy_out(coord)
        comm.barrier()
        J.destroy()
        coord.destroy()
        comm.destroy()
        env.finalize()
        return out, np.concatenate([n1, n2, n3])

    res = run_ranks(P, body)
    _, want, want_norms = _oracle(nx, ny, "ring", 22, 5)
    assert_slabs_equal_global([r[0] for r in res], want, P, "ring")
    assert np.allclose(res[0][1], want_norms, rtol=NORM_RTOL, atol=0)

    env = U.Env(0, 1, 0)
    comm = U.Comm(env, 0, 0)
    st = torch.cuda.Stream()
    coords = {m: U.Coord(comm, v, st.cuda_stream) for m, v in (("device", 1), ("host", 0), ("partial", 2))}
    J = U.Jacobi(comm, nx, ny)
    J.set_launch(4)
    for m, it in (("device", 6), ("host", 5), ("device", 4), ("partial", 3), ("device", 7), ("host", 2)):
        J.run(coords[m], it, 0)
        coords[m].sync()
    out = J.copy_out(coords["device"])
    J.destroy()
    for c in coords.values():
        c.destroy()
    comm.destroy()
    env.finalize()
    _, want, _ = _oracle(nx, ny, "ring", 27, 0)
    assert_slabs_equal_global([out], want, 1, "ring")


def test_hand_worked_4x4(golden_dir):
    """The pinned 4x4 example (dirichlet-y, NX = 4, NY = 2): 3 iterations = one two-iteration
    launch + one single; exact dyadic values and norms."""
    import math
    rows = [l.split()[1:] for l in open(f"{golden_dir}/hand4x4.txt") if l.startswith("init")]
    g = np.array(rows, dtype=np.float32)
    for P in (1, 2):
        res = solve_gpu(4, 2, P, "dirichlet", "device", 3, 2, init=g, variant=4)
        got = np.vstack([s[1:-1] for s in res["final"]])
        assert np.array_equal(got[:, 1:3], np.array([[4.53125, 6.25], [8.75, 13.28125]], np.float32))
        assert list(res["norms"]) == [math.sqrt(132.8125), math.sqrt(5.712890625)]


def test_subnormal_front_no_ftz():
    nx, ny = 96, 4
    a = np.zeros((ny + 2, nx), np.float32)
    a[:, 0] = 1.0
    for k in (64, 70, 74, 75):
        res = solve_gpu(nx, ny, 2, "ring", "device", k, 0, init=a, variant=4)
        s = res["final"][0]
        want = np.float32(2.0 ** (-2 * k)) if k <= 74 else np.float32(0.0)
        assert s[1, k] == want and s[1, k + 1] == 0.0
