"""GPU parity of the Jacobi hot path (C-ABI -> sm_100a kernels) against the CPU oracle.

Bar (BASELINE.json north_star): the fp32 grid bit-exact after N iterations; the norm within
1e-5 relative (reduction order differs; reading G12).  Multi-rank cases run as virtual ranks
(threads, one GPU): the device-mode put/signal protocol runs for real, peers in one process.
"""
import math

import numpy as np
import pytest

import oracle
from gpu_harness import assert_slabs_equal_global, bits, solve_gpu
from inputs import gen

pytestmark = pytest.mark.gpu

NORM_RTOL = 1e-5


def _oracle(nx, ny, topology, iters, norm_every, seed=gen.DEFAULT_SEED, zero_init=False, init=None):
    g = init if init is not None else gen.global_field(nx, ny, topology, seed, zero_init)
    out, sums = oracle.jacobi_run(g, iters, topology, norm_every)
    return g, out, np.sqrt(sums)


def _check(nx, ny, P, topology, mode, iters, norm_every=0, **kw):
    init = kw.pop("init", None)
    g0, want, want_norms = _oracle(nx, ny, topology, iters, norm_every, kw.get("seed", gen.DEFAULT_SEED),
                                   kw.get("zero_init", False), init)
    res = solve_gpu(nx, ny, P, topology, mode, iters, norm_every, init=init, **kw)
    if init is None:
        assert_slabs_equal_global(res["init"], g0, P, topology, "iteration 0 (generator parity)")
    assert_slabs_equal_global(res["final"], want, P, topology)
    assert len(res["norms"]) == len(want_norms)
    for r_norms in res["norms_all"]:  # every rank holds the same norms, bit for bit
        assert np.array_equal(r_norms, res["norms"])
    for a, b in zip(res["norms"], want_norms):
        assert a == b or abs(a - b) <= NORM_RTOL * abs(b), (a, b)
    return res


# --------------------------------------------------------------------------- C1 and shapes
@pytest.mark.parametrize("topology", ["ring", "dirichlet"])
@pytest.mark.parametrize("mode", ["device", "host"])
def test_c1_256_100_iterations(topology, mode):
    """BASELINE.json configs[0]: 256x256 fp32, 100 iterations, 1 GPU vs the oracle, bit-exact."""
    _check(256, 256, 1, topology, mode, 100, norm_every=10)


@pytest.mark.parametrize("nx,ny,iters", [(4, 2, 3), (8, 7, 20), (12, 5, 9), (1028, 64, 37), (2052, 33, 12),
                                         (4096, 40, 8)])
@pytest.mark.parametrize("topology", ["ring", "dirichlet"])
def test_ragged_shapes_single_rank(nx, ny, iters, topology):
    """Several strips with a ragged last strip (NX/4 not a multiple of the block), tiny grids,
    odd row counts."""
    _check(nx, ny, 1, topology, "device", iters, norm_every=4)


@pytest.mark.parametrize("nx", [1028, 4, 36])
def test_ragged_random_boundaries(nx):
    """Random values everywhere, including both fixed columns, with a ragged last strip: lanes
    past the row end must neither write nor enter the norm."""
    ny = 12
    rng = np.random.default_rng(nx)
    init = rng.random((ny + 2, nx), dtype=np.float32)
    init[0], init[-1] = init[ny], init[1]  # ring halos
    _check(nx, ny, 1, "ring", "device", 7, norm_every=2, init=init)
    _check(nx, ny, 2, "dirichlet", "device", 7, norm_every=2, init=init)


@pytest.mark.parametrize("P", [2, 3, 4, 8])
@pytest.mark.parametrize("topology", ["ring", "dirichlet"])
@pytest.mark.parametrize("variant", [1, 4])
def test_partition_invariance_device_mode(P, topology, variant):
    """Virtual ranks: P = 2..8 give the oracle's global grid bit for bit (invariant 6)."""
    _check(520, 24 * P, P, topology, "device", 25, norm_every=5, variant=variant)


@pytest.mark.parametrize("P,ny", [(2, 2), (4, 4), (3, 3), (2, 4)])
def test_one_or_two_rows_per_rank(P, ny):
    """n = 1 (one row does both boundary sides) and n = 2; P = 2 has top == bottom."""
    for topology in ("ring", "dirichlet"):
        _check(64, ny, P, topology, "device", 11, norm_every=2)


def test_host_mode_single_rank_nccl_self_exchange():
    _check(1028, 50, 1, "ring", "host", 13, norm_every=3)


@pytest.mark.parametrize("variant", [0, 1, 2])
@pytest.mark.parametrize("topology", ["ring", "dirichlet"])
def test_partial_device_mode(variant, topology):
    """PartialDevice (Listing 6): in-kernel posts without signals + stream-ordered
    Acknowledge.  P = 1 with norms (NCCL allreduce, single rank); P = 2..4 virtual ranks
    without norms (two NCCL ranks cannot share one GPU)."""
    _check(1028, 48, 1, topology, "partial", 17, norm_every=4, variant=variant)
    for P in (2, 3, 4):
        _check(1028, 48, P, topology, "partial", 17, norm_every=0, variant=variant)


def test_modes_interchangeable_on_one_solver():
    """Device, partial and (P = 1) host iterations can follow each other on one solver."""
    import torch

    import paper_conf_cluster_sagbilieinu25_b200 as U
    nx, ny = 520, 40
    env = U.Env(0, 1, 0)
    comm = U.Comm(env, 0, 0)
    st = torch.cuda.Stream()
    coords = {m: U.Coord(comm, MODES_[m], st.cuda_stream) for m in ("device", "partial", "host")}
    J = U.Jacobi(comm, nx, ny)
    for m in ("device", "partial", "host", "device", "partial"):
        J.run(coords[m], 5, 0)
        coords[m].sync()
    out = J.copy_out(coords["device"])
    J.destroy()
    for c in coords.values():
        c.destroy()
    comm.destroy()
    env.finalize()
    _, want, _ = _oracle(nx, ny, "ring", 25, 0)
    assert np.array_equal(bits(out), bits(gen.rank_slab(want, 0, 1)))


MODES_ = {"device": 1, "host": 0, "partial": 2}


def test_graph_and_stepwise_agree():
    a = solve_gpu(516, 64, 2, "ring", "device", 30, 7, use_graph=True)
    b = solve_gpu(516, 64, 2, "ring", "device", 30, 7, use_graph=False)
    c = solve_gpu(516, 64, 2, "ring", "device", 30, 1, stepwise=True)
    d = solve_gpu(516, 64, 2, "ring", "device", 30, 7, chunks_of_run=[3, 11, 16])
    for x in (b, c, d):
        for s1, s2 in zip(a["final"], x["final"]):
            assert np.array_equal(bits(s1), bits(s2))
    assert np.array_equal(a["norms"], b["norms"]) and np.array_equal(a["norms"], d["norms"])
    assert np.array_equal(a["norms"], c["norms"][[0, 7, 14, 21, 28]])


@pytest.mark.parametrize("variant", [0, 1, 2])
@pytest.mark.parametrize("block_x,bps,stages,tile", [(32, 1, 3, 5), (64, 2, 4, 1), (128, 0, 0, 0), (256, 1, 16, 33)])
def test_launch_geometries(variant, block_x, bps, stages, tile):
    """All kernel variants, different block widths / chunk counts / ring depths / tile heights
    change the blocking, not the results."""
    res = _check(1024, 96, 1, "ring", "device", 9, norm_every=3, block_x=block_x, blocks_per_sm=bps,
                 variant=variant, stages=stages, tile_rows=tile)
    assert res["launch"]["block"] == block_x + (32 if variant >= 1 else 0)
    assert res["launch"]["variant"] == variant


@pytest.mark.parametrize("variant", [1, 2])
@pytest.mark.parametrize("topology", ["ring", "dirichlet"])
@pytest.mark.parametrize("mode", ["device", "host"])
def test_staged_variants_c1(variant, topology, mode):
    _check(256, 256, 1, topology, mode, 100, norm_every=10, variant=variant)


@pytest.mark.parametrize("variant,tile", [(1, 0), (2, 0), (2, 3)])
@pytest.mark.parametrize("nx,ny,P", [(1028, 64, 1), (4, 2, 1), (2052, 33, 1), (520, 96, 4), (64, 3, 3),
                                     (36, 16, 8)])
def test_staged_variants_shapes(nx, ny, P, variant, tile):
    for topology in ("ring", "dirichlet"):
        _check(nx, ny, P, topology, "device", 13, norm_every=4, variant=variant, tile_rows=tile)


@pytest.mark.parametrize("P,topology,ne", [(1, "ring", 3), (1, "dirichlet", 1), (2, "ring", 5), (3, "dirichlet", 4),
                                           (4, "ring", 0), (8, "ring", 7)])
def test_persistent_variant(P, topology, ne):
    """Variant 3: one launch runs all iterations, blocks synchronise with their 4 neighbours,
    norm rounds use a grid barrier; virtual ranks share the GPU (grid sized for co-residency)."""
    res = _check(1028, 48 * P, P, topology, "device", 23, norm_every=ne, variant=3, chunks_of_run=[1, 9, 13])
    assert res["launch"]["variant"] == 3


def test_persistent_variant_stepwise_and_modes():
    _check(1028, 64, 2, "ring", "device", 6, norm_every=2, variant=3, stepwise=True)
    _check(1028, 64, 1, "ring", "host", 9, norm_every=2, variant=3)
    _check(1028, 64, 1, "ring", "partial", 9, norm_every=2, variant=3)


@pytest.mark.parametrize("variant", [0, 1, 2, 3, 4])
def test_full_size_each_variant(variant):
    """16384^2, device mode, 3 iterations, whole grid bit-exact for every kernel variant."""
    _check(16384, 16384, 1, "ring", "device", 3, norm_every=1, variant=variant)


def test_switch_variant_mid_run():
    """set_launch between runs (new strip layout, re-armed halo flags) keeps the iteration
    bit-exact: 7 iterations of variant 0 (256-wide strips), 13 of variant 1 (64-wide strips)."""
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
        n1 = J.run(coord, 7, 5)
        coord.sync()
        J.set_launch(1, 64, 0, 5)
        n2 = J.run(coord, 13, 5)
        coord.sync()
        out = J.copy_out(coord)
        comm.barrier()
        J.destroy()
        coord.destroy()
        comm.destroy()
        env.finalize()
        return out, np.concatenate([n1, n2])

    res = run_ranks(P, body)
    _, want, want_norms = _oracle(nx, ny, "ring", 20, 5)
    assert_slabs_equal_global([r[0] for r in res], want, P, "ring")
    assert np.allclose(res[0][1], want_norms, rtol=NORM_RTOL, atol=0)


# --------------------------------------------------------------------------- pinned examples
def _hand4x4(golden_dir):
    rows = [l.split()[1:] for l in open(f"{golden_dir}/hand4x4.txt") if l.startswith("init")]
    return np.array(rows, dtype=np.float32)


@pytest.mark.parametrize("P,mode", [(1, "device"), (2, "device"), (1, "host")])
def test_hand_worked_4x4(golden_dir, P, mode):
    g = _hand4x4(golden_dir)
    res = solve_gpu(4, 2, P, "dirichlet", mode, 3, 1, init=g)
    got = np.vstack([s[1:-1] for s in res["final"]])
    assert np.array_equal(got[:, 1:3], np.array([[4.53125, 6.25], [8.75, 13.28125]], np.float32))
    want = [math.sqrt(132.8125), math.sqrt(22.8515625), math.sqrt(5.712890625)]
    assert list(res["norms"]) == want  # dyadic sums: exact in any order


def test_subnormal_front_no_ftz():
    """4^-k front reaches subnormals (2^-128 .. 2^-148) bit-exactly: no FTZ on the GPU."""
    nx, ny = 96, 4
    a = np.zeros((ny + 2, nx), np.float32)
    a[:, 0] = 1.0
    for k in (64, 70, 74, 75):
        res = solve_gpu(nx, ny, 2, "ring", "device", k, 0, init=a)
        s = res["final"][0]
        want = np.float32(2.0 ** (-2 * k)) if k <= 74 else np.float32(0.0)
        assert s[1, k] == want and s[1, k + 1] == 0.0


def test_zero_init_unit_boundary_subnormals_match_oracle():
    a = np.zeros((4 + 2, 160), np.float32)
    a[:, 0] = 1.0
    a[2:4, 0] = 0.5
    _check(160, 4, 1, "ring", "device", 90, norm_every=10, init=a)


def test_constant_field_fixed_and_zero_norm():
    a = np.full((34, 64), 0.7, np.float32)
    res = solve_gpu(64, 32, 4, "ring", "device", 5, 1, init=a)
    for s in res["final"]:
        assert np.array_equal(bits(s), bits(np.full_like(s, 0.7)))
    assert not res["norms"].any()


# --------------------------------------------------------------------------- full size
def test_full_size_16384_single_gpu_bench_configuration():
    """BASELINE.json configs[2]/[3] at P = 1 (16384^2 fp32, 1 GiB per slab), in the launch
    configuration bench.py times (device mode, ring, CUDA graph, default geometry = variant 5,
    eight iterations per launch with two ghost lanes, 9-row ring): the whole grid bit-exact vs the
    oracle after 16 (two launches of 8, a norm on each), 14 (a norm cadence of 7 demotes to 7)
    and 25 iterations (8, 8, then the remainder split: 5, 4), norms within 1e-5 on every level."""
    res = _check(16384, 16384, 1, "ring", "device", 16, norm_every=8)
    assert res["launch"]["variant"] == 5 and res["launch"]["stages"] == 9 and res["launch"]["tile_rows"] == 8
    assert res["launch"]["block"] == 256 and res["counts"][8] == 2
    _check(16384, 16384, 1, "ring", "device", 14, norm_every=7)
    res = _check(16384, 16384, 1, "ring", "device", 25, norm_every=0)
    assert res["counts"][8] == 2 and res["counts"][5] == 1 and res["counts"][4] == 1


def test_full_size_host_mode():
    _check(16384, 16384, 1, "ring", "host", 2, norm_every=1)


@pytest.mark.parametrize("variant", [1, 4])
def test_config1_4096_2ranks_1000_iterations(variant):
    """BASELINE.json configs[1]: 4096 x 4096, 1000 iterations, row-split over 2 ranks, device
    put-signal (virtual ranks on one GPU), norm every 100: whole grid bit-exact."""
    _check(4096, 4096, 2, "ring", "device", 1000, norm_every=100, variant=variant)


@pytest.mark.parametrize("variant", [1, 4])
def test_config2_strong_16384_over_8_ranks(variant):
    """BASELINE.json configs[2] at P = 8 (2048 rows per rank), norm allreduce every other
    iteration here (every 100 in the benchmark): whole grid bit-exact after 4 iterations."""
    _check(16384, 16384, 8, "ring", "device", 4, norm_every=2, variant=variant)


@pytest.mark.parametrize("variant", [1, 4])
def test_config3_weak_16384_per_rank_2_ranks(variant):
    """BASELINE.json configs[3] at P = 2: 16384 x 32768 global, 16384 x 16384 per rank."""
    _check(16384, 32768, 2, "ring", "device", 4, norm_every=3, variant=variant)


def test_pageable_norm_outputs_virtual_ranks():
    """Norm outputs in pageable numpy memory (staged through page-locked memory and a stream host
    function, so the copy never blocks a virtual rank's thread): stepwise and run() paths agree
    with the pinned ones bit for bit."""
    import torch

    import paper_conf_cluster_sagbilieinu25_b200 as U
    from vranks import run_ranks
    nx, ny, P, iters = 516, 64, 2, 20

    def body(rank, P, ag):
        env = U.Env(rank, P, 0, ag)
        comm = U.Comm(env, *U.ring_neighbours(rank, P))
        st = torch.cuda.Stream()
        coord = U.Coord(comm, U.UC_MODE_DEVICE, st.cuda_stream)
        coord.set_timeout(5.0)
        J = U.Jacobi(comm, nx, ny)
        step_norms = np.zeros(iters, np.float64)  # pageable on purpose
        for i in range(iters):
            J.step(coord, True, step_norms[i:i + 1])
        coord.sync()
        run_norms = np.zeros(iters // 2, np.float64)
        J.run(coord, iters, 2, False, norms_out=run_norms)
        coord.sync()
        comm.barrier()
        J.destroy()
        coord.destroy()
        comm.destroy()
        env.finalize()
        return step_norms, run_norms

    res = run_ranks(P, body)
    _, _, want = _oracle(nx, ny, "ring", 2 * iters, 1)
    for step_norms, run_norms in res:
        assert np.allclose(step_norms, want[:iters], rtol=NORM_RTOL, atol=0)
        assert np.allclose(run_norms, want[iters::2], rtol=NORM_RTOL, atol=0)
