"""GPU parity of kernel variant 5 (T = 1..8 Jacobi iterations per launch, temporal blocking of
depth T, ghost-lane layout: one ghost lane per warp side for T <= 4, two for T = 5..8) against
the CPU oracle.

Variant 5 keeps A_{k+1}..A_{k+T-1} in registers and stores only A_{k+T}; the boundary rows of
every intermediate iterate are still exchanged with the neighbours (rounds 1..T per launch).
The bar is the north_star's: the grid bit-exact after N iterations, norms within 1e-5.  Counts
that are not multiples of T, norm cadences below T and thin slabs fall back to shorter launches
of the same layout; every mixture must stay bit-exact.
"""
import numpy as np
import pytest

from gpu_harness import assert_slabs_equal_global, bits, solve_gpu
from test_gpu_jacobi import NORM_RTOL, _check, _oracle

pytestmark = pytest.mark.gpu

TS = [1, 2, 3, 4, 5, 6, 7, 8]
TG = [2, 3, 4, 6, 8]  # both ghost layouts


def _v5(T, **kw):
    return dict(variant=5, tile_rows=T, **kw)


@pytest.mark.parametrize("T", TS)
@pytest.mark.parametrize("topology", ["ring", "dirichlet"])
@pytest.mark.parametrize("iters,ne", [(100, 10), (101, 10), (37, 3), (40, 0)])
def test_c1_256(T, topology, iters, ne):
    """configs[0] (256^2, 100 iterations, 1 GPU); odd counts and norm cadences below T."""
    res = _check(256, 256, 1, topology, "device", iters, norm_every=ne, **_v5(T))
    assert res["launch"]["variant"] == 5 and res["launch"]["tile_rows"] == T


@pytest.mark.parametrize("T", TG)
@pytest.mark.parametrize("nx,ny,iters", [(4, 8, 9), (8, 9, 20), (12, 16, 9), (1028, 64, 38), (2052, 33, 13),
                                         (4096, 40, 8), (36, 8, 12), (40, 9, 11), (964, 30, 17)])
@pytest.mark.parametrize("topology", ["ring", "dirichlet"])
def test_shapes_single_rank(T, nx, ny, iters, topology):
    """Ragged strips (NX/4 not a multiple of 30 owned lanes), tiny grids, thin slabs."""
    _check(nx, ny, 1, topology, "device", iters, norm_every=4, **_v5(T))


@pytest.mark.parametrize("T", TG)
@pytest.mark.parametrize("P", [2, 3, 4, 8])
@pytest.mark.parametrize("topology", ["ring", "dirichlet"])
def test_partition_invariance(T, P, topology):
    """Virtual ranks P = 2..8: every intermediate level's edge rows cross ranks (h buffers)."""
    _check(520, 24 * P, P, topology, "device", 27, norm_every=5, **_v5(T))


@pytest.mark.parametrize("T", [2, 3, 4, 5, 8])
@pytest.mark.parametrize("P,ny", [(2, 4), (2, 6), (3, 9), (2, 8), (4, 32), (2, 16), (2, 30)])
def test_few_rows_per_rank(T, P, ny):
    """n = 2..8: launches shrink to the deepest T' with n >= 2T'; one row chunk per strip."""
    for topology in ("ring", "dirichlet"):
        _check(64, ny, P, topology, "device", 13, norm_every=0, **_v5(T))


@pytest.mark.parametrize("T", [2, 4, 6, 8])
@pytest.mark.parametrize("block_x,bps,stages", [(32, 1, 9), (64, 2, 18), (128, 0, 9), (256, 1, 27), (96, 0, 0)])
def test_launch_geometries(T, block_x, bps, stages):
    """Strip width (ghost lanes meet strip edges), chunk count and ring depth: 4 ranks."""
    if T > 4:  # two ghost lanes: the launch bounds allow 7 consumer warps per block
        block_x = min(block_x, 224)
    res = _check(1028, 128, 4, "ring", "device", 12, norm_every=4, block_x=block_x, blocks_per_sm=bps,
                 stages=stages, **_v5(T))
    assert res["launch"]["variant"] == 5


@pytest.mark.parametrize("T", TG)
def test_random_values_everywhere(T):
    nx, ny = 1028, 48
    rng = np.random.default_rng(11)
    init = rng.random((ny + 2, nx), dtype=np.float32)
    init[0], init[-1] = init[ny], init[1]
    _check(nx, ny, 1, "ring", "device", 14, norm_every=7, init=init, **_v5(T))
    _check(nx, ny, 3, "ring", "device", 14, norm_every=4, init=init, **_v5(T))
    _check(nx, ny, 2, "dirichlet", "device", 14, norm_every=0, init=init, **_v5(T))


@pytest.mark.parametrize("T", [3, 4, 8])
def test_graph_eager_stepwise_chunked_agree(T):
    kw = _v5(T)
    a = solve_gpu(516, 64, 2, "ring", "device", 30, 7, use_graph=True, **kw)
    b = solve_gpu(516, 64, 2, "ring", "device", 30, 7, use_graph=False, **kw)
    c = solve_gpu(516, 64, 2, "ring", "device", 30, 1, stepwise=True, **kw)
    d = solve_gpu(516, 64, 2, "ring", "device", 30, 7, chunks_of_run=[3, 11, 16], **kw)
    e = solve_gpu(516, 64, 2, "ring", "device", 30, 7, chunks_of_run=[5, 5, 5, 15], use_graph=False, **kw)
    for x in (b, c, d, e):
        for s1, s2 in zip(a["final"], x["final"]):
            assert np.array_equal(bits(s1), bits(s2))
    for x in (b, d, e):
        assert np.array_equal(a["norms"], x["norms"])
    assert np.array_equal(a["norms"], c["norms"][[0, 7, 14, 21, 28]])
    _, want, want_norms = _oracle(516, 64, "ring", 30, 7)
    assert_slabs_equal_global(a["final"], want, 2, "ring")
    assert np.allclose(a["norms"], want_norms, rtol=NORM_RTOL, atol=0)


def test_switch_variants_and_modes_mid_run():
    """Variant 5 (T = 4, 3) <-> variant 4 <-> variant 1 on one solver; then variant 5 in host and
    partial mode (one-iteration launches of the ghost-lane layout + NCCL / Acknowledge)."""
    import torch

    import paper_conf_cluster_sagbilieinu25_b200 as U
    from vranks import run_ranks
    nx, ny, P = 1028, 64, 2

    def body(rank, P, ag):
        env = U.Env(rank, P, 0, ag)
        comm = U.Comm(env, *U.ring_neighbours(rank, P))
        st = torch.cuda.Stream()
        coord = U.Coord(comm, U.UC_MODE_DEVICE, st.cuda_stream)
        coord.set_timeout(5.0)
        J = U.Jacobi(comm, nx, ny)
        out = []
        for v, T, it in ((5, 4, 10), (4, 0, 5), (5, 3, 7), (1, 0, 3), (5, 8, 19), (5, 6, 8), (5, 4, 9)):
            J.set_launch(v, 0, 0, 0, T)
            out.append(J.run(coord, it, 5))
            coord.sync()
        slab = J.copy_out(coord)
        comm.barrier()
        J.destroy()
        coord.destroy()
        comm.destroy()
        env.finalize()
        return slab, np.concatenate(out)

    res = run_ranks(P, body)
    _, want, want_norms = _oracle(nx, ny, "ring", 61, 5)
    assert_slabs_equal_global([r[0] for r in res], want, P, "ring")
    assert np.allclose(res[0][1], want_norms, rtol=NORM_RTOL, atol=0)

    env = U.Env(0, 1, 0)
    comm = U.Comm(env, 0, 0)
    st = torch.cuda.Stream()
    coords = {m: U.Coord(comm, v, st.cuda_stream) for m, v in (("device", 1), ("host", 0), ("partial", 2))}
    J = U.Jacobi(comm, nx, ny)
    J.set_launch(5, 0, 0, 0, 4)
    for m, it in (("device", 8), ("host", 5), ("device", 6), ("partial", 3), ("device", 7), ("host", 2)):
        J.run(coords[m], it, 0)
        coords[m].sync()
    out = J.copy_out(coords["device"])
    J.destroy()
    for c in coords.values():
        c.destroy()
    comm.destroy()
    env.finalize()
    _, want, _ = _oracle(nx, ny, "ring", 31, 0)
    assert_slabs_equal_global([out], want, 1, "ring")


@pytest.mark.parametrize("T", [4, 8])
@pytest.mark.parametrize("mode", ["host", "partial"])
def test_host_and_partial_modes(mode, T):
    _check(1028, 40, 1, "ring", mode, 11, norm_every=3, **_v5(T))


@pytest.mark.parametrize("T", [4, 8])
def test_subnormal_front_no_ftz(T):
    nx, ny = 96, 16
    a = np.zeros((ny + 2, nx), np.float32)
    a[:, 0] = 1.0
    for k in (64, 70, 74, 75):
        res = solve_gpu(nx, ny, 1, "ring", "device", k, 0, init=a, **_v5(T))
        s = res["final"][0]
        want = np.float32(2.0 ** (-2 * k)) if k <= 74 else np.float32(0.0)
        assert s[1, k] == want and s[1, k + 1] == 0.0


@pytest.mark.parametrize("T", [2, 3, 4, 6, 8])
def test_full_size_16384(T):
    """16384^2 (configs[2]/[3] at P = 1): whole grid bit-exact, norms on every level."""
    _check(16384, 16384, 1, "ring", "device", 2 * T + 1, norm_every=T, **_v5(T))


def test_config2_strong_16384_over_8_ranks():
    _check(16384, 16384, 8, "ring", "device", 9, norm_every=4, **_v5(4))


@pytest.mark.parametrize("T", [4, 8])
def test_config1_4096_2ranks_1000_iterations(T):
    _check(4096, 4096, 2, "ring", "device", 1000, norm_every=100, **_v5(T))


# ---------------------------------------------------------------------------------------------
# The deep instances -- the shipped default jacobi_t_kernel<8, 2> and <6, 2> -- where the
# multi-rank protocol can break: distinct top and bottom peers (P >= 3), the chain ends, the
# thinnest slabs, full-size geometry.  A norm cadence below T demotes launches, so these runs use
# norm_every 0 or a multiple of T and assert (device launch counters, uc_jacobi_launch_counts)
# that depth-T launches really ran; the harness also checks every launch against the plan.
DEEP = [6, 8]


def _deep(res, T, n_expected):
    assert res["launch"]["variant"] == 5 and res["launch"]["tile_rows"] == T
    for c in res["counts_all"]:
        assert c[T] == n_expected, (T, c)


@pytest.mark.parametrize("T", DEEP)
@pytest.mark.parametrize("P", [3, 4, 8])
@pytest.mark.parametrize("topology,nem", [("ring", 0), ("ring", 1), ("dirichlet", 2)])
def test_deep_distinct_peers(T, P, topology, nem):
    res = _check(1028, 4 * T * P, P, topology, "device", 3 * T, norm_every=nem * T, **_v5(T))
    _deep(res, T, 3)


@pytest.mark.parametrize("T", DEEP)
@pytest.mark.parametrize("P,extra", [(3, 0), (4, 1), (2, 0)])
def test_deep_thinnest_slabs(T, P, extra):
    """n = 2T (every chunk is a boundary chunk) and n = 2T + 1 (ragged), two strips per rank."""
    for topology in ("ring", "dirichlet"):
        res = _check(2052, (2 * T + extra) * P, P, topology, "device", 2 * T, norm_every=T, **_v5(T))
        _deep(res, T, 2)


@pytest.mark.parametrize("T", DEEP)
def test_deep_random_values_p3(T):
    nx, ny = 1028, 12 * T
    rng = np.random.default_rng(T)
    init = rng.random((ny + 2, nx), dtype=np.float32)
    init[0], init[-1] = init[ny], init[1]
    res = _check(nx, ny, 3, "ring", "device", 4 * T, norm_every=T, init=init, **_v5(T))
    _deep(res, T, 4)


def test_default_is_t8_config1():
    """configs[1] (4096^2, 2 ranks, 1000 iterations, norm every 100) at the library default:
    T = 8, 125 launches of 8."""
    res = _check(4096, 4096, 2, "ring", "device", 1000, norm_every=100)
    _deep(res, 8, 125)


def test_t6_config1():
    """configs[1] at T = 6: 165 launches of 6 and two of 5 (the remainder 4 split with the launch
    before it)."""
    res = _check(4096, 4096, 2, "ring", "device", 1000, norm_every=100, **_v5(6))
    for c in res["counts_all"]:
        assert c[6] == 165 and c[5] == 2 and sum(c[:15]) == 167, c


@pytest.mark.parametrize("T", DEEP)
def test_deep_config3_two_ranks(T):
    """configs[3] at P = 2 (16384 x 32768 global, 16384^2 per rank: the bench's per-GPU geometry
    with real neighbours), 2T + 1 iterations with a norm every T: launches T, then the remainder
    1 split with the launch before it."""
    res = _check(16384, 32768, 2, "ring", "device", 2 * T + 1, norm_every=T, **_v5(T))
    _deep(res, T, 1)


def test_two_virtual_ranks_need_concurrent_kernels():
    """States the requirement the virtual-rank tests rely on: two ranks on ONE GPU run their
    device-mode kernels on two streams, and each kernel spins on flags the other sets, so both
    grids must make progress at the same time.  CUDA does not guarantee concurrent kernels (a
    profiler or MPS serialises them -- the paper notes the missing preemptive scheduling,
    P:115), which is why smoke() runs P = 1.  When the peer's kernel does NOT run alongside
    (here: rank 1 launches only after rank 0's spin timeout), the waits are bounded and the
    waiting rank reports UC_ERR_TIMEOUT instead of hanging the device."""
    import time

    import torch

    import paper_conf_cluster_sagbilieinu25_b200 as U
    from vranks import run_ranks

    def body(rank, P, ag):
        env = U.Env(rank, P, 0, ag)
        comm = U.Comm(env, *U.ring_neighbours(rank, P))
        st = torch.cuda.Stream()
        co = U.Coord(comm, U.UC_MODE_DEVICE, st.cuda_stream)
        co.set_timeout(0.5)
        J = U.Jacobi(comm, 1028, 48)
        comm.barrier()
        if rank == 1:
            time.sleep(2.0)
        t0 = time.time()
        J.run(co, 12, 0, use_graph=False)
        try:
            co.sync()
            status = U.UC_OK
        except U.UCError as e:
            status = e.status
        dt = time.time() - t0
        comm.barrier()
        J.destroy()
        co.destroy()
        comm.destroy()
        env.finalize()
        return status, dt

    res = run_ranks(2, body, timeout=60)
    # rank 0 waited for a peer that was not running: its bounded spin expired and it reports
    # UC_ERR_TIMEOUT (a waiter that gives up still completes its own puts and flags, so the late
    # rank finishes -- the error is the application's signal that the run is invalid); nobody hangs
    assert res[0][0] == U.UC_ERR_TIMEOUT, res
    assert all(dt < 10.0 for _, dt in res), res


# ---------------------------------------------------------------------------------------------
# Host mode (the NCCL comparator): the paper's one-exchange-per-iteration path, the
# deep-halo path (T rows exchanged once per T-iteration launch) and the overlapped split launch
# (edge chunks -> NCCL on a side stream || the other chunks).  One GPU: P = 1 ring (NCCL sends to
# itself; top == bottom) and chain; P >= 2 needs one GPU per rank (test_gpu_multiprocess.py).
@pytest.mark.parametrize("deep,overlap", [(0, 0), (1, 0), (0, 1), (1, 1)])
@pytest.mark.parametrize("topology", ["ring", "dirichlet"])
@pytest.mark.parametrize("iters,ne", [(25, 6), (13, 0), (20, 5), (7, 1)])
def test_host_paths(deep, overlap, topology, iters, ne):
    res = _check(1028, 192, 1, topology, "host", iters, norm_every=ne, host_path=(deep, overlap))
    if deep and ne in (0, 6):
        assert res["counts"][6] >= 1, res["counts"]


@pytest.mark.parametrize("deep,overlap", [(1, 0), (1, 1), (0, 1)])
def test_host_paths_full_size(deep, overlap):
    res = _check(16384, 16384, 1, "ring", "host", 13, norm_every=6, host_path=(deep, overlap))
    if deep:
        assert res["counts"][6] == 1 and res["counts"][4] == 1 and res["counts"][3] == 1, res["counts"]


@pytest.mark.parametrize("P,topology", [(3, "ring"), (2, "dirichlet")])
def test_t6_injected_flag_latency(monkeypatch, P, topology):
    """Every boundary-round flag released 20 us late (UC_INJECT_PUT_DELAY_NS, the knob behind
    bench.py --inject-delay-us): the waits absorb it, the grid stays bit-exact."""
    monkeypatch.setenv("UC_INJECT_PUT_DELAY_NS", "20000")
    res = _check(1028, 32 * P, P, topology, "device", 24, norm_every=8)
    assert all(c[8] == 3 for c in res["counts_all"])


# --------------------------------------------------------------------------- the scaled march
# Norm-free T-level launches drop the 0.25 products of levels 1..T-1: exact only
# while every nonzero |A_k| a warp reads lies in [2^(-103+2T), 2^110).  Outside that range the
# block re-runs its march unscaled; the device counts those blocks (launch_counts()[15]).  Each
# case below is bit-exact against the oracle AND checks which path ran.
def _scaled_case(nx, ny, P, T, iters, init, topology="ring"):
    _, want, _ = _oracle(nx, ny, topology, iters, 0, init=init)
    res = solve_gpu(nx, ny, P, topology, "device", iters, 0, init=init, **_v5(T))
    assert_slabs_equal_global(res["final"], want, P, topology)
    return [c[15] for c in res["counts_all"]]


@pytest.mark.parametrize("T", [6, 8])
def test_scaled_march_runs_on_ordinary_fields(T):
    """The generator's field (values in [0, 1) on a 2^-24 grid): no block leaves the scaled march."""
    from inputs import gen
    g = gen.global_field(2052, 96, "ring")
    assert _scaled_case(2052, 96, 2, T, 3 * T, g) == [0, 0]


@pytest.mark.parametrize("T", [6, 8])
@pytest.mark.parametrize("scale_log2", [-100, -60, 100, 112])
def test_scaled_march_falls_back_outside_its_range(T, scale_log2):
    """One launch of the generator's field scaled by 2^s (nonzero |values| in [2^(s-24), 2^s)).
    2^-100: tiny but normal, the unscaled iteration's values can reach the subnormal range within
    T levels; 2^112: scaled sums could overflow -- every interior block re-runs unscaled.  2^-60
    and 2^100 are inside [2^(-103+2T), 2^110) for T <= 8: no re-run."""
    from inputs import gen
    g = gen.global_field(2052, 96, "ring")
    g = (g.astype(np.float64) * 2.0 ** scale_log2).astype(np.float32)
    reruns = _scaled_case(2052, 96, 2, T, T, g)
    if -103 + 2 * T <= scale_log2 - 24 and scale_log2 < 110:
        assert reruns == [0, 0], reruns
    else:
        assert all(r > 0 for r in reruns), reruns


@pytest.mark.parametrize("T", [6, 8])
def test_scaled_march_spike_into_the_subnormals(T):
    """A single 1.0 in an interior column of a zero field, 12 launches: the front of the diamond
    decays by 4 per iteration into the subnormal range (2^-2k at distance k), so later launches
    meet values below 2^(-103+2T) in the blocks around the spike and re-run them unscaled, while
    far blocks stay scaled.  Bit-exact (no FTZ, no scaling error) either way."""
    nx, ny = 1028, 128
    a = np.zeros((ny + 2, nx), np.float32)
    a[64, 520] = 1.0
    reruns = _scaled_case(nx, ny, 1, T, 12 * T, a)
    assert reruns[0] > 0


@pytest.mark.parametrize("T", [8])
def test_scaled_march_inf_and_huge(T):
    """+inf and 2^126 values in one interior point: inf is out of the scaled range (re-run);
    the unscaled iteration spreads inf and large finite values exactly as the oracle does."""
    from inputs import gen
    g = gen.global_field(2052, 64, "ring")
    g[20, 700] = np.float32(np.inf)
    g[40, 1500] = np.float32(2.0 ** 126)
    reruns = _scaled_case(2052, 64, 1, T, 3 * T, g)
    assert reruns[0] > 0


# --------------------------------------------------------------------------- balanced chunks
# Device-mode T-level launches without a norm round take each block's (strip, chunk, rows) from
# a table re-partitioned from measured per-block march times.  Any valid table
# computes the same grid; norm launches keep the static chunking, so norms are independent of it.
def _rand_rates(seed):
    def f(rank, grid):
        rng = np.random.default_rng(seed + 7 * rank)
        return rng.uniform(0.2, 5.0, grid)
    return f


@pytest.mark.parametrize("T", [6, 8])
@pytest.mark.parametrize("P,topology", [(1, "ring"), (2, "ring"), (3, "dirichlet")])
def test_balanced_table_any_partition_is_exact(T, P, topology):
    """Wildly unequal forced rates (0.2 .. 5): blocks change strips and chunk sizes; grid bit-exact,
    norms bit-identical to the static chunking's (norm launches do not use the table)."""
    nx, ny, iters, ne = 2052, 1024 * P, 5 * T + 3, 2 * T
    res = _check(nx, ny, P, topology, "device", iters, norm_every=ne, balance_rates=_rand_rates(11), **_v5(T))
    tabs = res["balance_tables"]
    assert all(t is not None for t in tabs)
    info = res["launch"]
    for t in tabs:  # the table is a partition of every strip's rows, chunks in order
        assert sorted(map(tuple, t[:, :2].tolist())) == [(s, q) for s in range(info["strips"])
                                                         for q in range(info["chunks"])]
        assert not np.array_equal(t[:, 0], np.arange(len(t)) % info["strips"])  # not the static one
    ref = solve_gpu(nx, ny, P, topology, "device", iters, ne, balance=False, **_v5(T))
    assert ref["balance_tables"][0] is None
    assert np.array_equal(bits(res["norms"]), bits(ref["norms"]))


@pytest.mark.parametrize("T", [8])
def test_balance_adapts_over_runs_and_stays_exact(T):
    """Several runs: the table moves away from the equal split as measured rates come in (every
    run after the first reads the previous run's block times back), and every run is bit-exact.
    With equal rates the inner chunks of a strip differ by at most one row; SMs differ in speed
    by far more than that, so the adapted sizes spread."""
    nx, ny = 4100, 2048
    res = _check(nx, ny, 1, "ring", "device", 16 * T, norm_every=0, chunks_of_run=[2 * T] * 8, balance=True,
                 **_v5(T))
    t = res["balance_tables"][0]
    assert t is not None
    inner = [r[3] - r[2] + 1 for r in t if 0 < r[1] < res["launch"]["chunks"] - 1]
    assert max(inner) - min(inner) > 2, (min(inner), max(inner))
