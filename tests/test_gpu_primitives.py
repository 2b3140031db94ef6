"""GPU tests of the communication primitives behind the C-ABI: Post/Acknowledge (put_signal /
signal_wait), AllReduce<SUM>, LaunchKernel, timeouts."""
import ctypes as C

import numpy as np
import pytest

from vranks import run_ranks

pytestmark = pytest.mark.gpu


class _CudaArray:
    def __init__(self, ptr, nbytes):
        self.__cuda_array_interface__ = {"shape": (nbytes,), "typestr": "|u1", "data": (ptr, False),
                                         "version": 3, "strides": None}


def dev_bytes(ptr, nbytes):
    """uint8 torch view of library-owned device memory (test-only inspection)."""
    import torch
    return torch.as_tensor(_CudaArray(ptr, nbytes), device="cuda")


def _setup(rank, P, ag, mode):
    import torch

    import paper_conf_cluster_sagbilieinu25_b200 as U
    env = U.Env(rank, P, 0, ag)
    comm = U.Comm(env, *U.ring_neighbours(rank, P))
    stream = torch.cuda.Stream()
    coord = U.Coord(comm, mode, stream.cuda_stream)
    coord.set_timeout(5.0)
    return U, env, comm, stream, coord


def _teardown(env, comm, coord, *mems):
    comm.barrier()
    for m in mems:
        m.free()
    coord.destroy()
    comm.destroy()
    env.finalize()


@pytest.mark.parametrize("nbytes", [16, 4096, 65536 + 16, 4 << 20, (4 << 20) + 8])
@pytest.mark.parametrize("P", [1, 2, 4])
@pytest.mark.parametrize("put_path,wait_path", [(0, 0), (1, 0), (0, 1), (1, 1)])
def test_put_signal_ring(P, nbytes, put_path, wait_path):
    """Every rank puts a rank-tagged buffer into its bottom neighbour and waits for the one from
    its top (the halo pattern of §8 a7), three rounds with monotone signal values -- on every
    transport: SM stores or the copy engine for the put, the spin kernel or cuStreamWaitValue64
    for the wait."""
    import torch

    def body(rank, P, ag):
        U, env, comm, stream, coord = _setup(rank, P, ag, 1)
        coord.set_p2p_path(put_path, wait_path)
        dst = U.SymMem(comm, nbytes)
        sig = U.SymMem(comm, 64)
        outs = []
        try:
            with torch.cuda.stream(stream):
                src = torch.arange(nbytes, dtype=torch.int32, device="cuda").to(torch.uint8)
            for rnd in range(1, 4):
                with torch.cuda.stream(stream):
                    src.add_(1)
                coord.put_signal(src.data_ptr(), dst, 0, nbytes, sig, 3, rnd, comm.bottom)
                coord.signal_wait(dst, 0, nbytes, sig, 3, rnd, comm.top)
                coord.sync()
                outs.append(dev_bytes(dst.ptr(), nbytes).cpu().numpy())
                comm.barrier()  # nobody overwrites dst before everyone checked it
            return outs
        finally:
            _teardown(env, comm, coord, dst, sig)

    res = run_ranks(P, body)
    base = (np.arange(nbytes) % 256).astype(np.uint8)
    for rank, outs in enumerate(res):
        for rnd, o in enumerate(outs, start=1):
            assert np.array_equal(o, (base + rnd).astype(np.uint8)), (rank, rnd)


@pytest.mark.parametrize("P", [1, 2, 3])
@pytest.mark.parametrize("nbytes,blocks", [(4096, 0), (1 << 20, 0), (1 << 20, 7), ((3 << 20) + 16, 0)])
def test_p2p_bench_patterns_deliver_data(P, nbytes, blocks):
    """uc_p2p_bench (configs[4] machinery): ping-pong and window move the sender's bytes into
    the partner's landing zone; the halo pattern fills both neighbours' zones; repeated calls
    keep the signal bases of every (pattern, peer) pair in step."""
    import torch

    def body(rank, P, ag):
        U, env, comm, stream, coord = _setup(rank, P, ag, 1)
        buf = U.SymMem(comm, 3 * nbytes)
        sig = U.SymMem(comm, 64)
        try:
            with torch.cuda.stream(stream):
                mine = dev_bytes(buf.ptr(), 3 * nbytes)
                mine[:nbytes] = (torch.arange(nbytes, device="cuda", dtype=torch.int32) * (rank + 3) % 251).to(
                    torch.uint8)
            # never torch.cuda.synchronize() here: a device-wide sync in one virtual rank would
            # wait for a peer's kernel that spins on this rank's not-yet-launched kernel
            stream.synchronize()
            comm.barrier()
            got = {}
            for rnd in range(2):
                if P >= 2 and rank in (0, 1):
                    coord.p2p_bench(U.UC_P2P_PINGPONG, buf, sig, nbytes, 3, 1, 1 - rank, rank, blocks)
                    coord.p2p_bench(U.UC_P2P_WINDOW, buf, sig, nbytes, 2, 4, 1 - rank, rank, blocks)
                coord.p2p_bench(U.UC_P2P_HALO, buf, sig, nbytes, 3, 1, 0, 0, blocks)
                coord.sync()
                comm.barrier()
            got = mine.cpu().numpy()
            comm.barrier()
            return got
        finally:
            _teardown(env, comm, coord, buf, sig)

    res = run_ranks(P, body)

    def src(r):
        return ((np.arange(nbytes, dtype=np.int64) * (r + 3)) % 251).astype(np.uint8)

    for r in range(P):
        top, bot = (r - 1) % P, (r + 1) % P
        # halo: zone [bytes, 2 bytes) from top, [2 bytes, 3 bytes) from bottom
        assert np.array_equal(res[r][nbytes:2 * nbytes], src(top)), r
        assert np.array_equal(res[r][2 * nbytes:], src(bot)), r


@pytest.mark.parametrize("dtype", ["f32", "f64", "u64"])
@pytest.mark.parametrize("P", [1, 2, 3, 4, 8])
def test_allreduce_device_oneshot(P, dtype):
    import torch
    tdt = {"f32": torch.float32, "f64": torch.float64, "u64": torch.int64}[dtype]
    code = {"f32": 0, "f64": 1, "u64": 2}[dtype]
    count = 1000

    def body(rank, P, ag):
        U, env, comm, stream, coord = _setup(rank, P, ag, 1)
        try:
            outs = []
            for rnd in range(3):  # epochs alternate parity
                with torch.cuda.stream(stream):
                    x = (torch.arange(count, device="cuda", dtype=torch.float64) * (rank + 1) + rnd).to(tdt)
                    y = torch.empty_like(x)
                coord.allreduce_sum(x.data_ptr(), y.data_ptr(), count, code)
                coord.allreduce_sum(x.data_ptr(), x.data_ptr(), count, code)  # in place
                coord.sync()
                outs.append((y.cpu().numpy(), x.cpu().numpy()))
            return outs
        finally:
            _teardown(env, comm, coord)

    res = run_ranks(P, body)
    for rnd in range(3):
        want = sum(np.arange(count, dtype=np.float64) * (r + 1) + rnd for r in range(P))
        for r in range(P):
            y, x = res[r][rnd]
            assert np.array_equal(y, x)
            assert np.array_equal(y, res[0][rnd][0])  # bit-identical on every rank
            assert np.allclose(y.astype(np.float64), want, rtol=1e-6)


def test_allreduce_host_mode_nccl_single_rank():
    import torch

    def body(rank, P, ag):
        U, env, comm, stream, coord = _setup(rank, P, ag, 0)
        try:
            with torch.cuda.stream(stream):
                x = torch.arange(10, device="cuda", dtype=torch.float64)
            coord.allreduce_sum(x.data_ptr(), x.data_ptr(), 10, 1)
            coord.sync()
            return x.cpu().numpy()
        finally:
            _teardown(env, comm, coord)

    (x,) = run_ranks(1, body)
    assert np.array_equal(x, np.arange(10, dtype=np.float64))


def test_launch_builtin_kernel():
    import torch

    def body(rank, P, ag):
        U, env, comm, stream, coord = _setup(rank, P, ag, 1)
        try:
            fn = U.builtin_kernel("uc_fill_f32")
            with torch.cuda.stream(stream):
                t = torch.zeros(5000, device="cuda")
            coord.launch(fn, (8,), (128,), 0, [C.c_void_p(t.data_ptr()), C.c_uint64(5000), C.c_float(2.5)])
            coord.sync()
            return t.cpu().numpy()
        finally:
            _teardown(env, comm, coord)

    (t,) = run_ranks(1, body)
    assert np.all(t == 2.5)


def test_signal_wait_timeout_is_reported():
    def body(rank, P, ag):
        U, env, comm, stream, coord = _setup(rank, P, ag, 1)
        sig = U.SymMem(comm, 64)
        try:
            coord.set_timeout(0.2)
            coord.signal_wait(None, 0, 0, sig, 0, 1, 0)
            with pytest.raises(U.UCError, match="UC_ERR_TIMEOUT"):
                coord.sync()
            coord.sync()  # error word was reset
            return True
        finally:
            _teardown(env, comm, coord, sig)

    assert run_ranks(1, body) == [True]


def test_partial_mode_collectives_use_host_api():
    """PartialDevice: collectives behave as PureHost -> NCCL, created on first use."""
    import torch

    def body(rank, P, ag):
        U, env, comm, stream, coord = _setup(rank, P, ag, 2)
        try:
            with torch.cuda.stream(stream):
                x = torch.arange(10, device="cuda", dtype=torch.float64)
            coord.allreduce_sum(x.data_ptr(), x.data_ptr(), 10, 1)
            coord.sync()
            return x.cpu().numpy()
        finally:
            _teardown(env, comm, coord)

    (x,) = run_ranks(1, body)
    assert np.array_equal(x, np.arange(10, dtype=np.float64))
