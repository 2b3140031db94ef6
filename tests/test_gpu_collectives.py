"""The rest of the paper's collective interface (Listing 7) on the GPU:
Reduce/AllReduce with every ReductionOperator, Broadcast, AllGather(v), AlltoAll, Gather,
Scatter and the stream barrier -- device mode with 1..4 virtual ranks, host and partial mode
(NCCL) with one rank.  Results are compared with numpy element by element."""
import numpy as np
import pytest

from vranks import run_ranks

pytestmark = pytest.mark.gpu

OPS = {0: np.add, 1: np.multiply, 2: np.minimum, 3: np.maximum}


class _CudaArray:
    def __init__(self, ptr, nbytes):
        self.__cuda_array_interface__ = {"shape": (nbytes,), "typestr": "|u1", "data": (ptr, False),
                                         "version": 3, "strides": None}


def _view(ptr, nbytes):
    import torch
    return torch.as_tensor(_CudaArray(ptr, nbytes), device="cuda")


def _env(rank, P, ag, mode):
    import torch

    import paper_conf_cluster_sagbilieinu25_b200 as U
    env = U.Env(rank, P, 0, ag)
    comm = U.Comm(env, *U.ring_neighbours(rank, P))
    st = torch.cuda.Stream()
    co = U.Coord(comm, mode, st.cuda_stream)
    co.set_timeout(10.0)
    return U, env, comm, st, co


def _close(env, comm, co, *mems):
    comm.barrier()
    for m in mems:
        m.free()
    co.destroy()
    comm.destroy()
    env.finalize()


def _pattern(rank, nbytes, salt):
    return ((np.arange(nbytes, dtype=np.int64) * (2 * rank + 1) + 7 * salt + rank) % 251).astype(np.uint8)


CASES = [(1, 1), (2, 1), (3, 1), (4, 1), (1, 0), (1, 2)]  # (P, mode)


@pytest.mark.parametrize("P,mode", CASES)
@pytest.mark.parametrize("nbytes", [16, 4100, 1 << 20])
def test_data_collectives(P, mode, nbytes):
    import torch

    def body(rank, P, ag):
        U, env, comm, st, co = _env(rank, P, ag, mode)
        buf = U.SymMem(comm, P * nbytes)
        out = {}
        try:
            with torch.cuda.stream(st):
                src = torch.empty(P * nbytes, dtype=torch.uint8, device="cuda")
                recv = _view(buf.ptr(), P * nbytes)
            for rnd in range(2):  # two epochs of every collective
                mine = np.concatenate([_pattern(rank, nbytes, rnd * P + j) for j in range(P)])
                with torch.cuda.stream(st):
                    src.copy_(torch.from_numpy(mine))
                    recv.zero_()
                co.allgather(src.data_ptr(), buf, 0, nbytes)
                co.sync()
                out[("allgather", rnd)] = recv.cpu().numpy().copy()
                with torch.cuda.stream(st):
                    recv.zero_()
                co.alltoall(src.data_ptr(), buf, 0, nbytes)
                co.sync()
                out[("alltoall", rnd)] = recv.cpu().numpy().copy()
                root = rnd % P
                with torch.cuda.stream(st):
                    recv.zero_()
                co.gather(src.data_ptr(), buf, 0, nbytes, root)
                co.sync()
                out[("gather", rnd)] = recv.cpu().numpy().copy()
                with torch.cuda.stream(st):
                    recv.zero_()
                co.scatter(src.data_ptr() if rank == root else 0, buf, 0, nbytes, root)
                co.sync()
                out[("scatter", rnd)] = recv.cpu().numpy()[:nbytes].copy()
                with torch.cuda.stream(st):
                    recv.copy_(src)
                co.broadcast(buf, 0, nbytes, root)
                co.sync()
                out[("bcast", rnd)] = recv.cpu().numpy()[:nbytes].copy()
                counts = [max(0, nbytes - 16 * q) for q in range(P)]
                displs = list(np.cumsum([0] + counts[:-1]))
                with torch.cuda.stream(st):
                    recv.zero_()
                co.allgatherv(src.data_ptr(), counts[rank], buf, 0, counts, displs)
                co.barrier()
                co.sync()
                out[("allgatherv", rnd)] = (recv.cpu().numpy().copy(), counts, displs)
                comm.barrier()  # nobody starts the next round's writes before all checked
            return out
        finally:
            _close(env, comm, co, buf)

    res = run_ranks(P, body)
    for rnd in range(2):
        chunks = {r: [_pattern(r, nbytes, rnd * P + j) for j in range(P)] for r in range(P)}
        root = rnd % P
        for r in range(P):
            o = res[r]
            assert np.array_equal(o[("allgather", rnd)], np.concatenate([chunks[q][0] for q in range(P)])), r
            assert np.array_equal(o[("alltoall", rnd)], np.concatenate([chunks[q][r] for q in range(P)])), r
            if r == root:
                assert np.array_equal(o[("gather", rnd)], np.concatenate([chunks[q][0] for q in range(P)]))
            assert np.array_equal(o[("scatter", rnd)], chunks[root][r]), r
            assert np.array_equal(o[("bcast", rnd)], chunks[root][0]), r
            got, counts, displs = o[("allgatherv", rnd)]
            for q in range(P):
                assert np.array_equal(got[displs[q]:displs[q] + counts[q]], chunks[q][0][:counts[q]]), (r, q)


@pytest.mark.parametrize("P,mode", CASES)
@pytest.mark.parametrize("dtype", ["f32", "f64", "u64"])
def test_reductions_every_operator(P, mode, dtype):
    import torch
    tdt = {"f32": torch.float32, "f64": torch.float64, "u64": torch.int64}[dtype]
    code = {"f32": 0, "f64": 1, "u64": 2}[dtype]
    count = 777

    def data(rank, op):
        x = (np.arange(count, dtype=np.float64) % 13 + rank + 1) * (1 if op != 1 else 0.5)
        if dtype == "u64":
            x = np.floor(x * 4)
        return x

    def body(rank, P, ag):
        U, env, comm, st, co = _env(rank, P, ag, mode)
        try:
            out = {}
            for op in (0, 1, 2, 3):
                with torch.cuda.stream(st):
                    x = torch.from_numpy(data(rank, op)).to(device="cuda", dtype=tdt)
                    y = torch.zeros_like(x)
                    z = torch.zeros_like(x)
                co.allreduce(x.data_ptr(), y.data_ptr(), count, code, op)
                root = op % P
                co.reduce(x.data_ptr(), z.data_ptr(), count, code, op, root)
                co.sync()
                out[op] = (y.cpu().numpy(), z.cpu().numpy(), root)
            return out
        finally:
            _close(env, comm, co)

    res = run_ranks(P, body)
    npdt = {"f32": np.float32, "f64": np.float64, "u64": np.int64}[dtype]
    for op, fn in OPS.items():
        want = data(0, op).astype(npdt)
        for r in range(1, P):
            want = fn(want, data(r, op).astype(npdt))
        for r in range(P):
            y, z, root = res[r][op]
            assert np.allclose(y.astype(np.float64), want.astype(np.float64), rtol=1e-6), (op, r)
            assert np.array_equal(y, res[0][op][0]), (op, r)  # bit-identical on every rank
            if r == root:
                assert np.allclose(z.astype(np.float64), want.astype(np.float64), rtol=1e-6), (op, r)
