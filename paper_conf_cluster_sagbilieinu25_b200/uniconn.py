"""Thin Python binding of libuniconn_b200 -- the same names as the C-ABI (include/uniconn.h),
argument marshalling only.  Every step of the hot path runs in the library's CUDA kernels.

Objects mirror the paper's abstractions (§IV):
``Env`` (Environment), ``Comm`` (Communicator), ``SymMem`` (Memory), ``Coord`` (Coordinator)
and ``Jacobi`` (the §VI-C solver step).  Streams are plain ``cudaStream_t`` integers, e.g.
``torch.cuda.Stream().cuda_stream``.

Bootstrap allgathers (the library's only dependency on the caller's process group):
``torch_allgather()`` for one process per GPU (torch.distributed, gloo group) and
``ThreadAllgather`` for "virtual ranks" (one host thread per rank inside one process).
"""
from __future__ import annotations

import ctypes as C
import threading
from typing import Callable, Optional

import numpy as np

from ._lib import (UC_PUT_SM, UC_PUT_CE, UC_WAIT_KERNEL, UC_WAIT_STREAM, UC_PLAN_DEEP_HALO, UC_OK, UC_ERR_TIMEOUT, UC_ERR_STATE, UC_ERR_ARG, ALLGATHER_FN, UC_F32, UC_F64, UC_MODE_DEVICE, UC_MODE_HOST, UC_MODE_PARTIAL,  # noqa: F401
                   UC_MAX, UC_MIN, UC_P2P_HALO, UC_P2P_PINGPONG, UC_P2P_WINDOW, UC_PROD, UC_SUM, UC_TOPO_CHAIN,
                   UC_TOPO_NONE, UC_TOPO_RING, UC_U64,
                   UCError, check, lib)



AllgatherImpl = Callable[[bytes, int], bytes]  # (my bytes, bytes_per_rank) -> size*bytes_per_rank bytes


def _wrap_allgather(impl: Optional[AllgatherImpl]):
    if impl is None:
        return ALLGATHER_FN()  # NULL function pointer: only valid for world_size == 1

    def cb(send, recv, nbytes, _ctx):
        try:
            mine = C.string_at(send, nbytes)
            out = impl(mine, nbytes)
            C.memmove(recv, out, len(out))
            return 0
        except Exception:  # noqa: BLE001 -- reported as UC_ERR_BOOTSTRAP by the library
            import traceback
            traceback.print_exc()
            return 1

    return ALLGATHER_FN(cb)


def torch_allgather(group=None) -> AllgatherImpl:
    """Allgather over torch.distributed (CPU tensors; use a gloo group)."""
    import torch
    import torch.distributed as dist

    def impl(mine: bytes, nbytes: int) -> bytes:
        world = dist.get_world_size(group)
        t = torch.frombuffer(bytearray(mine), dtype=torch.uint8)
        outs = [torch.empty(nbytes, dtype=torch.uint8) for _ in range(world)]
        dist.all_gather(outs, t, group=group)
        return b"".join(bytes(o.numpy().tobytes()) for o in outs)

    return impl


class ThreadAllgather:
    """In-process allgather for virtual ranks (one host thread per rank)."""

    def __init__(self, size: int, timeout: float = 120.0):
        self.size = size
        self.timeout = timeout
        self._barrier = threading.Barrier(size)
        self._slots = [b""] * size

    def for_rank(self, rank: int) -> AllgatherImpl:
        def impl(mine: bytes, nbytes: int) -> bytes:
            self._slots[rank] = mine
            self._barrier.wait(self.timeout)
            out = b"".join(self._slots)
            self._barrier.wait(self.timeout)
            return out
        return impl


class Env:
    """Environment: world rank/size and the GPU this rank uses."""

    def __init__(self, rank: int = 0, size: int = 1, device: int = 0, allgather: Optional[AllgatherImpl] = None):
        self._cb = _wrap_allgather(allgather)
        h = C.c_void_p()
        check(lib.uc_env_init(rank, size, device, self._cb, None, C.byref(h)), "uc_env_init")
        self.h = h
        self.rank, self.size, self.device = rank, size, device

    def finalize(self):
        if self.h:
            check(lib.uc_env_finalize(self.h), "uc_env_finalize")
            self.h = None


class Comm:
    """Communicator: rank/size plus the top/bottom halo neighbours."""

    def __init__(self, env: Env, top: int, bottom: int):
        h = C.c_void_p()
        check(lib.uc_comm_create(env.h, top, bottom, C.byref(h)), "uc_comm_create")
        self.h, self.env = h, env
        r, s, t, b, topo = (C.c_int() for _ in range(5))
        check(lib.uc_comm_info(h, C.byref(r), C.byref(s), C.byref(t), C.byref(b), C.byref(topo)), "uc_comm_info")
        self.rank, self.size, self.top, self.bottom, self.topology = r.value, s.value, t.value, b.value, topo.value

    def device_view(self) -> int:
        p = C.c_void_p()
        check(lib.uc_comm_device_view(self.h, C.byref(p)), "uc_comm_device_view")
        return p.value

    def barrier(self, stream: int = 0):
        check(lib.uc_comm_barrier(self.h, C.c_void_p(stream)), "uc_comm_barrier")

    def destroy(self):
        if self.h:
            check(lib.uc_comm_destroy(self.h), "uc_comm_destroy")
            self.h = None


def ring_neighbours(rank: int, size: int):
    return (rank - 1 + size) % size, (rank + 1) % size


def chain_neighbours(rank: int, size: int):
    return (rank - 1 if rank > 0 else -1), (rank + 1 if rank < size - 1 else -1)


def launch_plan(variant: int, levels: int, mode: int, n_local: int, iters: int, norm_every: int) -> list:
    """uc_jacobi_launch_plan: iterations per launch of a uc_jacobi_run (host logic, no device)."""
    cnt = lib.uc_jacobi_launch_plan(variant, levels, mode, n_local, iters, norm_every, None, 0)
    if cnt < 0:
        check(-cnt, "uc_jacobi_launch_plan")
    buf = (C.c_int * max(1, cnt))()
    lib.uc_jacobi_launch_plan(variant, levels, mode, n_local, iters, norm_every, buf, cnt)
    return list(buf[:cnt])


def balance_plan(strips: int, chunks: int, n: int, shrink: int, levels: int, rates=None):
    """uc_balance_plan: the balanced chunk table for per-block rates (host logic, no device);
    returns an int array [strips * chunks, 4] of {strip, chunk, first row, last row}."""
    import numpy as np
    g = strips * chunks
    tab = np.zeros((g, 4), np.int32)
    r = None if rates is None else np.ascontiguousarray(rates, np.float64)
    rp = None if r is None else r.ctypes.data_as(C.POINTER(C.c_double))
    check(lib.uc_balance_plan(strips, chunks, n, shrink, levels, rp, tab.ctypes.data_as(C.POINTER(C.c_int))),
          "uc_balance_plan")
    return tab


class SymMem:
    """Symmetric memory: same-size, peer-addressable on every rank."""

    def __init__(self, comm: Comm, nbytes: int):
        h = C.c_void_p()
        check(lib.uc_mem_alloc_symmetric(comm.h, nbytes, C.byref(h)), "uc_mem_alloc_symmetric")
        self.h, self.comm, self.nbytes = h, comm, nbytes

    def ptr(self, rank: Optional[int] = None) -> Optional[int]:
        return lib.uc_mem_ptr(self.h, self.comm.rank if rank is None else rank)

    def free(self):
        if self.h:
            check(lib.uc_mem_free_symmetric(self.h), "uc_mem_free_symmetric")
            self.h = None


class Coord:
    """Coordinator bound to a stream and a launch mode."""

    def __init__(self, comm: Comm, mode: int, stream: int = 0):
        h = C.c_void_p()
        check(lib.uc_coord_create(comm.h, mode, C.c_void_p(stream), C.byref(h)), "uc_coord_create")
        self.h, self.comm, self.mode, self.stream = h, comm, mode, stream
        self._outputs = []  # host output arrays the library completes at uc_coord_sync

    def keep(self, arr: np.ndarray) -> np.ndarray:
        """Hold a host output array alive until the next sync (pageable outputs are written by
        uc_coord_sync from a page-locked staging copy)."""
        self._outputs.append(arr)
        return arr

    def sync(self):
        try:
            check(lib.uc_coord_sync(self.h), "uc_coord_sync")
        finally:
            self._outputs.clear()

    def set_p2p_path(self, put_path: int = 0, wait_path: int = 0):
        """uc_coord_set_p2p_path: UC_PUT_SM / UC_PUT_CE, UC_WAIT_KERNEL / UC_WAIT_STREAM."""
        check(lib.uc_coord_set_p2p_path(self.h, put_path, wait_path), "uc_coord_set_p2p_path")

    def set_timeout(self, seconds: float):
        check(lib.uc_coord_set_timeout(self.h, int(seconds * 1e9)), "uc_coord_set_timeout")

    def launch(self, cu_function: int, grid, block, smem: int, args: list):
        g = tuple(grid) + (1,) * (3 - len(grid))
        b = tuple(block) + (1,) * (3 - len(block))
        arr = (C.c_void_p * len(args))(*[C.cast(C.pointer(a), C.c_void_p) for a in args])
        check(lib.uc_launch(self.h, C.c_void_p(cu_function), *g, *b, smem, arr), "uc_launch")

    def group_start(self):
        check(lib.uc_group_start(self.h), "uc_group_start")

    def group_end(self):
        check(lib.uc_group_end(self.h), "uc_group_end")

    def put_signal(self, src: int, dst: SymMem, dst_off: int, nbytes: int, sig: Optional[SymMem], sig_idx: int,
                   sig_val: int, peer: int):
        check(lib.uc_put_signal(self.h, C.c_void_p(src), dst.h if dst else None, dst_off, nbytes,
                                sig.h if sig else None, sig_idx, sig_val, peer), "uc_put_signal")

    def signal_wait(self, dst: Optional[SymMem], dst_off: int, nbytes: int, sig: Optional[SymMem], sig_idx: int,
                    sig_val: int, peer: int):
        check(lib.uc_signal_wait(self.h, dst.h if dst else None, dst_off, nbytes, sig.h if sig else None, sig_idx,
                                 sig_val, peer), "uc_signal_wait")

    def p2p_bench(self, pattern: int, buf: SymMem, sig: SymMem, nbytes: int, iters: int, window: int = 1,
                  peer: int = 0, role: int = 0, blocks: int = 0):
        check(lib.uc_p2p_bench(self.h, pattern, buf.h, sig.h, nbytes, iters, window, peer, role, blocks),
              "uc_p2p_bench")

    def allreduce(self, send: int, recv: int, count: int, dtype: int, op: int = 0):
        check(lib.uc_allreduce(self.h, C.c_void_p(send), C.c_void_p(recv), count, dtype, op), "uc_allreduce")

    def reduce(self, send: int, recv: int, count: int, dtype: int, op: int, root: int):
        check(lib.uc_reduce(self.h, C.c_void_p(send), C.c_void_p(recv or None), count, dtype, op, root), "uc_reduce")

    def broadcast(self, buf: SymMem, off: int, nbytes: int, root: int):
        check(lib.uc_broadcast(self.h, buf.h, off, nbytes, root), "uc_broadcast")

    def allgather(self, send: int, recv: SymMem, recv_off: int, nbytes: int):
        check(lib.uc_allgather(self.h, C.c_void_p(send), recv.h, recv_off, nbytes), "uc_allgather")

    def allgatherv(self, send: int, nbytes: int, recv: SymMem, recv_off: int, counts, displs):
        n = len(counts)
        c_arr, d_arr = (C.c_size_t * n)(*counts), (C.c_size_t * n)(*displs)
        check(lib.uc_allgatherv(self.h, C.c_void_p(send), nbytes, recv.h, recv_off, c_arr, d_arr), "uc_allgatherv")

    def alltoall(self, send: int, recv: SymMem, recv_off: int, nbytes: int):
        check(lib.uc_alltoall(self.h, C.c_void_p(send), recv.h, recv_off, nbytes), "uc_alltoall")

    def gather(self, send: int, recv: SymMem, recv_off: int, nbytes: int, root: int):
        check(lib.uc_gather(self.h, C.c_void_p(send), recv.h, recv_off, nbytes, root), "uc_gather")

    def scatter(self, send: int, recv: SymMem, recv_off: int, nbytes: int, root: int):
        check(lib.uc_scatter(self.h, C.c_void_p(send or None), recv.h, recv_off, nbytes, root), "uc_scatter")

    def barrier(self):
        check(lib.uc_coord_barrier(self.h), "uc_coord_barrier")

    def allreduce_sum(self, send: int, recv: int, count: int, dtype: int):
        check(lib.uc_allreduce_sum(self.h, C.c_void_p(send), C.c_void_p(recv), count, dtype), "uc_allreduce_sum")

    def destroy(self):
        if self.h:
            check(lib.uc_coord_destroy(self.h), "uc_coord_destroy")
            self.h = None
            self._outputs.clear()


def builtin_kernel(name: str) -> int:
    p = C.c_void_p()
    check(lib.uc_builtin_kernel(name.encode(), C.byref(p)), "uc_builtin_kernel")
    return p.value


class CG:
    """The §VI-D Conjugate Gradient workload on the synthetic 3-D stencil matrix (uniconn.h)."""

    def __init__(self, comm: Comm, nx: int, ny: int, nz: int, stencil: int = 27, seed: int = 0xC6):
        h = C.c_void_p()
        check(lib.uc_cg_create(comm.h, nx, ny, nz, stencil, seed, C.byref(h)), "uc_cg_create")
        self.h, self.comm = h, comm
        n, nl, r0, nnz, it = (C.c_int64() for _ in range(5))
        check(lib.uc_cg_info(h, C.byref(n), C.byref(nl), C.byref(r0), C.byref(nnz), C.byref(it)), "uc_cg_info")
        self.N, self.n_local, self.row0, self.nnz_local = n.value, nl.value, r0.value, nnz.value

    def run(self, coord: Coord, iters: int, use_graph: bool = True,
            rr_out: Optional[np.ndarray] = None) -> np.ndarray:
        out = coord.keep(rr_out if rr_out is not None else np.zeros(iters, np.float64))
        check(lib.uc_cg_run(coord.h, self.h, iters, C.c_void_p(out.ctypes.data), int(use_graph)), "uc_cg_run")
        return out[:iters]

    def set_launch(self, lanes_per_row: int = 0, rows_in_flight: int = 0):
        check(lib.uc_cg_set_launch(self.h, lanes_per_row, rows_in_flight), "uc_cg_set_launch")

    def x(self, coord: Coord) -> np.ndarray:
        a = np.empty(self.n_local, np.float64)
        check(lib.uc_cg_copy_x(coord.h, self.h, C.c_void_p(a.ctypes.data)), "uc_cg_copy_x")
        return a

    def destroy(self):
        if self.h:
            check(lib.uc_cg_destroy(self.h), "uc_cg_destroy")
            self.h = None


class Jacobi:
    """The §VI-C Jacobi solver on this rank's slab (see uniconn.h for layout and semantics)."""

    def __init__(self, comm: Comm, nx: int, ny: int, seed: int = 0x5EED, zero_init: bool = False):
        h = C.c_void_p()
        check(lib.uc_jacobi_create(comm.h, nx, ny, seed, int(zero_init), C.byref(h)), "uc_jacobi_create")
        self.h, self.comm = h, comm
        a, n, b, r0, it = C.c_int(), C.c_int(), C.c_int(), C.c_int(), C.c_int64()
        check(lib.uc_jacobi_info(h, C.byref(a), C.byref(n), C.byref(b), C.byref(r0), C.byref(it)), "uc_jacobi_info")
        self.nx, self.n, self.ny, self.row0 = a.value, n.value, b.value, r0.value

    @property
    def iteration(self) -> int:
        it = C.c_int64()
        check(lib.uc_jacobi_info(self.h, None, None, None, None, C.byref(it)), "uc_jacobi_info")
        return it.value

    def step(self, coord: Coord, compute_norm: bool = False, norm_out: Optional[np.ndarray] = None):
        ptr = coord.keep(norm_out).ctypes.data if norm_out is not None else None
        check(lib.uc_jacobi_step(coord.h, self.h, int(compute_norm), C.c_void_p(ptr)), "uc_jacobi_step")

    def num_norms(self, iters: int, norm_every: int) -> int:
        return lib.uc_jacobi_num_norms(self.h, iters, norm_every)

    def run(self, coord: Coord, iters: int, norm_every: int = 0, use_graph: bool = True,
            norms_out: Optional[np.ndarray] = None) -> np.ndarray:
        cnt = self.num_norms(iters, norm_every)
        out = coord.keep(norms_out if norms_out is not None else np.zeros(cnt, np.float64))
        assert out.size >= cnt and out.dtype == np.float64
        check(lib.uc_jacobi_run(coord.h, self.h, iters, norm_every, C.c_void_p(out.ctypes.data if cnt else None),
                                int(use_graph)), "uc_jacobi_run")
        return out[:cnt]

    def copy_in(self, slab: np.ndarray):
        a = np.ascontiguousarray(slab, dtype=np.float32)
        assert a.shape == (self.n + 2, self.nx), a.shape
        check(lib.uc_jacobi_copy_in(self.h, C.c_void_p(a.ctypes.data)), "uc_jacobi_copy_in")

    def copy_out(self, coord: Optional[Coord] = None, which: int = 0) -> np.ndarray:
        a = np.empty((self.n + 2, self.nx), np.float32)
        check(lib.uc_jacobi_copy_out(coord.h if coord else None, self.h, C.c_void_p(a.ctypes.data), which),
              "uc_jacobi_copy_out")
        return a

    def copy_rows(self, coord: Optional[Coord], first_row: int, nrows: int) -> np.ndarray:
        a = np.empty((nrows, self.nx), np.float32)
        check(lib.uc_jacobi_copy_rows(coord.h if coord else None, self.h, first_row, nrows,
                                      C.c_void_p(a.ctypes.data)), "uc_jacobi_copy_rows")
        return a

    def copy_in_async(self, coord: Coord, host_ptr: int):
        check(lib.uc_jacobi_copy_in_async(coord.h, self.h, C.c_void_p(host_ptr)), "uc_jacobi_copy_in_async")

    def copy_out_async(self, coord: Coord, host_ptr: int):
        check(lib.uc_jacobi_copy_out_async(coord.h, self.h, C.c_void_p(host_ptr)), "uc_jacobi_copy_out_async")

    def set_launch(self, variant: int = -1, block_x: int = 0, blocks_per_sm: int = 0, stages: int = 0,
                   tile_rows: int = 0):
        """COLLECTIVE (see uc_jacobi_set_launch)."""
        check(lib.uc_jacobi_set_launch(self.h, variant, block_x, blocks_per_sm, stages, tile_rows),
              "uc_jacobi_set_launch")

    def solve(self, coord: Coord, max_iters: int, norm_every: int, tol: float):
        """uc_jacobi_solve: CPU-free convergence loop; returns (iterations run, last norm)."""
        it, nrm = C.c_int64(), C.c_double()
        check(lib.uc_jacobi_solve(coord.h, self.h, max_iters, norm_every, tol, C.byref(it), C.byref(nrm)),
              "uc_jacobi_solve")
        return it.value, nrm.value

    def set_host_path(self, deep_halo: bool = False, overlap: bool = False):
        """uc_jacobi_set_host_path (same call on every rank)."""
        check(lib.uc_jacobi_set_host_path(self.h, int(deep_halo), int(overlap)), "uc_jacobi_set_host_path")
        self.host_deep = bool(deep_halo)

    def set_balance(self, enable: bool):
        """uc_jacobi_set_balance: balanced chunks on (default) / off."""
        check(lib.uc_jacobi_set_balance(self.h, int(enable)), "uc_jacobi_set_balance")

    def balance_rates(self, coord, rates):
        """uc_jacobi_balance_rates: install the table for these per-block rates now."""
        import numpy as np
        r = np.ascontiguousarray(rates, np.float64)
        check(lib.uc_jacobi_balance_rates(coord.h, self.h, r.ctypes.data_as(C.POINTER(C.c_double)), len(r)),
              "uc_jacobi_balance_rates")

    def balance_table(self):
        """uc_jacobi_balance_table: [grid, 4] {strip, chunk, first row, last row}, or None (static)."""
        import numpy as np
        g = self.launch_info()["grid"]
        tab = np.zeros((g, 4), np.int32)
        n = C.c_int()
        check(lib.uc_jacobi_balance_table(self.h, tab.ctypes.data_as(C.POINTER(C.c_int)), g, C.byref(n)),
              "uc_jacobi_balance_table")
        return tab if n.value > 0 else None

    def plan(self, mode: int, iters: int, norm_every: int) -> list:
        """The launch plan uc_jacobi_run follows for this solver under a coordinator of `mode`."""
        info = self.launch_info()
        v = info["variant"]
        m = mode | (UC_PLAN_DEEP_HALO if mode == UC_MODE_HOST and getattr(self, "host_deep", False) else 0)
        return launch_plan(v, info["tile_rows"] if v == 5 else 1, m, self.n, iters, norm_every)

    def launch_counts(self) -> list:
        """uc_jacobi_launch_counts: completed launches by iterations per launch (index t = 1..8;
        0 = persistent launches), from device counters -- what really ran.  After Coord.sync."""
        buf = (C.c_uint64 * 16)()
        check(lib.uc_jacobi_launch_counts(self.h, buf, 16), "uc_jacobi_launch_counts")
        return list(buf)

    def launch_info(self) -> dict:
        v, g, b, s, c, st, tr = (C.c_int() for _ in range(7))
        check(lib.uc_jacobi_launch_info(self.h, C.byref(v), C.byref(g), C.byref(b), C.byref(s), C.byref(c),
                                        C.byref(st), C.byref(tr)), "uc_jacobi_launch_info")
        return {"variant": v.value, "grid": g.value, "block": b.value, "strips": s.value, "chunks": c.value,
                "stages": st.value, "tile_rows": tr.value}

    def destroy(self):
        if self.h:
            check(lib.uc_jacobi_destroy(self.h), "uc_jacobi_destroy")
            self.h = None
