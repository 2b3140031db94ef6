"""User kernels on the header-only device API (include/uniconn_device.cuh) launched through
uc_launch: put-with-signal + wait in THREAD, WARP and BLOCK granularity,
around a ring of virtual ranks.  examples/device_api_ring.cu is the user code."""
import ctypes as C
import os

import numpy as np
import pytest

from vranks import run_ranks

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


class _CudaArray:
    def __init__(self, ptr, nbytes):
        self.__cuda_array_interface__ = {"shape": (nbytes // 4,), "typestr": "<f4", "data": (ptr, False),
                                         "version": 3, "strides": None}


@pytest.mark.parametrize("group", [0, 1, 2])
@pytest.mark.parametrize("P", [1, 2, 3])
def test_user_kernel_ring_put_signal(P, group):
    import torch

    import paper_conf_cluster_sagbilieinu25_b200 as U
    ex = C.CDLL(os.path.join(ROOT, "examples", "libuc_device_example.so"))
    ex.uc_example_ring_kernel.restype = C.c_void_p
    ex.uc_example_ring_kernel.argtypes = [C.c_int]
    n = 3000

    def body(rank, P, ag):
        fn = ex.uc_example_ring_kernel(group)
        assert fn
        env = U.Env(rank, P, 0, ag)
        comm = U.Comm(env, *U.ring_neighbours(rank, P))
        st = torch.cuda.Stream()
        co = U.Coord(comm, U.UC_MODE_DEVICE, st.cuda_stream)
        buf = U.SymMem(comm, n * 4)
        sig = U.SymMem(comm, 64)
        err = U.SymMem(comm, 64)  # any device word for the timeout flag
        try:
            with torch.cuda.stream(st):
                scratch = torch.empty(n, dtype=torch.float32, device="cuda")
            got = []
            for rnd in (1, 2):
                args = [C.c_void_p(scratch.data_ptr()), C.c_void_p(buf.ptr(comm.bottom)),
                        C.c_void_p(sig.ptr(comm.bottom)), C.c_void_p(sig.ptr()), C.c_int(n), C.c_int(rank),
                        C.c_uint64(rnd), C.c_ulonglong(10 ** 10), C.c_void_p(err.ptr())]
                co.launch(fn, (2,), (128,), 0, args)
                co.sync()
                with torch.cuda.stream(st):
                    got.append(torch.as_tensor(_CudaArray(buf.ptr(), n * 4), device="cuda").cpu().numpy().copy())
                comm.barrier()
            return got
        finally:
            comm.barrier()
            for m in (buf, sig, err):
                m.free()
            co.destroy()
            comm.destroy()
            env.finalize()

    res = run_ranks(P, body)
    for r in range(P):
        top = (r - 1) % P
        for i, rnd in enumerate((1, 2)):
            want = (top * 1000 + rnd) + 0.5 * np.arange(n, dtype=np.float32)
            assert np.array_equal(res[r][i], want.astype(np.float32)), (r, rnd)
