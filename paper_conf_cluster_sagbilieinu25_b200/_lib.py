"""ctypes declarations of libuniconn_b200.so (include/uniconn.h).  Argument marshalling only.

The library is the product: there is no Python or CPU fallback.  If the shared library is
missing this module raises ImportError (build it with ``python -m
paper_conf_cluster_sagbilieinu25_b200/build.py`` or ``__graft_entry__.build()``).
"""
from __future__ import annotations

import ctypes as C
import os

_PKG = os.path.dirname(os.path.abspath(__file__))
# UC_LIB_PATH selects an A/B build of the same CUDA sources (build.py --define ... --out ...).
LIB_PATH = os.environ.get("UC_LIB_PATH") or os.path.join(_PKG, "libuniconn_b200.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is missing: run `python paper_conf_cluster_sagbilieinu25_b200/build.py` "
                      "(the CUDA path has no fallback)")

lib = C.CDLL(LIB_PATH, mode=C.RTLD_GLOBAL)

# enums (uniconn.h)
UC_OK, UC_ERR_ARG, UC_ERR_CUDA, UC_ERR_NCCL, UC_ERR_BOOTSTRAP, UC_ERR_TIMEOUT, UC_ERR_STATE, \
    UC_ERR_UNSUPPORTED, UC_ERR_OOM = range(9)
UC_MODE_HOST, UC_MODE_DEVICE, UC_MODE_PARTIAL = 0, 1, 2
UC_F32, UC_F64, UC_U64 = 0, 1, 2
UC_TOPO_NONE, UC_TOPO_RING, UC_TOPO_CHAIN = 0, 1, 2
UC_P2P_PINGPONG, UC_P2P_WINDOW, UC_P2P_HALO = 0, 1, 2
UC_SUM, UC_PROD, UC_MIN, UC_MAX = 0, 1, 2, 3
UC_MAX_RANKS = 8
UC_PLAN_DEEP_HALO = 0x100
UC_PUT_SM, UC_PUT_CE = 0, 1
UC_WAIT_KERNEL, UC_WAIT_STREAM = 0, 1

ALLGATHER_FN = C.CFUNCTYPE(C.c_int, C.c_void_p, C.c_void_p, C.c_size_t, C.c_void_p)

vp, i32, u64, i64, sz, dp = C.c_void_p, C.c_int, C.c_uint64, C.c_int64, C.c_size_t, C.POINTER(C.c_double)
P = C.POINTER

_SIGS = {
    "uc_env_init": (i32, [i32, i32, i32, ALLGATHER_FN, vp, P(vp)]),
    "uc_env_finalize": (i32, [vp]),
    "uc_env_info": (i32, [vp, P(i32), P(i32), P(i32)]),
    "uc_comm_create": (i32, [vp, i32, i32, P(vp)]),
    "uc_comm_destroy": (i32, [vp]),
    "uc_comm_info": (i32, [vp, P(i32), P(i32), P(i32), P(i32), P(i32)]),
    "uc_comm_device_view": (i32, [vp, P(vp)]),
    "uc_comm_barrier": (i32, [vp, vp]),
    "uc_mem_alloc_symmetric": (i32, [vp, sz, P(vp)]),
    "uc_mem_ptr": (vp, [vp, i32]),
    "uc_mem_size": (sz, [vp]),
    "uc_mem_free_symmetric": (i32, [vp]),
    "uc_coord_create": (i32, [vp, i32, vp, P(vp)]),
    "uc_coord_destroy": (i32, [vp]),
    "uc_coord_sync": (i32, [vp]),
    "uc_coord_set_timeout": (i32, [vp, u64]),
    "uc_launch": (i32, [vp, vp, C.c_uint, C.c_uint, C.c_uint, C.c_uint, C.c_uint, C.c_uint, sz, P(vp)]),
    "uc_builtin_kernel": (i32, [C.c_char_p, P(vp)]),
    "uc_group_start": (i32, [vp]),
    "uc_group_end": (i32, [vp]),
    "uc_put_signal": (i32, [vp, vp, vp, sz, sz, vp, sz, u64, i32]),
    "uc_signal_wait": (i32, [vp, vp, sz, sz, vp, sz, u64, i32]),
    "uc_allreduce_sum": (i32, [vp, vp, vp, sz, i32]),
    "uc_p2p_bench": (i32, [vp, i32, vp, vp, sz, i32, i32, i32, i32, i32]),
    "uc_allreduce": (i32, [vp, vp, vp, sz, i32, i32]),
    "uc_reduce": (i32, [vp, vp, vp, sz, i32, i32, i32]),
    "uc_broadcast": (i32, [vp, vp, sz, sz, i32]),
    "uc_allgather": (i32, [vp, vp, vp, sz, sz]),
    "uc_allgatherv": (i32, [vp, vp, sz, vp, sz, P(sz), P(sz)]),
    "uc_alltoall": (i32, [vp, vp, vp, sz, sz]),
    "uc_gather": (i32, [vp, vp, vp, sz, sz, i32]),
    "uc_scatter": (i32, [vp, vp, vp, sz, sz, i32]),
    "uc_coord_barrier": (i32, [vp]),
    "uc_cg_create": (i32, [vp, i32, i32, i32, i32, u64, P(vp)]),
    "uc_cg_run": (i32, [vp, vp, i32, vp, i32]),
    "uc_cg_copy_x": (i32, [vp, vp, vp]),
    "uc_cg_info": (i32, [vp, P(i64), P(i64), P(i64), P(i64), P(i64)]),
    "uc_cg_destroy": (i32, [vp]),
    "uc_cg_set_launch": (i32, [vp, i32, i32]),
    "uc_jacobi_create": (i32, [vp, i32, i32, u64, i32, P(vp)]),
    "uc_jacobi_step": (i32, [vp, vp, i32, vp]),
    "uc_jacobi_run": (i32, [vp, vp, i32, i32, vp, i32]),
    "uc_jacobi_num_norms": (i32, [vp, i32, i32]),
    "uc_jacobi_launch_counts": (i32, [vp, P(u64), i32]),
    "uc_jacobi_set_host_path": (i32, [vp, i32, i32]),
    "uc_jacobi_set_balance": (i32, [vp, i32]),
    "uc_jacobi_balance_rates": (i32, [vp, vp, dp, i32]),
    "uc_jacobi_balance_table": (i32, [vp, P(i32), i32, P(i32)]),
    "uc_balance_plan": (i32, [i32, i32, i32, i32, i32, dp, P(i32)]),
    "uc_jacobi_solve": (i32, [vp, vp, i32, i32, C.c_double, P(i64), dp]),
    "uc_coord_set_p2p_path": (i32, [vp, i32, i32]),
    "uc_jacobi_launch_plan": (i32, [i32, i32, i32, i32, i32, i32, P(i32), i32]),
    "uc_jacobi_copy_in": (i32, [vp, vp]),
    "uc_jacobi_copy_out": (i32, [vp, vp, vp, i32]),
    "uc_jacobi_copy_in_async": (i32, [vp, vp, vp]),
    "uc_jacobi_copy_rows": (i32, [vp, vp, i32, i32, vp]),
    "uc_jacobi_copy_out_async": (i32, [vp, vp, vp]),
    "uc_jacobi_info": (i32, [vp, P(i32), P(i32), P(i32), P(i32), P(i64)]),
    "uc_jacobi_destroy": (i32, [vp]),
    "uc_jacobi_set_launch": (i32, [vp, i32, i32, i32, i32, i32]),
    "uc_jacobi_launch_info": (i32, [vp, P(i32), P(i32), P(i32), P(i32), P(i32), P(i32), P(i32)]),
    "uc_last_error": (C.c_char_p, []),
    "uc_status_string": (C.c_char_p, [i32]),
    "uc_version": (i32, []),
}

for _name, (_res, _args) in _SIGS.items():
    _f = getattr(lib, _name)
    _f.restype = _res
    _f.argtypes = _args

EXPORTED = tuple(_SIGS)


class UCError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        msg = lib.uc_last_error().decode(errors="replace")
        super().__init__(f"{where}: {lib.uc_status_string(status).decode()} -- {msg}")


def check(status: int, where: str) -> None:
    if status != UC_OK:
        raise UCError(status, where)
