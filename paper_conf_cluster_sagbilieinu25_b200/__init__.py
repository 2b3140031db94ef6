"""paper_conf_cluster_sagbilieinu25_b200 -- B200-native Jacobi halo/stencil hot path of UNICONN.

The product is ``libuniconn_b200.so`` (C-ABI in ``include/uniconn.h``; CUDA for sm_100a in
``csrc/``).  This package is its thin Python binding; importing it without the built library
raises ImportError -- there is no CPU or PyTorch fallback.
"""
from .uniconn import (UC_PUT_SM, UC_PUT_CE, UC_WAIT_KERNEL, UC_WAIT_STREAM, UC_PLAN_DEEP_HALO, UC_OK, UC_ERR_TIMEOUT, UC_ERR_STATE, UC_ERR_ARG, UC_F32, UC_F64, UC_MODE_DEVICE, UC_MODE_HOST, UC_MODE_PARTIAL,  # noqa: F401
                      UC_P2P_HALO, UC_P2P_PINGPONG, UC_P2P_WINDOW, UC_SUM, UC_PROD, UC_MIN, UC_MAX,
                      UC_TOPO_CHAIN, UC_TOPO_NONE, UC_TOPO_RING, UC_U64, CG, Comm, Coord, Env, Jacobi, SymMem,
                      ThreadAllgather, UCError, balance_plan, builtin_kernel, chain_neighbours, launch_plan,
                      ring_neighbours, torch_allgather)
from ._lib import EXPORTED, LIB_PATH, lib  # noqa: F401

__all__ = ["Env", "Comm", "SymMem", "Coord", "Jacobi", "CG", "ThreadAllgather", "torch_allgather", "UCError",
           "builtin_kernel", "ring_neighbours", "chain_neighbours", "launch_plan", "balance_plan", "lib", "LIB_PATH",
           "EXPORTED"]
