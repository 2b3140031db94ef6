/* nccl_dev_jacobi.h -- in-box "native" comparator for the Jacobi halo path: the
 * paper's Listing 3 (the native NVSHMEM device-initiated Jacobi: dedicated
 * boundary blocks compute the first/last rows, put them into the neighbours' halos and
 * synchronise, the other blocks compute the interior) written against NCCL 2.28's device API
 * instead of NVSHMEM: the halo rows are stored through LSA (load/store accessible) peer pointers
 * of an NCCL symmetric window (ncclGetLsaPointer) and each boundary block ends with an LSA
 * barrier across the ranks (ncclLsaBarrierSession::sync, release/acquire).  One Jacobi iteration
 * per launch, one float4 column per thread, no TMA, no temporal blocking: the paper's structure
 * on NCCL's device API.  It is a comparison point, not the product (libuniconn_b200.so); it
 * shares no code with it, and is checked bit for bit against the oracle (tests/test_gpu_native.py).
 *
 * Layout: one symmetric window per rank holding two slabs (ping-pong) of (n+2) x nx fp32, row 0 =
 * halo from top, rows 1..n owned, row n+1 = halo from bottom (reading G9); columns 0 and
 * nx-1 fixed (reading G2); update 0.25f*((l+r)+(t+b)) in IEEE fp32, no FMA (reading G1).
 * Topology: top/bottom are world ranks or -1 (fixed halo row).
 *
 * Every function returns 0 on success, else a positive code; ucn_last_error() has the message.
 * Errors: 1 = bad argument, 2 = CUDA error, 3 = NCCL error.  Handles are opaque.
 */
#ifndef UC_NCCL_DEV_JACOBI_H
#define UC_NCCL_DEV_JACOBI_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct ucn_jacobi ucn_jacobi;

/* NCCL's unique id (128 bytes, ncclUniqueId) for rank 0 to broadcast; out: 128 bytes, caller-owned. */
int ucn_unique_id(void* out);
/* COLLECTIVE over nranks processes (one GPU each, the current device): ncclCommInitRank, ncclMemAlloc
 * of the two slabs, ncclCommWindowRegister (NCCL_WIN_COLL_SYMMETRIC), ncclDevCommCreate with one
 * LSA barrier per column strip.  nx % 4 == 0, nx >= 8, n >= 1. */
int ucn_create(int rank, int nranks, const void* unique_id, int nx, int n, int top, int bottom, ucn_jacobi** out);
/* host_slab: (n+2) x nx floats (halo rows included), copied into both slabs (synchronous). */
int ucn_copy_in(ucn_jacobi* J, const float* host_slab);
/* host_slab: (n+2) x nx floats of the current iterate (synchronous). */
int ucn_copy_out(ucn_jacobi* J, float* host_slab);
/* Enqueue `iters` iterations (one launch each) on `stream` (a cudaStream_t; NULL = default). */
int ucn_run(ucn_jacobi* J, int iters, void* stream);
/* COLLECTIVE: deregister the window, free the slabs, destroy the device and host communicators. */
int ucn_destroy(ucn_jacobi* J);
const char* ucn_last_error(void);

#ifdef __cplusplus
}
#endif
#endif
