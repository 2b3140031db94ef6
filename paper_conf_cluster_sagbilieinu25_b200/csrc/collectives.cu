// collectives.cu -- the rest of the paper's collective interface (Listing 7, P:291-314;
// SURVEY §8 f4): Reduce, Broadcast, AllGather(v) (the CG exchange), AlltoAll, Gather,
// Scatter and a stream-ordered device Barrier, plus reduction operators for AllReduce/Reduce
// (ReductionOperator).
//
// Host and partial modes map onto NCCL on the coordinator's stream -- directly where NCCL has
// the collective, as grouped send/recv where it does not (the paper's NCCL backend does the
// same).  Device mode is one-sided over the symmetric heap (the paper's NVSHMEM backend
// emulates missing collectives with puts + barriers): three stream-ordered steps --
//   1. ready:  every rank release-stores "epoch e reached" into every peer's ready[rank] flag and
//              waits for all P ready flags (every rank's earlier stream work on the buffers is
//              done: no write-after-read on the destination);
//   2. copy:   SM stores of every outgoing chunk straight into the destination ranks' buffers
//              (multi-block, 16-byte vectors);
//   3. done:   fence.sys, release "epoch e delivered" into the done[rank] flag of every rank this
//              rank wrote to; wait for the done flags of every rank this rank receives from.
// Epochs are per coordinator and advance by one per collective call, so all ranks must call the
// collectives in the same order (MPI / NCCL semantics).
#include <cstring>

#include "device_api.cuh"
#include "uc_internal.h"

namespace uc {
using namespace dev;

struct CollSeg {
  const char* src;
  char* dst;
  size_t bytes;
};
struct CollCopy {
  CollSeg seg[UC_MAX_RANKS];
  int nseg;
};

__global__ void coll_copy_kernel(CollCopy c) {
  const size_t tid = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  for (int s = 0; s < c.nseg; ++s) {
    const CollSeg g = c.seg[s];
    if ((((uintptr_t)g.src | (uintptr_t)g.dst) & 15) == 0) {
      const size_t n16 = g.bytes / 16;
      const uint4* src = reinterpret_cast<const uint4*>(g.src);
      uint4* dst = reinterpret_cast<uint4*>(g.dst);
      for (size_t i = tid; i < n16; i += stride) dst[i] = src[i];
      for (size_t i = n16 * 16 + tid; i < g.bytes; i += stride) g.dst[i] = g.src[i];
    } else {
      for (size_t i = tid; i < g.bytes; i += stride) g.dst[i] = g.src[i];
    }
  }
}

struct CollFlags {
  uint64_t* peer[UC_MAX_RANKS];  // peer q's flag array ([ready P][done P], kFlagStride each)
  uint64_t* mine;
  int rank, size;
  unsigned notify, wait;  // rank bitmasks
  int done_phase;         // 0: ready flags, 1: done flags
  uint64_t epoch;
  unsigned long long timeout_ns;
  unsigned int* err;
};

__global__ void coll_flags_kernel(CollFlags f) {
  if (threadIdx.x != 0) return;
  const size_t base = (size_t)f.done_phase * f.size;
  if (f.done_phase) __threadfence_system();  // the copy kernel's peer stores before the signal
  for (int q = 0; q < f.size; ++q)
    if (f.notify >> q & 1u) st_release_sys(f.peer[q] + (base + f.rank) * kFlagStride, f.epoch);
  for (int q = 0; q < f.size; ++q)
    if (f.wait >> q & 1u) wait_ge(f.mine + (base + q) * kFlagStride, f.epoch, f.timeout_ns, f.err);
}

namespace {

int flags_launch(uc_coord* k, int done_phase, unsigned notify, unsigned wait, uint64_t epoch) {
  const uc_comm* c = k->comm;
  CollFlags f{};
  for (int q = 0; q < c->size; ++q) f.peer[q] = (uint64_t*)uc_mem_ptr(k->coll_flags, q);
  f.mine = (uint64_t*)k->coll_flags->local;
  f.rank = c->rank;
  f.size = c->size;
  f.notify = notify;
  f.wait = wait;
  f.done_phase = done_phase;
  f.epoch = epoch;
  f.timeout_ns = k->timeout_ns;
  f.err = k->err;
  coll_flags_kernel<<<1, 32, 0, k->stream>>>(f);
  UC_CUDA(cudaGetLastError());
  return UC_OK;
}

int copy_launch(uc_coord* k, const CollCopy& cp) {
  size_t total = 0;
  for (int s = 0; s < cp.nseg; ++s) total += cp.seg[s].bytes;
  if (total == 0) return UC_OK;
  size_t blocks = total / 65536;
  if (blocks < 1) blocks = 1;
  if (blocks > 296) blocks = 296;
  coll_copy_kernel<<<(unsigned)blocks, 256, 0, k->stream>>>(cp);
  UC_CUDA(cudaGetLastError());
  return UC_OK;
}

// ready -> copy -> done, as described at the top of the file
int device_collective(uc_coord* k, const CollCopy& cp, unsigned notify, unsigned wait) {
  const unsigned all = (1u << k->comm->size) - 1u;
  const uint64_t epoch = ++k->coll_epoch;
  UC_TRY(flags_launch(k, 0, all, all, epoch));
  UC_TRY(copy_launch(k, cp));
  return flags_launch(k, 1, notify, wait, epoch);
}

ncclDataType_t nccl_type(uc_dtype dt) {
  return dt == UC_F32 ? ncclFloat32 : dt == UC_F64 ? ncclFloat64 : ncclUint64;
}
ncclRedOp_t nccl_op(uc_redop op) {
  return op == UC_PROD ? ncclProd : op == UC_MIN ? ncclMin : op == UC_MAX ? ncclMax : ncclSum;
}

int check_coord(uc_coord* k, uc_mem* m, size_t off, size_t bytes_needed) {
  if (!k) return fail(UC_ERR_ARG, "coord is NULL");
  if (k->in_group) return fail(UC_ERR_STATE, "collectives cannot be placed inside uc_group_start/end");
  UC_CUDA(cudaSetDevice(k->comm->env->device));
  if (m && off + bytes_needed > m->bytes)
    return fail(UC_ERR_ARG, "collective needs %zu bytes at offset %zu of a %zu-byte buffer", bytes_needed, off,
                m->bytes);
  if (k->mode != UC_MODE_DEVICE) return ensure_nccl(k);
  return UC_OK;
}

char* at(uc_mem* m, int rank, size_t off) { return (char*)uc_mem_ptr(m, rank) + off; }

}  // namespace
}  // namespace uc

using namespace uc;

extern "C" {

int uc_reduce(uc_coord* k, const void* send, void* recv, size_t count, uc_dtype dt, uc_redop op, int root) {
  UC_TRY(check_coord(k, nullptr, 0, 0));
  const uc_comm* c = k->comm;
  if (root < 0 || root >= c->size) return fail(UC_ERR_ARG, "root %d out of range", root);
  if (!send || (c->rank == root && !recv)) return fail(UC_ERR_ARG, "NULL buffer");
  if (op < UC_SUM || op > UC_MAX) return fail(UC_ERR_ARG, "unknown reduction op %d", (int)op);
  if (count == 0) return UC_OK;
  if (k->mode != UC_MODE_DEVICE) {
    UC_NCCL(ncclReduce(send, recv, count, nccl_type(dt), nccl_op(op), root, k->nccl, k->stream));
    return UC_OK;
  }
  // the ready round orders this one-shot after every rank's previous use of the slots
  const unsigned all = (1u << c->size) - 1u;
  UC_TRY(flags_launch(k, 0, all, all, ++k->coll_epoch));
  return oneshot_reduce(k, send, recv, count, dt, op, root);
}

int uc_allreduce(uc_coord* k, const void* send, void* recv, size_t count, uc_dtype dt, uc_redop op) {
  UC_TRY(check_coord(k, nullptr, 0, 0));
  if (!send || !recv) return fail(UC_ERR_ARG, "NULL buffer");
  if (op < UC_SUM || op > UC_MAX) return fail(UC_ERR_ARG, "unknown reduction op %d", (int)op);
  if (count == 0) return UC_OK;
  if (k->mode != UC_MODE_DEVICE) {
    UC_NCCL(ncclAllReduce(send, recv, count, nccl_type(dt), nccl_op(op), k->nccl, k->stream));
    return UC_OK;
  }
  return oneshot_reduce(k, send, recv, count, dt, op, -1);
}

int uc_broadcast(uc_coord* k, uc_mem* buf, size_t off, size_t bytes, int root) {
  if (!buf) return fail(UC_ERR_ARG, "buf is NULL");
  UC_TRY(check_coord(k, buf, off, bytes));
  const uc_comm* c = k->comm;
  if (root < 0 || root >= c->size) return fail(UC_ERR_ARG, "root %d out of range", root);
  if (bytes == 0) return UC_OK;
  if (k->mode != UC_MODE_DEVICE) {
    char* p = at(buf, c->rank, off);
    UC_NCCL(ncclBroadcast(p, p, bytes, ncclUint8, root, k->nccl, k->stream));
    return UC_OK;
  }
  CollCopy cp{};
  if (c->rank == root)
    for (int q = 0; q < c->size; ++q)
      if (q != root) cp.seg[cp.nseg++] = {at(buf, root, off), at(buf, q, off), bytes};
  const unsigned others = ((1u << c->size) - 1u) & ~(1u << root);
  return device_collective(k, cp, c->rank == root ? others : 0u, c->rank == root ? 0u : (1u << root));
}

int uc_allgatherv(uc_coord* k, const void* send, size_t bytes, uc_mem* recv, size_t recv_off, const size_t* counts,
                  const size_t* displs) {
  if (!recv || !counts || !displs) return fail(UC_ERR_ARG, "NULL argument");
  const uc_comm* c = k ? k->comm : nullptr;
  if (!c) return fail(UC_ERR_ARG, "coord is NULL");
  size_t need = 0;
  for (int q = 0; q < c->size; ++q) need = std::max(need, displs[q] + counts[q]);
  UC_TRY(check_coord(k, recv, recv_off, need));
  if (counts[c->rank] != bytes) return fail(UC_ERR_ARG, "counts[rank] must equal the bytes this rank sends");
  if (bytes && !send) return fail(UC_ERR_ARG, "send is NULL");
  if (k->mode != UC_MODE_DEVICE) {
    UC_NCCL(ncclGroupStart());
    for (int q = 0; q < c->size; ++q) {
      if (bytes) UC_NCCL(ncclSend(send, bytes, ncclUint8, q, k->nccl, k->stream));
      if (counts[q]) UC_NCCL(ncclRecv(at(recv, c->rank, recv_off + displs[q]), counts[q], ncclUint8, q, k->nccl,
                                      k->stream));
    }
    UC_NCCL(ncclGroupEnd());
    return UC_OK;
  }
  CollCopy cp{};
  for (int q = 0; q < c->size; ++q)
    if (bytes) cp.seg[cp.nseg++] = {(const char*)send, at(recv, q, recv_off + displs[c->rank]), bytes};
  const unsigned all = (1u << c->size) - 1u;
  return device_collective(k, cp, all, all);
}

int uc_allgather(uc_coord* k, const void* send, uc_mem* recv, size_t recv_off, size_t bytes) {
  if (!k) return fail(UC_ERR_ARG, "coord is NULL");
  const int P = k->comm->size;
  if (k->mode != UC_MODE_DEVICE && recv) {
    UC_TRY(check_coord(k, recv, recv_off, bytes * P));
    if (bytes == 0) return UC_OK;
    UC_NCCL(ncclAllGather(send, at(recv, k->comm->rank, recv_off), bytes, ncclUint8, k->nccl, k->stream));
    return UC_OK;
  }
  size_t counts[UC_MAX_RANKS], displs[UC_MAX_RANKS];
  for (int q = 0; q < P; ++q) {
    counts[q] = bytes;
    displs[q] = (size_t)q * bytes;
  }
  return uc_allgatherv(k, send, bytes, recv, recv_off, counts, displs);
}

int uc_alltoall(uc_coord* k, const void* send, uc_mem* recv, size_t recv_off, size_t bytes) {
  if (!recv) return fail(UC_ERR_ARG, "recv is NULL");
  if (!k) return fail(UC_ERR_ARG, "coord is NULL");
  const uc_comm* c = k->comm;
  UC_TRY(check_coord(k, recv, recv_off, bytes * c->size));
  if (bytes == 0) return UC_OK;
  if (!send) return fail(UC_ERR_ARG, "send is NULL");
  const char* s = (const char*)send;
  if (k->mode != UC_MODE_DEVICE) {
    UC_NCCL(ncclGroupStart());
    for (int q = 0; q < c->size; ++q) {
      UC_NCCL(ncclSend(s + (size_t)q * bytes, bytes, ncclUint8, q, k->nccl, k->stream));
      UC_NCCL(ncclRecv(at(recv, c->rank, recv_off + (size_t)q * bytes), bytes, ncclUint8, q, k->nccl, k->stream));
    }
    UC_NCCL(ncclGroupEnd());
    return UC_OK;
  }
  CollCopy cp{};
  for (int q = 0; q < c->size; ++q)
    cp.seg[cp.nseg++] = {s + (size_t)q * bytes, at(recv, q, recv_off + (size_t)c->rank * bytes), bytes};
  const unsigned all = (1u << c->size) - 1u;
  return device_collective(k, cp, all, all);
}

int uc_gather(uc_coord* k, const void* send, uc_mem* recv, size_t recv_off, size_t bytes, int root) {
  if (!recv) return fail(UC_ERR_ARG, "recv is NULL");
  if (!k) return fail(UC_ERR_ARG, "coord is NULL");
  const uc_comm* c = k->comm;
  if (root < 0 || root >= c->size) return fail(UC_ERR_ARG, "root %d out of range", root);
  UC_TRY(check_coord(k, recv, recv_off, bytes * c->size));
  if (bytes == 0) return UC_OK;
  if (!send) return fail(UC_ERR_ARG, "send is NULL");
  if (k->mode != UC_MODE_DEVICE) {
    UC_NCCL(ncclGroupStart());
    UC_NCCL(ncclSend(send, bytes, ncclUint8, root, k->nccl, k->stream));
    if (c->rank == root)
      for (int q = 0; q < c->size; ++q)
        UC_NCCL(ncclRecv(at(recv, root, recv_off + (size_t)q * bytes), bytes, ncclUint8, q, k->nccl, k->stream));
    UC_NCCL(ncclGroupEnd());
    return UC_OK;
  }
  CollCopy cp{};
  cp.seg[cp.nseg++] = {(const char*)send, at(recv, root, recv_off + (size_t)c->rank * bytes), bytes};
  const unsigned all = (1u << c->size) - 1u;
  return device_collective(k, cp, 1u << root, c->rank == root ? all : 0u);
}

int uc_scatter(uc_coord* k, const void* send, uc_mem* recv, size_t recv_off, size_t bytes, int root) {
  if (!recv) return fail(UC_ERR_ARG, "recv is NULL");
  if (!k) return fail(UC_ERR_ARG, "coord is NULL");
  const uc_comm* c = k->comm;
  if (root < 0 || root >= c->size) return fail(UC_ERR_ARG, "root %d out of range", root);
  UC_TRY(check_coord(k, recv, recv_off, bytes));
  if (bytes == 0) return UC_OK;
  if (c->rank == root && !send) return fail(UC_ERR_ARG, "send is NULL on the root");
  const char* s = (const char*)send;
  if (k->mode != UC_MODE_DEVICE) {
    UC_NCCL(ncclGroupStart());
    if (c->rank == root)
      for (int q = 0; q < c->size; ++q)
        UC_NCCL(ncclSend(s + (size_t)q * bytes, bytes, ncclUint8, q, k->nccl, k->stream));
    UC_NCCL(ncclRecv(at(recv, c->rank, recv_off), bytes, ncclUint8, root, k->nccl, k->stream));
    UC_NCCL(ncclGroupEnd());
    return UC_OK;
  }
  CollCopy cp{};
  if (c->rank == root)
    for (int q = 0; q < c->size; ++q) cp.seg[cp.nseg++] = {s + (size_t)q * bytes, at(recv, q, recv_off), bytes};
  const unsigned all = (1u << c->size) - 1u;
  return device_collective(k, cp, c->rank == root ? all : 0u, 1u << root);
}

int uc_coord_barrier(uc_coord* k) {
  UC_TRY(check_coord(k, nullptr, 0, 0));
  if (k->mode != UC_MODE_DEVICE) {
    UC_NCCL(ncclAllReduce(k->nccl_scratch, k->nccl_scratch, 1, ncclFloat32, ncclSum, k->nccl, k->stream));
    return UC_OK;
  }
  const unsigned all = (1u << k->comm->size) - 1u;
  return flags_launch(k, 0, all, all, ++k->coll_epoch);
}

}  // extern "C"
