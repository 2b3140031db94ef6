/*
 * uniconn_device.cuh -- header-only device API of libuniconn_b200 for user kernels.
 *
 * The paper inlines its device API in headers and compiles it with the application;
 * primitives come in THREAD, WARP and BLOCK granularity (ThreadGroup) and follow the
 * one-sided Post/Acknowledge semantics: a put of data into a peer's symmetric buffer
 * followed by an atomic signal update, and a wait on a local signal.
 *
 * Peer addresses come from the host: uc_mem_ptr(mem, peer) (CUDA IPC or in-process peer
 * pointers over NVLink / NVSwitch); the communicator's {rank, size, top, bottom} from
 * uc_comm_device_view.  Launch user kernels with uc_launch (or any CUDA launch on the
 * coordinator's stream).  All signals are 64-bit, system scope (the peer is another GPU).
 *
 *   uc_dev_put<G>(dst, src, bytes)                 cooperative copy by the group G
 *   uc_dev_put_signal<G>(dst, src, bytes, sig, v, op)   copy, group sync, one thread signals
 *   uc_dev_signal(sig, v, op)                      UC_DEV_SIGNAL_SET: release-store v;
 *                                                  UC_DEV_SIGNAL_ADD: release atomic add v
 *   uc_dev_wait_ge(sig, v, timeout_ns, err)        spin until *sig >= v (acquire), bounded
 *   uc_dev_fence()                                 order all prior stores before later ones
 *                                                  at system scope (nvshmem_fence analogue)
 */
#ifndef UNICONN_DEVICE_CUH
#define UNICONN_DEVICE_CUH

#include <stddef.h>
#include <stdint.h>

enum uc_dev_group { UC_DEV_THREAD = 0, UC_DEV_WARP = 1, UC_DEV_BLOCK = 2 };
enum uc_dev_signal_op { UC_DEV_SIGNAL_SET = 0, UC_DEV_SIGNAL_ADD = 1 };

static __device__ __forceinline__ unsigned long long uc_dev_globaltimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

static __device__ __forceinline__ uint64_t uc_dev_ld_acquire(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

static __device__ __forceinline__ uint64_t uc_dev_ld_relaxed(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.relaxed.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

static __device__ __forceinline__ void uc_dev_fence() { asm volatile("fence.sc.sys;" ::: "memory"); }

static __device__ __forceinline__ void uc_dev_signal(uint64_t* sig, uint64_t v, int op = UC_DEV_SIGNAL_SET) {
  if (op == UC_DEV_SIGNAL_ADD)
    asm volatile("red.release.sys.global.add.u64 [%0], %1;" ::"l"(sig), "l"(v) : "memory");
  else
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(sig), "l"(v) : "memory");
}

/* Acknowledge for one thread: spin until *sig >= v (monotone signals), then acquire.  Gives up
 * after timeout_ns, or at once when *err is already non-zero; sets bit 0 of *err on timeout and
 * returns false. */
static __device__ __forceinline__ bool uc_dev_wait_ge(const uint64_t* sig, uint64_t v, unsigned long long timeout_ns,
                                                      unsigned int* err) {
  if (uc_dev_ld_acquire(sig) >= v) return true;
  const unsigned long long t0 = uc_dev_globaltimer();
  unsigned ns = 32;
  while (uc_dev_ld_relaxed(sig) < v) {  // relaxed polls: no L1 invalidation per poll
    if (uc_dev_globaltimer() - t0 > timeout_ns || *(volatile unsigned int*)err) {
      atomicOr(err, 1u);
      return false;
    }
    __nanosleep(ns);
    if (ns < 256) ns <<= 1;
  }
  asm volatile("fence.acq_rel.sys;" ::: "memory");  // the observing load + fence = acquire
  return true;
}

/* rank of the calling thread inside its group, and the group's size (1-D blocks) */
template <int G>
static __device__ __forceinline__ unsigned uc_dev_group_rank() {
  return G == UC_DEV_THREAD ? 0u : G == UC_DEV_WARP ? (threadIdx.x & 31u) : threadIdx.x;
}
template <int G>
static __device__ __forceinline__ unsigned uc_dev_group_size() {
  return G == UC_DEV_THREAD ? 1u : G == UC_DEV_WARP ? 32u : blockDim.x;
}
template <int G>
static __device__ __forceinline__ void uc_dev_group_sync() {
  if (G == UC_DEV_WARP) __syncwarp();
  if (G == UC_DEV_BLOCK) __syncthreads();
}

/* Cooperative copy of `bytes` by every thread of the group (16-byte vectors when both
 * addresses are 16-byte aligned).  dst may be a peer's symmetric address. */
template <int G>
static __device__ __forceinline__ void uc_dev_put(void* dst, const void* src, size_t bytes) {
  const unsigned r = uc_dev_group_rank<G>(), n = uc_dev_group_size<G>();
  if ((((uintptr_t)dst | (uintptr_t)src) & 15u) == 0) {
    const size_t n16 = bytes / 16;
    uint4* d = reinterpret_cast<uint4*>(dst);
    const uint4* s = reinterpret_cast<const uint4*>(src);
    for (size_t i = r; i < n16; i += n) d[i] = s[i];
    for (size_t i = n16 * 16 + r; i < bytes; i += n) static_cast<char*>(dst)[i] = static_cast<const char*>(src)[i];
  } else {
    for (size_t i = r; i < bytes; i += n) static_cast<char*>(dst)[i] = static_cast<const char*>(src)[i];
  }
}

/* Post (put with signal): the group copies, synchronises, and its first thread
 * fences at system scope and updates the peer's signal. */
template <int G>
static __device__ __forceinline__ void uc_dev_put_signal(void* dst, const void* src, size_t bytes, uint64_t* sig,
                                                         uint64_t v, int op = UC_DEV_SIGNAL_SET) {
  uc_dev_put<G>(dst, src, bytes);
  uc_dev_group_sync<G>();
  if (uc_dev_group_rank<G>() == 0) {
    __threadfence_system();
    uc_dev_signal(sig, v, op);
  }
}

#endif /* UNICONN_DEVICE_CUH */
