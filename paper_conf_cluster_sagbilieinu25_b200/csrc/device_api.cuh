// device_api.cuh -- header-only device primitives of libuniconn_b200 (the paper inlines its
// device API in headers).  System-scope (.sys) release/acquire because the peer is
// another GPU reached over NVLink (reading G10); a bounded spin turns a hang into an error.
#pragma once
#include <cstdint>

namespace uc {
namespace dev {

__device__ __forceinline__ unsigned long long globaltimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

__device__ __forceinline__ uint64_t ld_acquire_sys(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

__device__ __forceinline__ void st_release_sys(uint64_t* p, uint64_t v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ void st_relaxed_sys_f64(double* p, double v) {
  asm volatile("st.relaxed.sys.global.f64 [%0], %1;" ::"l"(p), "d"(v) : "memory");
}

__device__ __forceinline__ double ld_relaxed_sys_f64(const double* p) {
  double v;
  asm volatile("ld.relaxed.sys.global.f64 %0, [%1];" : "=d"(v) : "l"(p) : "memory");
  return v;
}

// Acknowledge / nvshmem_signal_wait_until(GE) for one thread.  Returns false on timeout (and
// sets bit 0 of *err).  Monotone ">=" instead of the listing's "==": a neighbour one
// iteration ahead must not hang us (reading G10).
__device__ __forceinline__ bool wait_ge(const uint64_t* flag, uint64_t v, unsigned long long timeout_ns,
                                        unsigned int* err) {
  if (ld_acquire_sys(flag) >= v) return true;
  unsigned long long t0 = globaltimer();
  unsigned ns = 32;
  while (ld_acquire_sys(flag) < v) {
    // give up at the timeout, or at once if an earlier wait already timed out (so a broken
    // peer costs one timeout, not one per pending wait)
    if (globaltimer() - t0 > timeout_ns || *(volatile unsigned int*)err) {
      atomicOr(err, 1u);
      return false;
    }
    __nanosleep(ns);
    if (ns < 256) ns <<= 1;
  }
  return true;
}

// Block-wide signal release after the block's stores (put_signal_nbi_block): every
// thread's stores are ordered before the barrier; one thread fences at system scope and
// release-stores the flag.
__device__ __forceinline__ void block_signal_release(uint64_t* flag, uint64_t v) {
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence_system();
    st_release_sys(flag, v);
  }
}

// splitmix64 finaliser (Steele, Lea, Flood 2014) -- the input recipe's counter-based generator.
__device__ __forceinline__ uint64_t splitmix64(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

}  // namespace dev
}  // namespace uc
