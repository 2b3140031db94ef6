// device_api.cuh -- header-only device primitives of libuniconn_b200 (the paper inlines its
// device API in headers).  System-scope (.sys) release/acquire because the peer is
// another GPU reached over NVLink (reading G10); a bounded spin turns a hang into an error.
#pragma once
#include <cstdint>

#include "uniconn_device.cuh"  // the public device API: signals, waits, grouped puts

namespace uc {
namespace dev {

__device__ __forceinline__ unsigned long long globaltimer() { return uc_dev_globaltimer(); }
__device__ __forceinline__ uint64_t ld_acquire_sys(const uint64_t* p) { return uc_dev_ld_acquire(p); }
__device__ __forceinline__ void st_release_sys(uint64_t* p, uint64_t v) { uc_dev_signal(p, v, UC_DEV_SIGNAL_SET); }

__device__ __forceinline__ void st_relaxed_sys_f64(double* p, double v) {
  asm volatile("st.relaxed.sys.global.f64 [%0], %1;" ::"l"(p), "d"(v) : "memory");
}

__device__ __forceinline__ double ld_relaxed_sys_f64(const double* p) {
  double v;
  asm volatile("ld.relaxed.sys.global.f64 %0, [%1];" : "=d"(v) : "l"(p) : "memory");
  return v;
}

// Acknowledge / nvshmem_signal_wait_until(GE) for one thread (uc_dev_wait_ge).  Returns false
// on timeout (and sets bit 0 of *err).  Monotone ">=" instead of the listing's "==": a
// neighbour one iteration ahead must not hang us (reading G10).  Once one wait has timed out the
// others give up at once, so a broken peer costs one timeout, not one per pending wait.
__device__ __forceinline__ bool wait_ge(const uint64_t* flag, uint64_t v, unsigned long long timeout_ns,
                                        unsigned int* err) {
  return uc_dev_wait_ge(flag, v, timeout_ns, err);
}


// ---- mbarrier + bulk-copy (TMA engine) helpers, sm_90+ PTX, used by the staged y-march
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint64_t* bar, unsigned count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
// arrive only if `pred`, as a predicated instruction (no divergent branch around it)
__device__ __forceinline__ void mbar_arrive_if(uint64_t* bar, bool pred) {
  asm volatile(
      "{\n .reg .pred p;\n setp.ne.u32 p, %1, 0;\n @p mbarrier.arrive.shared::cta.b64 _, [%0];\n}" ::"r"(smem_u32(bar)),
      "r"((unsigned)pred)
      : "memory");
}
// UC_WAIT_HINT_NS > 0: try_wait's suspend-time hint -- the waiting warp sleeps up to that long in
// ONE try_wait (woken when the phase completes) instead of re-issuing try_wait + branch in a
// loop, which takes issue slots from the warps that have work
#ifndef UC_WAIT_HINT_NS
#define UC_WAIT_HINT_NS 0
#endif
__device__ __forceinline__ void mbar_wait(uint64_t* bar, unsigned parity) {
#if UC_WAIT_HINT_NS > 0
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "UC_WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1, %2;\n"
      "@!p bra UC_WAIT_%=;\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(parity), "n"(UC_WAIT_HINT_NS)
      : "memory");
#else
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "UC_WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra UC_WAIT_%=;\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
#endif
}
// Non-blocking phase test (mbarrier.test_wait, acquire on success): issued a row ahead, its
// latency overlaps the current row's arithmetic instead of sitting on the critical path.
__device__ __forceinline__ bool mbar_test(uint64_t* bar, unsigned parity) {
  unsigned r;
  asm volatile(
      "{\n .reg .pred p;\n mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}"
      : "=r"(r) : "r"(smem_u32(bar)), "r"(parity) : "memory");
  return r != 0;
}
// mbar_wait unless `done` (an earlier mbar_test of the same phase succeeded): one asm block, so
// the skip is a predicated branch around the wait loop
__device__ __forceinline__ void mbar_wait_unless(uint64_t* bar, unsigned parity, bool done) {
  asm volatile(
      "{\n"
      ".reg .pred p, d;\n"
      "setp.ne.u32 d, %2, 0;\n"
      "@d bra UC_SKIP_%=;\n"
      "UC_WAIT_%=:\n"
#if UC_WAIT_HINT_NS > 0
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1, %3;\n"
#else
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
#endif
      "@!p bra UC_WAIT_%=;\n"
      "UC_SKIP_%=:\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(parity), "r"((unsigned)done), "n"(UC_WAIT_HINT_NS > 0 ? UC_WAIT_HINT_NS : 1)
      : "memory");
}
// 1-D bulk copy global -> shared through the TMA engine, completion counted in bytes on `bar`.
// dst, src 16-byte aligned; bytes a multiple of 16.
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, unsigned bytes, uint64_t* bar,
                                         uint64_t policy) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::
          "r"(smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(policy)
      : "memory");
}
// Orders this thread's view of generic-proxy global writes (made visible to it by an acquire)
// before its subsequent async-proxy (TMA) global reads.
__device__ __forceinline__ void fence_proxy_async_global() {
  asm volatile("fence.proxy.async.global;" ::: "memory");
}
__device__ __forceinline__ uint64_t policy_evict_normal() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t policy_evict_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}

// Barrier among the first `count` threads of the block (count a multiple of 32), id 1..15.
__device__ __forceinline__ void named_barrier_sync(int id, int count) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(count) : "memory");
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
