// stencil_common.cuh -- device code shared by the Jacobi kernels of libuniconn_b200
// (kernels.cu: variants 0-4 and the P2P/collective kernels; multistep.cu: variant 5): the
// stencil formula (reading G1), the row update with cross-warp edge values, streaming stores,
// the per-strip flag waits, the block reduction and the end-of-launch bookkeeping (norm
// publication, iteration counter, slab parity offset).  Internal; not part of the C-ABI.
#pragma once
#include <cmath>

#include "device_api.cuh"
#include "uc_internal.h"

namespace uc {
using namespace dev;

constexpr unsigned kFull = 0xffffffffu;
// Compile-time tuning knobs (A/B builds via build.py --define; defaults are the product build).
#ifndef UC_KR
#define UC_KR 4
#endif
#ifndef UC_STORE_CS
#define UC_STORE_CS 1
#endif
#ifndef UC_MINBLOCKS
#define UC_MINBLOCKS 1
#endif
constexpr int kR = UC_KR;      // rows per prefetch batch
#ifndef UC_STAGE_PAD
#define UC_STAGE_PAD 4
#endif
constexpr int kPad = UC_STAGE_PAD;  // staged ring: halo floats copied on each side of a strip
#ifndef UC_L2_EVICT_FIRST
#define UC_L2_EVICT_FIRST 1
#endif
// two-iteration kernel: steady-state loop unroll and min blocks per SM (register cap 72 at 3);
// sweep in profiles/r1_two_step_sweep.txt
#ifndef UC_TWO_STEP_UNROLL
#define UC_TWO_STEP_UNROLL 2
#endif
constexpr int kTwoStepUnroll = UC_TWO_STEP_UNROLL;
// T-level kernel (variant 5): min blocks per SM (2: 113-register cap, no spills at T = 4) and
// the unroll of the row loop (3 = the period of the register rotation: no moves); sweep in
// profiles/r1_multi_step_sweep.txt
#ifndef UC_T_MINBLOCKS
#define UC_T_MINBLOCKS 2
#endif
// the same for the two-ghost-lane layout (T up to 8: twice the register window, 165 registers at
// T = 8): one block per SM of up to UC_T8_MAXTHREADS threads (12 warps: 3 per SM sub-partition,
// so the 16K-register file of a sub-partition allows 170 registers per thread)
#ifndef UC_T8_MINBLOCKS
#define UC_T8_MINBLOCKS 2
#endif
#ifndef UC_T8_MAXTHREADS
#define UC_T8_MAXTHREADS 256
#endif
constexpr int kMaxBlockG2 = UC_T8_MAXTHREADS - 32;  // consumer threads per block, two ghost lanes
#ifndef UC_T_UNROLL
#define UC_T_UNROLL 3
#endif
#ifndef UC_PACKED_F32X2
#define UC_PACKED_F32X2 1
#endif
constexpr int kTUnroll = UC_T_UNROLL;
#ifndef UC_TWO_STEP_MINBLOCKS
#define UC_TWO_STEP_MINBLOCKS 3
#endif
#ifndef UC_BLOCK_ORDER
#define UC_BLOCK_ORDER 0
#endif

__device__ __forceinline__ void st4(float* p, float4 v) {
#if UC_STORE_CS
  __stcs(reinterpret_cast<float4*>(p), v);  // streaming: the result is read next iteration from HBM
#else
  *reinterpret_cast<float4*>(p) = v;
#endif
}
constexpr int kMaxBlock = 256; // threads per block (upper bound)

// ------------------------------------------------------------------------------ stencil math
// Reading G1: new = 0.25f*((l+r)+(t+b)); __fadd_rn/__fmul_rn are never contracted into FMA
// and do not flush subnormals (no --use_fast_math).
__device__ __forceinline__ float upd(float l, float r, float t, float b) {
  return __fmul_rn(0.25f, __fadd_rn(__fadd_rn(l, r), __fadd_rn(t, b)));
}

// New values of the 4 columns [4*x4, 4*x4+3] of row c, given the rows above (up) and below
// (dn).  e is this lane's cross-warp neighbour: lane 0 holds column 4*x4-1, lane 31 holds
// column 4*x4+4.  Columns 0 and NX-1 are Dirichlet (reading G2) and keep their value.
// Must be called by all 32 lanes (shuffles).
__device__ __forceinline__ float4 row_update(float4 up, float4 c, float4 dn, float e, int lane, int x4, int nx4) {
  float L = __shfl_up_sync(kFull, c.w, 1);
  float R = __shfl_down_sync(kFull, c.x, 1);
  if (lane == 0) L = e;
  if (lane == 31) R = e;
  float4 o;
  o.x = (x4 == 0) ? c.x : upd(L, c.y, up.x, dn.x);
  o.y = upd(c.x, c.z, up.y, dn.y);
  o.z = upd(c.y, c.w, up.z, dn.z);
  o.w = (x4 == nx4 - 1) ? c.w : upd(c.z, R, up.w, dn.w);
  return o;
}

__device__ __forceinline__ void acc_sq(double& acc, float4 o, float4 c) {
  // d in fp32 (bit-identical to the oracle's d); (double)d*(double)d is exact.
  const float d0 = __fsub_rn(o.x, c.x), d1 = __fsub_rn(o.y, c.y);
  const float d2 = __fsub_rn(o.z, c.z), d3 = __fsub_rn(o.w, c.w);
  acc += (double)d0 * (double)d0;
  acc += (double)d1 * (double)d1;
  acc += (double)d2 * (double)d2;
  acc += (double)d3 * (double)d3;
}

// Read-only (non-coherent path) loads for rows that only this rank's previous kernel wrote.
__device__ __forceinline__ float4 ld4_ro(const float* row, int x4, bool valid) {
  return valid ? __ldg(reinterpret_cast<const float4*>(row) + x4) : make_float4(0.f, 0.f, 0.f, 0.f);
}
__device__ __forceinline__ float ld_edge_ro(const float* row, int x4, int lane, int nx4, bool valid) {
  if (!valid) return 0.f;
  if (lane == 0 && x4 > 0) return __ldg(row + 4 * x4 - 1);
  if (lane == 31 && x4 + 1 < nx4) return __ldg(row + 4 * x4 + 4);
  return 0.f;
}
// Coherent loads for the boundary rows (a neighbour may have just written the halo row).
__device__ __forceinline__ float4 ld4_co(const float* row, int x4, bool valid) {
  return valid ? reinterpret_cast<const float4*>(row)[x4] : make_float4(0.f, 0.f, 0.f, 0.f);
}
__device__ __forceinline__ float ld_edge_co(const float* row, int x4, int lane, int nx4, bool valid) {
  if (!valid) return 0.f;
  if (lane == 0 && x4 > 0) return row[4 * x4 - 1];
  if (lane == 31 && x4 + 1 < nx4) return row[4 * x4 + 4];
  return 0.f;
}

// Wait until the halo-row flags of strips s-1, s, s+1 on one side reach v.  The flag of strip s
// says both "the neighbour's strip-s halo data of A_v is here" and "the neighbour's block of
// strip s has finished reading the halo row we are about to overwrite"; the two-iteration
// kernel (variant 4) also reads one column across each strip edge, so a writer or reader of
// strip s waits for the adjacent strips' flags too.
__device__ __forceinline__ void wait_strip_flags(const JacobiParams& p, int base, int s, uint64_t v) {
  const int s0 = s > 0 ? s - 1 : 0;
  const int s1 = s + 1 < p.strips ? s + 1 : s;
  for (int j = s0; j <= s1; ++j) wait_ge(p.my_flags + (size_t)(base + j) * kFlagStride, v, p.timeout_ns, p.err);
}

// The same waits executed by ALL 32 lanes of one warp, with warp-vote loop conditions: the loop is
// provably warp-uniform, so the code after it stays provably converged (a single-thread spin
// loop makes the compiler guard every later shuffle with a divergence check and every later
// mbarrier wait with a reconvergence region -- ~10 % more instructions in the march).
__device__ __forceinline__ uint64_t ld_acquire_gpu(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint64_t ld_relaxed_gpu(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_gpu(uint64_t* p, uint64_t v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
// gpu = true when every party of the protocol is on this GPU (.gpu scope suffices)
__device__ __forceinline__ bool wait_ge_warp(const uint64_t* sig, uint64_t v, unsigned long long timeout_ns,
                                             unsigned int* err, bool gpu = false) {
  if (__all_sync(kFull, (gpu ? ld_acquire_gpu(sig) : uc_dev_ld_acquire(sig)) >= v)) return true;
  const unsigned long long t0 = uc_dev_globaltimer();
  unsigned ns = 32;
  while (!__all_sync(kFull, (gpu ? ld_relaxed_gpu(sig) : uc_dev_ld_relaxed(sig)) >= v)) {
    const bool give_up = uc_dev_globaltimer() - t0 > timeout_ns || *(volatile unsigned int*)err;
    if (__any_sync(kFull, give_up)) {
      if ((threadIdx.x & 31) == 0) atomicOr(err, 1u);
      return false;
    }
    __nanosleep(ns);
    if (ns < 256) ns <<= 1;
  }
  // the observing relaxed load + fence = acquire
  if (gpu) asm volatile("fence.acq_rel.gpu;" ::: "memory");
  else asm volatile("fence.acq_rel.sys;" ::: "memory");
  return true;
}
__device__ __forceinline__ void wait_strip_flags_warp(const JacobiParams& p, int base, int s, uint64_t v) {
  const int s0 = s > 0 ? s - 1 : 0;
  const int s1 = s + 1 < p.strips ? s + 1 : s;
  for (int j = s0; j <= s1; ++j)
    wait_ge_warp(p.my_flags + (size_t)(base + j) * kFlagStride, v, p.timeout_ns, p.err, p.gpu_scope != 0);
}
// warp index, broadcast from lane 0: branches on it are known warp-uniform
__device__ __forceinline__ int warp_id_uniform() { return __shfl_sync(kFull, (int)threadIdx.x >> 5, 0); }

// ------------------------------------------------------------------------------ reductions
__device__ __forceinline__ double block_sum(double v, double* smem) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(kFull, v, o);
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5;
  __syncthreads();
  if (lane == 0) smem[w] = v;
  __syncthreads();
  double t = 0.0;
  if (w == 0) {
    t = lane < nw ? smem[lane] : 0.0;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) t += __shfl_xor_sync(kFull, t, o);
  }
  return t;  // valid in thread 0
}

// Thread 0 of the block that summed the rank's partials: publish the norm round.
__device__ inline void norm_publish(const JacobiParams& p, double tot) {
  if (p.device_mode == 1) {
    // one-shot P2P allreduce of the rank partial (§8 a5): write slot[rank] on every rank,
    // release a flag, wait for all P flags, sum slots 0..P-1 in rank order (reading G12).
    const uint64_t m = p.k_dev[1];
    const int par = (int)(m & 1);
    for (int q = 0; q < p.size; ++q) st_relaxed_sys_f64(p.norm_slot[q] + par * p.size + p.rank, tot);
    __threadfence_system();
    for (int q = 0; q < p.size; ++q)
      st_release_sys(p.norm_flag[q] + (size_t)(par * p.size + p.rank) * kFlagStride, m + 1);
    double g = 0.0;
    for (int q = 0; q < p.size; ++q) {
      wait_ge(p.norm_flag[p.rank] + (size_t)(par * p.size + q) * kFlagStride, m + 1, p.timeout_ns, p.err);
      g += ld_relaxed_sys_f64(p.norm_slot[p.rank] + par * p.size + q);
    }
    p.norm_hist[m % (uint64_t)p.norm_cap] = sqrt(g);
    p.k_dev[1] = m + 1;
  } else {
    *p.rank_sum = tot;  // host/partial mode: ncclAllReduce + norm_finish_kernel complete it
  }
}

// Last block: deterministic sum of the block partials, cross-rank norm (device mode), counter bumps.
// advance = iterations done by this launch (2 for the two-iteration kernel, which also flips
// the slab parity offset k_dev[2]).
__device__ inline void finish_iteration(const JacobiParams& p, bool do_norm, double* smem, int advance) {
  double tot = 0.0;
  if (do_norm) {
    double v = 0.0;
    for (int i = threadIdx.x; i < (int)gridDim.x; i += blockDim.x) v += p.partials[i];
    tot = block_sum(v, smem);
  }
  if (threadIdx.x == 0) {
    if (do_norm) norm_publish(p, tot);
    p.k_dev[0] = p.k_dev[0] + (unsigned long long)advance;
    if ((advance & 1) == 0) p.k_dev[2] = p.k_dev[2] ^ 1ull;  // A_{k+advance} went to the other slab
    p.launch_hist[advance < 15 ? advance : 15] += 1ull;      // what really ran (uc_jacobi_launch_counts)
    *p.done = 0;
    *p.work = 0;  // variant 2 tile counter
    __threadfence();
  }
}

struct RingCursor {
  int st;
  unsigned ph;
};

}  // namespace uc
