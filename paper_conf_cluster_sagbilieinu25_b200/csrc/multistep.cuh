// multistep.cuh -- kernel variant 5 of libuniconn_b200: T Jacobi iterations per launch (device
// templates; instantiated by multistep.cu for G = 1 ghost lane, multistep_g2.cu for G = 2).
// (§VI-C stencil; Listing 3 P:52-74 halo exchange, once per iteration.)
#pragma once
#include "stencil_common.cuh"

namespace uc {

// A/B instrumentation only (build.py --define UC_TRACE=1 --out ...): %globaltimer stamps per block
// of the deep-T launches (kernel start, after round 1, after the march, after each later round,
// end) into a managed buffer the host reads with uc_debug_trace_buffer().  Off in the product.
#ifndef UC_TRACE
#define UC_TRACE 0
#endif
#if UC_TRACE
static __device__ unsigned long long* uc_trace_ptr;
#define UC_TRACE_AT(slot)                                                                       \
  do {                                                                                         \
    if (threadIdx.x == 0 && uc_trace_ptr) uc_trace_ptr[blockIdx.x * 16 + (slot)] = globaltimer(); \
  } while (0)
#else
#define UC_TRACE_AT(slot) \
  do {                    \
  } while (0)
#endif

// Bounds checks of the T-level kernel's geometry (build.py --define UC_DEBUG_CHECKS=1 --out ...):
// compute-sanitizer is not available on the GPU pool, so a debug build asserts what the
// kernel's memory safety rests on (rows read and written, ring offsets, balanced tables) and
// traps on the first violation.  Off in the product.
#ifndef UC_DEBUG_CHECKS
#define UC_DEBUG_CHECKS 0
#endif
#if UC_DEBUG_CHECKS
#define UC_CHECK(cond)                                                                          \
  do {                                                                                         \
    if (!(cond)) {                                                                             \
      printf("UC_CHECK failed: %s (block %d thread %d, %s:%d)\n", #cond, blockIdx.x, threadIdx.x, \
             __FILE__, __LINE__);                                                              \
      __trap();                                                                                \
    }                                                                                          \
  } while (0)
#else
#define UC_CHECK(cond) \
  do {                 \
  } while (0)
#endif

// System-scope fence before the release-store of a round's flag to a neighbour on another GPU
// (A/B: 0 relies on st.release.sys cumulativity after the block barrier alone)
#ifndef UC_ROUND_SYS_FENCE
#define UC_ROUND_SYS_FENCE 1
#endif

// ------------------------------------------------------------------------------ T iterations per launch
// Variant 5: one launch advances A_k -> A_{k+T}, T = 1..8 (temporal blocking of depth T).  The
// staged march keeps T register levels: from the A_k row r streamed through the TMA ring it
// computes the A_{k+1} row r-1, the A_{k+2} row r-2, ..., and stores only the A_{k+T} row r-T:
// 8 HBM bytes per point per launch, 8/T per point-iteration.
//
// Horizontal neighbours across warp edges: "ghost lanes".  With G ghost lanes per side a warp owns
// the 32 - 2G float4 columns of its lanes G..31-G; lanes 0..G-1 and 32-G..31 hold copies of the
// neighbouring warps' (or strips') edge columns, loaded from the ring, and run the same stencil.
// Their own results go wrong one column per level from the outer side (their missing
// neighbour), so after T <= 4G levels the 4G columns of the ghost lanes may be wrong but every
// owned lane is exact: no cross-warp exchange, no barrier.  G = 1 (30 owned lanes) serves
// T <= 4, G = 2 (28 owned lanes) T <= 8.  A strip is (32 - 2G) * (consumers / 32) float4
// columns (the last warps of a block may own fewer).
//
// Boundary rows: level j (A_{k+j}) rows near the slab edge depend on the neighbour's level j-1
// rows, so the first/last row-chunk block of each strip runs T "rounds" per side: round j waits
// for the neighbour's level j-1 edge row (round 1: the A_k halo row), recomputes levels 1..j of
// the first few rows from A_k and the neighbour's rows, and puts its own level j edge row to the
// neighbour (levels < T: the h buffers; level T: the halo row of the output slab) with a
// release flag k + j.  Round 1 runs before the march (its puts overlap the whole sweep), rounds
// 2..T after it.  Every level of every boundary row is exchanged, as in the one-iteration
// kernel: only the HBM traffic of the interior changes.

// G ghost lanes per warp side: T <= 4 levels need G = 1 (a ghost lane holds 4 columns), T <= 8
// need G = 2.  A warp owns 32 - 2G float4 columns (lanes G..31-G); the ring rows carry 4G floats
// of halo on each side of a strip.
template <int G>
struct Ghost {
  static constexpr int kOwn = 32 - 2 * G;
  static constexpr int kPadG = 4 * G;
};

// Packed fp32x2 arithmetic of sm_100 (FADD2 / FMUL2): two IEEE round-to-nearest operations per
// instruction, no FTZ (no .ftz), never contracted -- bit-identical to two __fadd_rn / __fmul_rn.
__device__ __forceinline__ void add2_rn(float a0, float a1, float b0, float b1, float& r0, float& r1) {
  asm("{\n .reg .b64 a, b, r;\n mov.b64 a, {%2, %3};\n mov.b64 b, {%4, %5};\n"
      " add.rn.f32x2 r, a, b;\n mov.b64 {%0, %1}, r;\n}"
      : "=f"(r0), "=f"(r1) : "f"(a0), "f"(a1), "f"(b0), "f"(b1));
}
__device__ __forceinline__ void quarter2_rn(float a0, float a1, float& r0, float& r1) {
  asm("{\n .reg .b64 a, q, r;\n mov.b64 a, {%2, %3};\n mov.b64 q, {%4, %4};\n"
      " mul.rn.f32x2 r, a, q;\n mov.b64 {%0, %1}, r;\n}"
      : "=f"(r0), "=f"(r1) : "f"(a0), "f"(a1), "f"(0.25f));
}

// row_update for the ghost-lane layout (no cross-warp operand): new = 0.25f*((l+r)+(t+b)) with
// the vertical sums t+b, the outer sums and the products packed two columns per instruction.
// L, R: the left neighbour of column 4*x4 and the right neighbour of column 4*x4+3 (the
// adjacent lanes' c.w and c.x).
template <bool DIRI = true>
__device__ __forceinline__ float4 row_update_lr(float4 up, float4 c, float4 dn, float L, float R, int x4, int nx4) {
#if UC_PACKED_F32X2
  const float hx = __fadd_rn(L, c.y), hy = __fadd_rn(c.x, c.z);
  const float hz = __fadd_rn(c.y, c.w), hw = __fadd_rn(c.z, R);
  float vx, vy, vz, vw, sx, sy, sz, sw, ox, oy, oz, ow;
  add2_rn(up.x, up.y, dn.x, dn.y, vx, vy);
  add2_rn(up.z, up.w, dn.z, dn.w, vz, vw);
  add2_rn(hx, hy, vx, vy, sx, sy);
  add2_rn(hz, hw, vz, vw, sz, sw);
  quarter2_rn(sx, sy, ox, oy);
  quarter2_rn(sz, sw, oz, ow);
  float4 o;
  o.x = (DIRI && x4 == 0) ? c.x : ox;  // DIRI = false: no lane of the block holds a fixed column
  o.y = oy;
  o.z = oz;
  o.w = (DIRI && x4 == nx4 - 1) ? c.w : ow;
#else
  float4 o;
  o.x = (x4 == 0) ? c.x : upd(L, c.y, up.x, dn.x);
  o.y = upd(c.x, c.z, up.y, dn.y);
  o.z = upd(c.y, c.w, up.z, dn.z);
  o.w = (x4 == nx4 - 1) ? c.w : upd(c.z, R, up.w, dn.w);
#endif
  return o;
}
template <bool DIRI = true>
__device__ __forceinline__ float4 row_update_g(float4 up, float4 c, float4 dn, int x4, int nx4) {
  const float L = __shfl_up_sync(kFull, c.w, 1);    // lane 0: its own value (ghost lane, discarded)
  const float R = __shfl_down_sync(kFull, c.x, 1);  // lane 31: likewise
  return row_update_lr<DIRI>(up, c, dn, L, R, x4, nx4);
}

// ---- the march's register frame
// A row's four columns x0..x3 live in two 64-bit register pairs, P = (x0, x3) and Q = (x1, x2),
// instead of (x0, x1) | (x2, x3).  Then both horizontal sums of a level are single packed adds on
// pairs as they stand: (h0, h3) = (L, R) + Q, with the two shuffled neighbours landing in one
// pair, and (h1, h2) = P + swap(Q), the swap being a free FADD2 operand modifier (.LO_HI).  A
// level is 8 packed FP32 instructions + 2 shuffles (row_update_lr: 4 FADD + 6 packed + 2
// shuffles).  Every value is the same IEEE operation on the same two operands as in
// row_update_lr (addition commutes exactly): bit-identical.  The pairs are 64-bit values in the
// source, so the register allocator keeps them as aligned pairs (with float4 rows it kept the
// natural order and rebuilt the pairs at every use).  A row is permuted into the frame once as it
// leaves the ring; the last level is computed straight into the natural order for the store.
using pair_t = unsigned long long;
struct Row2 {
  pair_t p, q;  // (x0, x3), (x1, x2): f32x2 (lo, hi)
};
__device__ __forceinline__ pair_t pk2(float lo, float hi) {
  pair_t r;
  asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(lo), "f"(hi));
  return r;
}
__device__ __forceinline__ void upk2(pair_t v, float& lo, float& hi) {
  asm("mov.b64 {%0, %1}, %2;" : "=f"(lo), "=f"(hi) : "l"(v));
}
__device__ __forceinline__ pair_t f2add(pair_t a, pair_t b) {
  pair_t r;
  asm("add.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
  return r;
}
__device__ __forceinline__ pair_t f2add_swapped(pair_t a, pair_t b) {  // a + (b.hi, b.lo)
  pair_t r;
  asm("{\n .reg .b32 lo, hi;\n .reg .b64 s;\n mov.b64 {lo, hi}, %2;\n mov.b64 s, {hi, lo};\n"
      " add.rn.f32x2 %0, %1, s;\n}"
      : "=l"(r) : "l"(a), "l"(b));
  return r;
}
__device__ __forceinline__ pair_t f2quarter(pair_t a) {
  pair_t r;
  asm("{\n .reg .b64 q;\n mov.b64 q, {%2, %2};\n mul.rn.f32x2 %0, %1, q;\n}" : "=l"(r) : "l"(a), "f"(0.25f));
  return r;
}
__device__ __forceinline__ Row2 to_row2(float4 n) { return Row2{pk2(n.x, n.w), pk2(n.y, n.z)}; }
// A ring row into the frame.  An LDS.128 lands in natural order, and a permutation by register
// moves is a copy the allocator rematerialises at every use of the row (~14 moves per row of the
// march); four exact scalar adds of -0 (x + -0 = x for every non-NaN x, -0 and subnormals
// included) make the permuted pairs values of their own, one instruction per column.  The warps
// that hold a fixed column (DIRI) copy, so a NaN payload in a Dirichlet column passes unchanged.
#ifndef UC_PQ_ADD_PERMUTE
#define UC_PQ_ADD_PERMUTE 1
#endif
template <bool DIRI>
__device__ __forceinline__ Row2 ring_row2(float4 n) {
  if (UC_PQ_ADD_PERMUTE && !DIRI)
    return Row2{pk2(__fadd_rn(n.x, -0.f), __fadd_rn(n.w, -0.f)), pk2(__fadd_rn(n.y, -0.f), __fadd_rn(n.z, -0.f))};
  return to_row2(n);
}
__device__ __forceinline__ float4 from_row2(Row2 r) {
  float4 n;
  upk2(r.p, n.x, n.w);
  upk2(r.q, n.y, n.z);
  return n;
}
// the horizontal neighbours (L, R) of a row as one pair: x3 of the lane on the left, x0 of the
// lane on the right (lanes 0 / 31: their own values -- ghost lanes, discarded)
__device__ __forceinline__ pair_t row2_lr(const Row2& c) {
  float x0, x3;
  upk2(c.p, x0, x3);
  return pk2(__shfl_up_sync(kFull, x3, 1), __shfl_down_sync(kFull, x0, 1));
}
// new = 0.25f*((l+r)+(t+b)) for the 4 columns, in the frame
template <bool DIRI, bool SC = false>
__device__ __forceinline__ Row2 row2_update(const Row2& up, const Row2& c, const Row2& dn, pair_t lr, int x4, int nx4) {
  static_assert(!(DIRI && SC), "fixed columns are not scaled");
  const pair_t hp = f2add(lr, c.q);          // (L + x1, R + x2)  = (h0, h3)
  const pair_t hq = f2add_swapped(c.p, c.q); // (x0 + x2, x3 + x1) = (h1, h2)
  const pair_t vp = f2add(up.p, dn.p), vq = f2add(up.q, dn.q);
  // SC (the scaled march, below): the level's sums themselves, 4x the level's values
  Row2 o{SC ? f2add(hp, vp) : f2quarter(f2add(hp, vp)), SC ? f2add(hq, vq) : f2quarter(f2add(hq, vq))};
  if (DIRI) {  // fixed columns 0 (x0) and NX-1 (x3), both in P
    float a0, a3, c0, c3;
    upk2(o.p, a0, a3);
    upk2(c.p, c0, c3);
    o.p = pk2(x4 == 0 ? c0 : a0, x4 == nx4 - 1 ? c3 : a3);
  }
  return o;
}
// the same level with the products as scalar multiplies written in natural column order (the
// last level of the march: its row is only stored)
template <bool DIRI, bool SC = false, int T = 1>
__device__ __forceinline__ float4 row2_update_natural(const Row2& up, const Row2& c, const Row2& dn, pair_t lr, int x4,
                                                      int nx4) {
  static_assert(!(DIRI && SC), "fixed columns are not scaled");
  const pair_t hp = f2add(lr, c.q);
  const pair_t hq = f2add_swapped(c.p, c.q);
  const pair_t vp = f2add(up.p, dn.p), vq = f2add(up.q, dn.q);
  float s0, s3, s1, s2;
  upk2(f2add(hp, vp), s0, s3);
  upk2(f2add(hq, vq), s1, s2);
  // SC: the sums are 4^(T-1) x the unscaled level's sums; 4^-T undoes the scale and the 0.25
  constexpr float m = SC ? 1.0f / (float)(1u << (2 * T)) : 0.25f;
  float4 o = make_float4(__fmul_rn(s0, m), __fmul_rn(s1, m), __fmul_rn(s2, m), __fmul_rn(s3, m));
  if (DIRI) {
    float c0, c3;
    upk2(c.p, c0, c3);
    o.x = x4 == 0 ? c0 : o.x;
    o.w = x4 == nx4 - 1 ? c3 : o.w;
  }
  return o;
}

// Level 1 from natural-order rows (UC_LEVEL1_NATURAL, T >= 2): the A_k rows stay in the pairs
// the ring load lands them in, (x0, x1) | (x2, x3), and level 1 forms its sums with scalar adds
// written straight into the frame's pairs -- 8 FADD + 2 FADD2 instead of four permuting adds
// per row plus 8 packed FP32 instructions (the same IEEE operations on the same operands).
#ifndef UC_LEVEL1_NATURAL
#define UC_LEVEL1_NATURAL 1
#endif
__device__ __forceinline__ Row2 nat_row2(float4 n) { return Row2{pk2(n.x, n.y), pk2(n.z, n.w)}; }
__device__ __forceinline__ float4 nat_float4(const Row2& r) {
  float4 n;
  upk2(r.p, n.x, n.y);
  upk2(r.q, n.z, n.w);
  return n;
}
__device__ __forceinline__ pair_t nat_lr(const Row2& c) {
  float x0, x1, x2, x3;
  upk2(c.p, x0, x1);
  upk2(c.q, x2, x3);
  (void)x1;
  (void)x2;
  return pk2(__shfl_up_sync(kFull, x3, 1), __shfl_down_sync(kFull, x0, 1));
}
template <bool DIRI, bool SC>
__device__ __forceinline__ Row2 row2_update_nat_in(const Row2& up, const Row2& c, const Row2& dn, pair_t lr, int x4,
                                                   int nx4) {
  float u0, u1, u2, u3, c0, c1, c2, c3, d0, d1, d2, d3, L, R;
  upk2(up.p, u0, u1);
  upk2(up.q, u2, u3);
  upk2(c.p, c0, c1);
  upk2(c.q, c2, c3);
  upk2(dn.p, d0, d1);
  upk2(dn.q, d2, d3);
  upk2(lr, L, R);
  const pair_t hp = pk2(__fadd_rn(L, c1), __fadd_rn(c2, R));   // (h0, h3)
  const pair_t hq = pk2(__fadd_rn(c0, c2), __fadd_rn(c1, c3));  // (h1, h2)
  const pair_t vp = pk2(__fadd_rn(u0, d0), __fadd_rn(u3, d3));
  const pair_t vq = pk2(__fadd_rn(u1, d1), __fadd_rn(u2, d2));
  Row2 o{SC ? f2add(hp, vp) : f2quarter(f2add(hp, vp)), SC ? f2add(hq, vq) : f2quarter(f2add(hq, vq))};
  if (DIRI) {
    float a0, a3;
    upk2(o.p, a0, a3);
    o.p = pk2(x4 == 0 ? c0 : a0, x4 == nx4 - 1 ? c3 : a3);
  }
  return o;
}

struct GhostLayout {
  int x4;        // float4 column of this thread (ghost lanes: the neighbour's edge column)
  bool in_grid;  // 0 <= x4 < nx4 (may be loaded)
  bool own;      // owned column of this strip: stored, put, counted in the norm
  int ring_off;  // float offset of x4 in a ring row (ring row starts at column 4*xs4 - 4G)
};
template <int G>
__device__ __forceinline__ GhostLayout ghost_layout(const JacobiParams& p, int s) {
  constexpr int OWN = Ghost<G>::kOwn;
  const int t = threadIdx.x, lane = t & 31, w = t >> 5;
  const int xs4 = s * p.strip4;
  const int xe4 = min(xs4 + p.strip4, p.nx4);
  GhostLayout g;
  g.x4 = xs4 + w * OWN + lane - G;
  g.in_grid = g.x4 >= 0 && g.x4 < p.nx4;
  g.own = lane >= G && lane < 32 - G && g.x4 < xe4 && t < p.consumers;
  g.ring_off = 4 * (w * OWN + lane - G) + Ghost<G>::kPadG;
  return g;
}

// Row chunk q of the slab, first/last chunks shortened by p.chunk_shrink rows (their blocks
// also run the boundary rounds).
__device__ __forceinline__ void chunk_rows(const JacobiParams& p, int q, int& lo, int& hi) {
  const long long nv = (long long)p.n + 2LL * p.chunk_shrink;
  const long long a = (long long)q * nv / p.chunks - p.chunk_shrink;
  const long long b = (long long)(q + 1) * nv / p.chunks - p.chunk_shrink;
  lo = 1 + (int)max(0LL, min(a, (long long)p.n));
  hi = (int)max(0LL, min(b, (long long)p.n));
}

// One boundary round j (1..T) of one side.  Rows are counted from the slab edge inward:
// i = 0 is the halo row (top: slab row 0, bottom: slab row n+1), i = 1 the edge row (row 1 / n).
// The stencil is symmetric in t and b, so the mirrored order gives bit-identical values.
template <int T, int NL>
__device__ __forceinline__ void t_round(const JacobiParams& p, const float* src, float* dst, int np, int s,
                                        const GhostLayout& g, uint64_t k, int j, bool top, bool cta_sync,
                                        double& acc) {
  constexpr int PT = T > 1 ? T - 1 : 1;  // edge rows of A_{k+T} produced here (1..PT)
  constexpr int NR = PT + T + 1;         // A_k rows 0..PT+T read
  const bool has = top ? p.has_top : p.has_bot;
  const bool dev = p.device_mode == 1;
  const size_t pitch = (size_t)p.nx;
  const int side = top ? 0 : 1;          // our h rows: 0 = from top, 1 = from bottom
  // warp 0 waits (all its lanes, warp-uniform loops: keeps the march after round 1 provably
  // converged), the block follows at the barrier
  const int wid = warp_id_uniform();
  if (wid == 0 && has && dev) {
    if (j == 1) wait_strip_flags_warp(p, top ? 0 : p.flag_half, s, k);  // A_k halo rows
    else {  // the neighbour's level j-1 edge row (its round j-1)
      const uint64_t* f = p.h1_flags + (size_t)(j - 2) * 2 * p.flag_half * kFlagStride;
      const int base = top ? 0 : p.flag_half;
      const int s0 = s > 0 ? s - 1 : 0, s1 = s + 1 < p.strips ? s + 1 : s;
      for (int q = s0; q <= s1; ++q)
        wait_ge_warp(f + (size_t)(base + q) * kFlagStride, k + j - 1, p.timeout_ns, p.err, p.gpu_scope != 0);
    }
  }
  if (cta_sync) __syncthreads();
  else named_barrier_sync(1, p.consumers);
  if (wid >= (p.consumers >> 5)) return;  // the producer warp (cta_sync rounds only)
  float4 a[NR];
#pragma unroll
  for (int i = 0; i < NR; ++i) {
    const int y = top ? i : p.n + 1 - i;
    a[i] = g.in_grid ? reinterpret_cast<const float4*>(src + (size_t)y * pitch)[g.x4] : make_float4(0.f, 0.f, 0.f, 0.f);
  }
#pragma unroll
  for (int m = 1; m <= T; ++m) {
    if (m <= j) {
      // level m rows 1 .. NR-1-m from level m-1 rows 0 .. NR-m (in place, ascending)
      float4 prev = a[0];
#pragma unroll
      for (int i = 1; i < NR - m; ++i) {
        const float4 o = row_update_g(prev, a[i], a[i + 1], g.x4, p.nx4);
        if (NL == m && m == j && i <= PT && g.own) acc_sq(acc, o, a[i]);
        prev = a[i];
        a[i] = o;
      }
      // level m row 0: the neighbour's (waited for in round m+1 <= j), or the fixed row
      if (m < j && has && g.in_grid)
        a[0] = reinterpret_cast<const float4*>(p.h1_rows + ((size_t)(m - 1) * 2 + side) * pitch)[g.x4];
    }
  }
  const bool put = has && p.device_mode != 0;
  if (j < T) {
    // our level j edge row -> the neighbour's h row of level j (top neighbour: its "from bottom")
    if (put && g.own) {
      float* nb = (top ? p.top_h1_rows : p.bot_h1_rows) + ((size_t)(j - 1) * 2 + (top ? 1 : 0)) * pitch;
      reinterpret_cast<float4*>(nb)[g.x4] = a[1];
    }
  } else {
#pragma unroll
    for (int i = 1; i <= PT; ++i) {
      const int y = top ? i : p.n + 1 - i;
      if (g.own) reinterpret_cast<float4*>(dst + (size_t)y * pitch)[g.x4] = a[i];
    }
    if (put && g.own) {
      if (top) reinterpret_cast<float4*>(p.top_slab[np] + (size_t)(p.n + 1) * pitch)[g.x4] = a[1];
      else reinterpret_cast<float4*>(p.bot_slab[np])[g.x4] = a[1];
    }
  }
  if (has && dev) {
    named_barrier_sync(1, p.consumers);
    if (wid == 0) {
      // the block's row stores (ordered before this warp by the barrier) become visible before
      // the flag: a fence at the protocol's scope, then the release store
      if (p.gpu_scope) __threadfence();
#if UC_ROUND_SYS_FENCE
      else __threadfence_system();
#endif
      if (p.put_delay_ns) {  // injected link latency (measurement knob): the flag arrives later
        const unsigned long long t0 = __shfl_sync(kFull, globaltimer(), 0);
        while (__shfl_sync(kFull, globaltimer(), 0) - t0 < p.put_delay_ns) {
        }
      }
      uint64_t* f;
      if (j < T)
        f = (top ? p.top_h1_flags : p.bot_h1_flags) + (size_t)(j - 1) * 2 * p.flag_half * kFlagStride +
            (size_t)((top ? p.flag_half : 0) + s) * kFlagStride;
      else if (top)
        f = p.top_flags + (size_t)(p.flag_half + s) * kFlagStride;  // top's from_bottom[s]
      else
        f = p.bot_flags + (size_t)s * kFlagStride;                  // bottom's from_top[s]
      if ((threadIdx.x & 31) == 0) {
        if (p.gpu_scope) st_release_gpu(f, j < T ? k + j : k + T);
        else st_release_sys(f, j < T ? k + j : k + T);
      }
    }
  }
}

// The T-level staged march: A_{k+T} rows a..b of strip s (rows outside the boundary rounds').
// The producer streams the A_k rows a-T..b+T; consumers keep two rows per level.
// One row of the T-level march: take the next A_k row from the ring, advance every level, store
// the A_{k+T} row (STORE: from the 2T-th row on).
// Take the next A_k row from the ring (wait for its stage, read it, release the stage).
__device__ __forceinline__ float4 t_fetch(const float* ring, uint64_t* full, uint64_t* empty, int ST, int NS,
                                          const GhostLayout& g, RingCursor& cur) {
  mbar_wait(full + cur.st, cur.ph);
  const float4 nv = *reinterpret_cast<const float4*>(ring + (size_t)cur.st * ST + g.ring_off);
  __syncwarp();
  mbar_arrive_if(empty + cur.st, (threadIdx.x & 31) == 0);
  if (++cur.st == NS) {
    cur.st = 0;
    cur.ph ^= 1u;
  }
  return nv;
}



// Shuffle the neighbours of the next step's first HOIST levels before its ring wait, the rest
// after it.  Measured per instance (profiles/r1_t8_sweep.txt, passes 7, 9): hoisting every level
// gains 2-8 % at T = 4, 5, 7, 8; at <6, 2>, whose 128 registers are exactly the cap, hoisting all
// six loses 2.5 % and hoisting three gains 1.7 %.
#ifndef UC_HOIST_ALL
#define UC_HOIST_ALL 0  // A/B knob: 1 = hoist every level on every instance, -1 = none
#endif
#ifndef UC_HOIST_62
#define UC_HOIST_62 3  // levels hoisted at <6, 2> (A/B: 0 / 2 / 3 / 4 -> 3509 / 3546 / 3568 / 3530 GLUPS)
#endif
#ifndef UC_HOIST_82
#define UC_HOIST_82 8  // levels hoisted at <8, 2> (A/B in the pair frame + scaled march, profiles/r2_pq_scaled_ab.txt: 0/2/4/8 -> 0.446/0.443/0.443/0.439 ms)
#endif
#ifndef UC_HOIST_72
#define UC_HOIST_72 7  // levels hoisted at <7, 2> (A/B)
#endif
// levels whose neighbours are shuffled before the ring wait (the rest after it)
template <int T, int G>
constexpr int kHoistLevels = UC_HOIST_ALL == 1    ? T
                             : UC_HOIST_ALL == -1 ? 0
                             : (T == 6 && G == 2) ? UC_HOIST_62
                             : (T == 7 && G == 2) ? UC_HOIST_72
                             : (T == 8 && G == 2) ? UC_HOIST_82
                                                  : T;


// Grouped march (UC_MARCH_GROUPED, the product build): the steady-state row loop runs in groups
// of kGroup rows = kGroup ring stages, so every stage index, mbarrier address and ring offset of
// the group is a compile-time constant (one ring phase flip per group instead of per-row stage
// bookkeeping), and kGroup is a multiple of the register-rotation period 3 (no moves at the loop
// back edge).  The ring stride is the compile-time maximum row (4 x the launch bounds' consumer
// threads + the halo floats), so ring loads use immediate offsets.  The ring has a multiple of
// kGroup stages.
#ifndef UC_MARCH_GROUPED
#define UC_MARCH_GROUPED 1
#endif
#ifndef UC_GROUP_ROWS
#define UC_GROUP_ROWS 9
#endif
constexpr int kGroup = UC_GROUP_ROWS;
// test the next row's ring phase right after taking the current row (mbarrier.test_wait), so
// the phase check's latency overlaps the arithmetic; the blocking wait runs only if it failed
#ifndef UC_RING_TEST_AHEAD
#define UC_RING_TEST_AHEAD 1
#endif
static_assert(kGroup % 3 == 0, "the group must be a multiple of the rotation period");
template <int G>
constexpr int kStageFloats = 4 * (G == 1 ? kMaxBlock : kMaxBlockG2) + 2 * Ghost<G>::kPadG;


// ---- the scaled march (UC_SCALED_MARCH, the product build; norm-free launches, warps without a
// fixed column).  The 0.25 product of levels 1..T-1 is a quarter of the FP32 work of a level.  It is
// dropped: level j keeps W_j = 4^j A_{k+j} (its plain sums (l+r)+(t+b) of level j-1's W), and the
// last level multiplies by 4^-T.  Binary floating point rounds scale-invariantly by powers of two
// as long as no value is subnormal or overflows, so then every W_j is exactly 4^j times the
// unscaled iterate and A_{k+T} comes out bit-identical.  When is nothing subnormal?  If every
// nonzero |A_k| value the warp reads is >= 2^(e) with e = -103 + 2T, all of them are integer
// multiples of q = 2^(e-23) = 2^(-126+2T); sums and their roundings of multiples of q are again
// multiples of q (a rounded result is a multiple of its own ulp, and ulp >= q or the sum is exact),
// so a nonzero level-j value of the unscaled iteration is a multiple of q 4^-j >= 2^-126: normal,
// and so is every scaled one (larger by 4^j).  Overflow: |W_j| <= 4^j max|A_k| (Jacobi averages),
// so max|A_k| < 2^110 keeps 4^T max|A_k| far below 2^128 for T <= 8.  Each warp tracks the range
// of the A_k rows it takes from the ring (max |x|; min over nonzero |x| as an unsigned min of
// (bits << 1) - 1, zero wrapping to the top); inf is out of range; a NaN propagates as the same
// canonical NaN in both forms.  If any warp of a block saw a value out of range, the whole block
// re-runs its march unscaled (the ring continues; A_k is untouched and the march's rows of A_{k+T}
// are rewritten) -- the answer is always the unscaled iteration's.
#ifndef UC_SCALED_MARCH
#define UC_SCALED_MARCH 1
#endif
struct RowRange {
  float amax;     // max |x|
  unsigned wmin;  // min ((bits << 1) - 1): nonzero |x|'s biased exponent in the top byte, zero -> ~0
};
__device__ __forceinline__ void range_add(RowRange& r, float4 n) {
  r.amax = fmaxf(fmaxf(r.amax, fabsf(n.x)), fmaxf(fmaxf(fabsf(n.y), fabsf(n.z)), fabsf(n.w)));
  const unsigned w0 = (__float_as_uint(n.x) << 1) - 1u, w1 = (__float_as_uint(n.y) << 1) - 1u;
  const unsigned w2 = (__float_as_uint(n.z) << 1) - 1u, w3 = (__float_as_uint(n.w) << 1) - 1u;
  r.wmin = min(min(r.wmin, w0), min(min(w1, w2), w3));
}
template <int T>
__device__ __forceinline__ bool range_ok(const RowRange& r) {
  constexpr unsigned kMinBiasedExp = 24 + 2 * T;  // 2^(-103+2T)
  return r.amax < 0x1p110f && r.wmin >= (kMinBiasedExp << 24) - 1u;
}

// One row of the T-level march: fetch the next A_k row, advance every level, store the A_{k+T}
// row (STORE: from the 2T-th row on).  The horizontal neighbours of every level's middle row
// (w1[j], known before the step's new row arrives) are shuffled up front, off the level chain
// (new row -> level 1 -> ... -> level T); the first HOIST levels' before the ring wait.
template <int T>
constexpr bool kNat0 = UC_LEVEL1_NATURAL && T >= 2;  // level-0 rows in natural pairs
template <int T, int J0, int J1>
__device__ __forceinline__ void t_neighbours2(const Row2 (&w1)[T], pair_t (&lr)[T]) {
#pragma unroll
  for (int j = J0; j < J1; ++j) lr[j] = (kNat0<T> && j == 0) ? nat_lr(w1[j]) : row2_lr(w1[j]);
}
template <int T, int NL, bool DIRI, bool STORE, bool SC>
__device__ __forceinline__ void t_levels2(const Row2& n0, const GhostLayout& g, int nx4, int a, int b, int i,
                                          Row2 (&w0)[T], Row2 (&w1)[T], const pair_t (&lr)[T], float*& out,
                                          size_t pitch, double& acc) {
  static_assert(!(SC && NL != 0), "norm launches run unscaled");
  Row2 nv = n0;
#pragma unroll
  for (int j = 0; j < T - 1; ++j) {
    const bool nat = kNat0<T> && j == 0;  // level 1 from natural-order A_k rows
    const Row2 o = nat ? row2_update_nat_in<DIRI, SC>(w0[j], w1[j], nv, lr[j], g.x4, nx4)
                       : row2_update<DIRI, SC>(w0[j], w1[j], nv, lr[j], g.x4, nx4);  // level j+1, row r-j-1
    if (NL == j + 1 && g.own) {
      const int y = a - T + i - j - 1;
      if (y >= a && y <= b) acc_sq(acc, from_row2(o), nat ? nat_float4(w1[j]) : from_row2(w1[j]));
    }
    w0[j] = w1[j];
    w1[j] = nv;
    nv = o;
  }
  // level T (natural column order: only stored)
  const float4 o = row2_update_natural<DIRI, SC, T>(w0[T - 1], w1[T - 1], nv, lr[T - 1], g.x4, nx4);
  if (NL == T && g.own) {
    const int y = a + i - 2 * T;  // a - T + i - j - 1 at j = T - 1
    if (y >= a && y <= b) acc_sq(acc, o, from_row2(w1[T - 1]));
  }
  w0[T - 1] = w1[T - 1];
  w1[T - 1] = nv;
  if (STORE) {
    if (g.own) st4(out, o);
    out += pitch;
  }
}
template <int T, int NL, bool DIRI, bool STORE, int HOIST, bool SC>
__device__ __forceinline__ void t_step2(const float* ring, uint64_t* full, uint64_t* empty, int ST, int NS,
                                        const GhostLayout& g, int nx4, int a, int b, int i, RingCursor& cur,
                                        Row2 (&w0)[T], Row2 (&w1)[T], float*& out, size_t pitch, double& acc,
                                        RowRange& rng) {
  pair_t lr[T];
  t_neighbours2<T, 0, HOIST>(w1, lr);
  const float4 n = t_fetch(ring, full, empty, ST, NS, g, cur);
  if (SC) range_add(rng, n);
  const Row2 nv = kNat0<T> ? nat_row2(n) : ring_row2<DIRI>(n);
  t_neighbours2<T, HOIST, T>(w1, lr);
  t_levels2<T, NL, DIRI, STORE, SC>(nv, g, nx4, a, b, i, w0, w1, lr, out, pitch, acc);
}
// One group of kGroup rows starting at ring stage gbase (a multiple of kGroup), phase ph.
template <int T, int NL, bool DIRI, int G, int HOIST, bool SC>
__device__ __forceinline__ void t_group2(const float* ringp, uint64_t* full, uint64_t* empty, unsigned ph,
                                         const GhostLayout& g, int nx4, int a, int b, int i0, Row2 (&w0)[T],
                                         Row2 (&w1)[T], float*& out, size_t pitch, double& acc, RowRange& rng) {
  constexpr int ST = kStageFloats<G>;
  const bool lane0 = (threadIdx.x & 31) == 0;
#if UC_RING_TEST_AHEAD
  bool ready = false;
#endif
#pragma unroll
  for (int u = 0; u < kGroup; ++u) {
    pair_t lr[T];
    t_neighbours2<T, 0, HOIST>(w1, lr);
#if UC_RING_TEST_AHEAD
    mbar_wait_unless(full + u, ph, ready);
#else
    mbar_wait(full + u, ph);
#endif
    const float4 n = *reinterpret_cast<const float4*>(ringp + u * ST);
    if (SC) range_add(rng, n);
    const Row2 nv = kNat0<T> ? nat_row2(n) : ring_row2<DIRI>(n);
    __syncwarp();
    mbar_arrive_if(empty + u, lane0);
#if UC_RING_TEST_AHEAD
    if (u + 1 < kGroup) ready = mbar_test(full + u + 1, ph);
#endif
    t_neighbours2<T, HOIST, T>(w1, lr);
    t_levels2<T, NL, DIRI, true, SC>(nv, g, nx4, a, b, i0 + u, w0, w1, lr, out, pitch, acc);
  }
}

// The march of one block over A_{k+T} rows a..b.  gi0: ring rows this block has already used in
// this launch (a re-run continues the ring's stage and phase sequence).  SC: the scaled march;
// returns true when this warp saw an A_k value outside its range (consumers only).
template <int T, int NL, bool DIRI, int G, bool SC>
__device__ __forceinline__ bool march_t(const JacobiParams& p, const float* src, float* dst, int s,
                                        const GhostLayout& g, int a, int b, double& acc, float* ring,
                                        uint64_t* full, uint64_t* empty, bool proxy_fence, int gi0) {
  const int nc = p.consumers, NS = p.stages;
  constexpr int PAD = Ghost<G>::kPadG;
#if UC_MARCH_GROUPED
  constexpr int ST = kStageFloats<G>;
  // warp-uniform role split: the compiler sees a branch on a broadcast value, so the consumer
  // path is known converged (no divergence checks around its shuffles and warp syncs)
  const int wid = __shfl_sync(kFull, (int)threadIdx.x >> 5, 0);
  const bool producer = wid >= (nc >> 5);
#else
  const int ST = 4 * nc + 2 * PAD;
  const bool producer = (int)threadIdx.x >= nc;
#endif
  const size_t pitch = (size_t)p.nx;
  const int rows = b - a + 1 + 2 * T;
  if (producer) {
    if ((threadIdx.x & 31) == 0) {
      const int xs = 4 * s * p.strip4;
      const int xe = min(xs + 4 * p.strip4, p.nx);
      const int left = xs >= PAD ? xs - PAD : 0;
      const int right = min(xe + PAD, p.nx);
      const unsigned bytes = (unsigned)(right - left) * 4u;
      const int off = left - (xs - PAD);
      UC_CHECK(off >= 0 && off + (int)(bytes / 4) <= ST && (bytes & 15u) == 0u && NS * ST * 4 + 128 <= 200 * 1024);
#if UC_L2_EVICT_FIRST
      const uint64_t pol = policy_evict_first();
#else
      const uint64_t pol = policy_evict_normal();
#endif
      if (proxy_fence) fence_proxy_async_global();
      int st = gi0 % NS;
      unsigned ph = (unsigned)(gi0 / NS) & 1u;
      for (int i = 0; i < rows; ++i) {
        if (gi0 + i >= NS) mbar_wait(empty + st, ph ^ 1u);
        mbar_arrive_expect_tx(full + st, bytes);
#ifdef UC_PROTO_L2_ROWS  // A/B measurement only (scripts/proto): cycle over a few L2-resident rows
        bulk_g2s(ring + (size_t)st * ST + off, src + (size_t)(a - T + i % UC_PROTO_L2_ROWS) * pitch + left, bytes,
                 full + st, pol);
#else
        bulk_g2s(ring + (size_t)st * ST + off, src + (size_t)(a - T + i) * pitch + left, bytes, full + st, pol);
#endif
        if (++st == NS) {
          st = 0;
          ph ^= 1u;
        }
      }
    }
    return false;
  }
  const int nx4 = p.nx4;
  Row2 w0[T], w1[T];  // level j: rows r-j-1 (w0) and r-j (w1) before row r arrives
#pragma unroll
  for (int j = 0; j < T; ++j) w0[j] = w1[j] = Row2{0ull, 0ull};
  RowRange rng{0.f, ~0u};
  RingCursor cur{gi0 % NS, (unsigned)(gi0 / NS) & 1u};
  constexpr int H = kHoistLevels<T, G>;
  float* out = dst + (size_t)a * pitch + 4 * (size_t)g.x4;  // the A_{k+T} row a comes out at i = 2T
  // the first 2T rows only fill the levels (rows >= 2T + 1 since a <= b)
#pragma unroll
  for (int i = 0; i < 2 * T; ++i)
    t_step2<T, NL, DIRI, false, H, SC>(ring, full, empty, ST, NS, g, nx4, a, b, i, cur, w0, w1, out, pitch, acc, rng);
#if UC_MARCH_GROUPED
  int i = 2 * T;
  // single rows up to the next group boundary (ring stage 0 mod kGroup)
  for (; i < rows && cur.st % kGroup != 0; ++i)
    t_step2<T, NL, DIRI, true, H, SC>(ring, full, empty, ST, NS, g, nx4, a, b, i, cur, w0, w1, out, pitch, acc, rng);
  const float* ringl = ring + g.ring_off;
  for (; i + kGroup <= rows; i += kGroup) {
    t_group2<T, NL, DIRI, G, H, SC>(ringl + cur.st * ST, full + cur.st, empty + cur.st, cur.ph, g, nx4, a, b, i, w0,
                                    w1, out, pitch, acc, rng);
    cur.st += kGroup;
    if (cur.st == NS) {
      cur.st = 0;
      cur.ph ^= 1u;
    }
  }
  for (; i < rows; ++i)
    t_step2<T, NL, DIRI, true, H, SC>(ring, full, empty, ST, NS, g, nx4, a, b, i, cur, w0, w1, out, pitch, acc, rng);
#else
#pragma unroll(kTUnroll)
  for (int i = 2 * T; i < rows; ++i)
    t_step2<T, NL, DIRI, true, H, SC>(ring, full, empty, ST, NS, g, nx4, a, b, i, cur, w0, w1, out, pitch, acc, rng);
#endif
  // a warp whose lanes are all outside the grid (the tail of the last strip) computes nothing kept
  return SC && g.in_grid && !range_ok<T>(rng);
}

// Boundary rounds 2..T after the march, out of line: the march's register allocation then does not
// carry the rounds' state (their row window, the block's geometry) across its loop.
#ifndef UC_ROUNDS_NOINLINE
#define UC_ROUNDS_NOINLINE 0  // A/B: out of line spills more (0.4131 vs 0.4086 ms, scripts/proto)
#endif
template <int T, int NL, int G>
__device__ __noinline__ double t_rounds_after(const JacobiParams& p, const float* src, float* dst, int par, int s,
                                              uint64_t k, bool rtop, bool rbot) {
  const GhostLayout g = ghost_layout<G>(p, s);
  double acc = 0.0;
  for (int j = 2; j <= T; ++j) {  // consumers only (named barrier 1)
    if (rtop) t_round<T, NL>(p, src, dst, par ^ 1, s, g, k, j, true, false, acc);
    if (rbot) t_round<T, NL>(p, src, dst, par ^ 1, s, g, k, j, false, false, acc);
  }
  return acc;
}

template <int T, int NL, int G>
__device__ __forceinline__ double t_body(const JacobiParams& p, uint64_t k, int par, float* ring, uint64_t* full,
                                         uint64_t* empty, unsigned long long t_entry = 0) {
  constexpr int PT = T > 1 ? T - 1 : 1;
  const float* src = p.slab[par];
  float* dst = p.slab[par ^ 1];
  int s, q, lo, hi;
  if (NL == 0 && p.bal_tab != nullptr) {
    // balanced launch: this block's (strip, chunk, rows) from the table uc_jacobi_run maintains
    // (any partition of every strip's rows into its chunks in order is exact; norm launches keep
    // the static chunking, so the block partials -- and the norm -- do not depend on timing)
    const int4 w = p.bal_tab[blockIdx.x];
    s = w.x;
    q = w.y;
    lo = w.z;
    hi = w.w;
  } else {
    s = blockIdx.x % p.strips;
    // part 0: every row chunk; part 1 (host overlap): the first and last chunk only (grid 2 x strips);
    // part 2: the others (chunks 1..chunks-2)
    q = p.part == 0 ? blockIdx.x / p.strips
        : p.part == 1 ? (blockIdx.x < p.strips ? 0 : p.chunks - 1)
                      : blockIdx.x / p.strips + 1;
    chunk_rows(p, q, lo, hi);
  }
  const GhostLayout g = ghost_layout<G>(p, s);
  const bool top_blk = q == 0, bot_blk = q == p.chunks - 1;
  // deep-halo host mode: a side with a neighbour holds T halo rows of A_k (the host exchanged T
  // rows), so the march covers the edge rows too (it streams rows 1-T..0 / n+1..n+T) and that
  // side runs no boundary rounds; a side without a neighbour keeps its rounds (fixed row)
  const bool deep_top = p.deep_halo && p.has_top, deep_bot = p.deep_halo && p.has_bot;
  const bool rtop = top_blk && !deep_top, rbot = bot_blk && !deep_bot;
  double acc = 0.0;
  // round 1 before the march (all threads: the producer must not read halo rows before the wait)
  UC_TRACE_AT(0);
#if UC_TRACE
  if (threadIdx.x == 0 && uc_trace_ptr) {
    unsigned smid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    uc_trace_ptr[blockIdx.x * 16 + 14] = smid;
  }
#endif
  if (rtop) t_round<T, NL>(p, src, dst, par ^ 1, s, g, k, 1, true, true, acc);
  if (rbot) t_round<T, NL>(p, src, dst, par ^ 1, s, g, k, 1, false, true, acc);
  UC_TRACE_AT(1);
  const int a = deep_top ? lo : max(lo, PT + 1);
  const int b = deep_bot ? hi : min(hi, p.n - PT);
  UC_CHECK(s >= 0 && s < p.strips && q >= 0 && q < p.chunks && lo >= 1 && hi <= p.n);
  // the march streams A_k rows a-T .. b+T: only a first/last chunk (which waited for the halo
  // flags in round 1, or holds a deep halo) may reach row 0 / n+1 and beyond
  UC_CHECK(a > b || a - T >= (deep_top ? 1 - T : top_blk ? 0 : 1));
  UC_CHECK(a > b || b + T <= (deep_bot ? p.n + T : bot_blk ? p.n + 1 : p.n));
  UC_CHECK((int)threadIdx.x >= p.consumers || !g.in_grid || g.ring_off + 4 <= kStageFloats<G>);  // consumers
  if (a <= b) {
    // fixed columns (0, NX-1) among the block's lanes, ghosts included: keep them fixed
    const int xs4 = s * p.strip4;
    // per WARP, not per block: only the warps whose lanes (ghosts included) hold column 0 or
    // NX-1 need the select that keeps it fixed (2 FSEL per float4 per level); the other warps of
    // the two edge strips run the plain march (the edge strips were the slowest blocks, trace
    // in profiles/r2_trace_blocks.txt).  The producer warp's path is the same in both instances.
    const int wx0 = xs4 + warp_id_uniform() * Ghost<G>::kOwn - G;  // float4 column of lane 0
    const bool diri = (wx0 <= 0 && 0 < wx0 + 32) || (wx0 <= p.nx4 - 1 && p.nx4 - 1 < wx0 + 32);
    const bool pf = top_blk || bot_blk;
    constexpr bool kScaled = UC_SCALED_MARCH && NL == 0;
    bool bad = false;
    if (diri) march_t<T, NL, true, G, false>(p, src, dst, s, g, a, b, acc, ring, full, empty, pf, 0);
    else bad = march_t<T, NL, false, G, kScaled>(p, src, dst, s, g, a, b, acc, ring, full, empty, pf, 0);
    if (kScaled && __syncthreads_or(bad)) {  // a value outside the scaled range: redo unscaled
      if (threadIdx.x == 0) atomicAdd(p.launch_hist + 15, 1ull);  // uc_jacobi_launch_counts()[15]
      const int gi = b - a + 1 + 2 * T;
      if (diri) march_t<T, NL, true, G, false>(p, src, dst, s, g, a, b, acc, ring, full, empty, false, gi);
      else march_t<T, NL, false, G, false>(p, src, dst, s, g, a, b, acc, ring, full, empty, false, gi);
    }
  }
  if (NL == 0 && p.bal_ns != nullptr && T == p.bal_T) {
    // the block's march time (kernel entry to the end of its march: round 1 included, the later
    // rounds not -- the first/last chunks' allowance for them is the static chunk_shrink)
    __syncthreads();
    if (threadIdx.x == 0) p.bal_ns[blockIdx.x] = globaltimer() - t_entry;
  }
  UC_TRACE_AT(2);
  if ((rtop || rbot) && (int)threadIdx.x < p.consumers) {
#if UC_ROUNDS_NOINLINE
    acc += t_rounds_after<T, NL, G>(p, src, dst, par, s, k, rtop, rbot);
#else
    for (int j = 2; j <= T; ++j) {  // consumers only (named barrier 1)
      if (rtop) t_round<T, NL>(p, src, dst, par ^ 1, s, g, k, j, true, false, acc);
      if (rbot) t_round<T, NL>(p, src, dst, par ^ 1, s, g, k, j, false, false, acc);
      UC_TRACE_AT(1 + j);
    }
#endif
  }
  return acc;
}

// t_body for the norm level nl (NL..T), resolved at compile time
template <int T, int NL, int G>
__device__ __forceinline__ double t_body_nl(const JacobiParams& p, uint64_t k, int par, float* ring, uint64_t* full,
                                            uint64_t* empty, int nl) {
  if constexpr (NL < T) {
    if (nl != NL) return t_body_nl<T, NL + 1, G>(p, k, par, ring, full, empty, nl);
  }
  return t_body<T, NL, G>(p, k, par, ring, full, empty);
}

// Balanced chunks: the last block of a timed launch folds every block's march time
// into its rate (rows per ns, smoothed 1:1 with the previous value) and re-cuts each strip's rows
// among its chunks in proportion to the rates of the blocks serving them: sizes in effective rows
// (E = n + 2 shrink, the first/last chunk carrying the static allowance for their boundary rounds),
// water-filled above per-chunk minimums (first/last levels + 1 rows, others levels, +1 of slack
// for the floor of the cumulative cuts), so a non-edge chunk never reaches a halo row.  Thread s
// cuts strip s; scratch: the block's ring (free after its march).
static __device__ __noinline__ void bal_resize(const JacobiParams& p, unsigned char* scratch, size_t scratch_bytes) {
  const int S = p.strips, Q = p.chunks, NG = S * Q;
  if ((size_t)NG * (sizeof(double) + 1) > scratch_bytes) return;  // keep the cuts (tiny rings only)
  double* rt = reinterpret_cast<double*>(scratch);
  unsigned char* pin = scratch + sizeof(double) * NG;
  for (int e = threadIdx.x; e < NG; e += blockDim.x) {
    const int b = p.bal_inv[e];
    const int4 w = p.bal_tab[b];
    const unsigned long long ns = p.bal_ns[b];
    float r = p.bal_rate[b];
    const int rows = w.w - w.z + 1;
    if (ns > 0 && rows > 0) {
      const float smp = (float)rows / (float)ns;
      r = r > 0.f ? 0.5f * (r + smp) : smp;
      p.bal_rate[b] = r;
    }
    rt[e] = r;
    pin[e] = 0;
  }
  __syncthreads();
  const long long E = (long long)p.n + 2LL * p.chunk_shrink;
  for (int s = threadIdx.x; s < S; s += blockDim.x) {
    double* r = rt + (size_t)s * Q;
    unsigned char* pn = pin + (size_t)s * Q;
    bool all = true;
    double msum = 0.0;
    for (int q = 0; q < Q; ++q) {
      all &= r[q] > 0.0;
      msum += Q == 1 ? (double)E : (q == 0 || q == Q - 1) ? (double)(p.chunk_shrink + p.bal_levels + 2)
                                                            : (double)(p.bal_levels + 1);
    }
    if (!all || msum > (double)E) continue;  // no rates yet / no room: keep this strip's cuts
    const auto mn = [&](int q) {
      return Q == 1 ? (double)E : (q == 0 || q == Q - 1) ? (double)(p.chunk_shrink + p.bal_levels + 2)
                                                         : (double)(p.bal_levels + 1);
    };
    double rest = 0.0, rs = 0.0;
    for (bool again = true; again;) {
      again = false;
      rest = (double)E;
      rs = 0.0;
      for (int q = 0; q < Q; ++q) {
        if (pn[q]) rest -= mn(q);
        else rs += r[q];
      }
      for (int q = 0; q < Q; ++q)
        if (!pn[q] && rest * r[q] / rs < mn(q)) pn[q] = 1, again = true;
    }
    double cum = 0.0;
    long long prev = 0;
    for (int q = 0; q < Q; ++q) {
      cum += pn[q] ? mn(q) : rest * r[q] / rs;
      const long long B = q == Q - 1 ? E : (long long)floor(cum + 1e-6);
      const int lo = 1 + (int)max(0LL, min(prev - p.chunk_shrink, (long long)p.n));
      const int hi = (int)max(0LL, min(B - p.chunk_shrink, (long long)p.n));
      UC_CHECK(B >= prev && lo <= hi + 1 && (q == 0 ? lo == 1 : true) && (q == Q - 1 ? hi == p.n : true));
      UC_CHECK(q == 0 || q == Q - 1 || hi - lo + 1 >= p.bal_levels);
      p.bal_tab[p.bal_inv[s * Q + q]] = make_int4(s, q, lo, hi);
      prev = B;
    }
  }
}

// T iterations per launch with G ghost lanes per warp side (T <= 4G).  Device mode: n >= 2T, at
// most one norm round per launch; partial mode and paper-faithful host mode: T = 1 (the host API
// exchanges the halos after the kernel); deep-halo host mode: T per launch, T halo rows exchanged
// by the host API after it (p.deep_halo).  p.part splits a launch into its edge chunks and the
// rest (host overlap: NCCL moves the edge rows while the rest computes).
template <int T, int G>
__global__ void __launch_bounds__(G == 1 ? kMaxBlock + 32 : UC_T8_MAXTHREADS, G == 1 ? UC_T_MINBLOCKS : UC_T8_MINBLOCKS)
    jacobi_t_kernel(const __grid_constant__ JacobiParams p) {
  static_assert(T >= 1 && T <= 4 * G, "a ghost lane covers 4 levels");
  __shared__ double smem[32];
  __shared__ int s_last;
  extern __shared__ __align__(128) unsigned char dyn[];
  const int NS = p.stages;
  uint64_t* full = reinterpret_cast<uint64_t*>(dyn);
  uint64_t* empty = full + NS;
  float* ring = reinterpret_cast<float*>(dyn + ((32 * NS + 127) / 128) * 128);
  if (threadIdx.x == 0) {
    for (int i = 0; i < NS; ++i) {
      mbar_init(full + i, 1);
      mbar_init(empty + i, p.consumers / 32);
    }
    fence_mbar_init();
  }
  __syncthreads();
  const unsigned long long t_entry = globaltimer();
  const uint64_t k = p.k_dev[0];
  const int par = (int)((k + p.k_dev[2]) & 1);
  int nl = 0;  // level (1..T) whose iteration k+nl-1 is a norm iteration
  if (p.norm_every > 0) {
    const uint64_t ne = (uint64_t)p.norm_every;
    const uint64_t first = ((k + ne - 1) / ne) * ne;
    if (first < k + T) nl = (int)(first - k) + 1;
  }
  // the same in every thread, but loaded from memory: broadcast it so the compiler knows the
  // NL dispatch below is warp-uniform (otherwise every shuffle of the march gets a divergence
  // check and every ring wait a reconvergence region)
  nl = __shfl_sync(kFull, nl, 0);
  double acc = 0.0;
  if (nl == 0) t_body<T, 0, G>(p, k, par, ring, full, empty, t_entry);
  else acc = t_body_nl<T, 1, G>(p, k, par, ring, full, empty, nl);
  if (nl > 0) {
    const double t = block_sum(acc, smem);
    if (threadIdx.x == 0) p.partials[p.partial_base + blockIdx.x] = t;
  }
  if (p.part != 0) return;  // split launch: overlap_finish_kernel sums the partials and advances k
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    const unsigned t = atomicAdd(p.done, 1u);
    s_last = (t == gridDim.x - 1);
  }
  __syncthreads();
  if (s_last) {
    __threadfence();
    finish_iteration(p, nl > 0, smem, T);
    if (nl == 0 && p.bal_tab != nullptr && T == p.bal_T) {
      __syncthreads();
      bal_resize(p, reinterpret_cast<unsigned char*>(ring), (size_t)NS * kStageFloats<G> * sizeof(float));
    }
  }
  UC_TRACE_AT(15);
}

}  // namespace uc
