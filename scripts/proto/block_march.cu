// Prototype harness (A/B measurement, not the product): the PRODUCT's T-level staged march
// (multistep.cuh march_t, the block-wide TMA ring with a producer warp) over the interior rows of a
// 16384^2 slab, without the boundary rounds -- a fast-compiling stand-in for jacobi_t_kernel<T, G>
// to measure changes to the march.  Checked bit-exactly against T sweeps of a plain kernel.
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "multistep.cuh"
using namespace uc;

#ifndef PROTO_T
#define PROTO_T 6
#endif
#ifndef PROTO_G
#define PROTO_G 2
#endif

#define CK(x)                                                                      \
  do {                                                                             \
    cudaError_t e_ = (x);                                                          \
    if (e_ != cudaSuccess) {                                                       \
      printf("CUDA %s at %s:%d\n", cudaGetErrorString(e_), __FILE__, __LINE__);   \
      exit(1);                                                                     \
    }                                                                              \
  } while (0)

template <int T, int G>
__global__ void __launch_bounds__(G == 1 ? kMaxBlock + 32 : UC_T8_MAXTHREADS, G == 1 ? UC_T_MINBLOCKS : UC_T8_MINBLOCKS)
    proto_kernel(const JacobiParams p) {
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
  const int s = blockIdx.x % p.strips, q = blockIdx.x / p.strips;
  const GhostLayout g = ghost_layout<G>(p, s);
  int lo, hi;
  chunk_rows(p, q, lo, hi);
  const int a = max(lo, T + 1), b = min(hi, p.n - T);
  double acc = 0.0;
#ifdef PROTO_R1
  const uint64_t k = p.k_dev[0];
  const int par = (int)((k + p.k_dev[2]) & 1);
  if (q == 0) t_round<T, 0>(p, p.slab[par], p.slab[par ^ 1], par ^ 1, s, g, k, 1, true, true, acc);
#endif
  if (a <= b) {
    const int xs4 = s * p.strip4;
    const int wx0 = xs4 + warp_id_uniform() * Ghost<G>::kOwn - G;
    const bool diri = (wx0 <= 0 && 0 < wx0 + 32) || (wx0 <= p.nx4 - 1 && p.nx4 - 1 < wx0 + 32);
    if (diri) march_t<T, 0, true, G>(p, p.slab[0], p.slab[1], s, g, a, b, acc, ring, full, empty, false);
    else march_t<T, 0, false, G>(p, p.slab[0], p.slab[1], s, g, a, b, acc, ring, full, empty, false);
  }
}

__global__ void ref_iter(const float* src, float* dst, int nx, int n) {
  const int x = blockIdx.x * blockDim.x + threadIdx.x;
  const int y = blockIdx.y + 1;
  if (x < 1 || x >= nx - 1 || y > n) return;
  const size_t i = (size_t)y * nx + x;
  dst[i] = __fmul_rn(0.25f, __fadd_rn(__fadd_rn(src[i - 1], src[i + 1]), __fadd_rn(src[i - nx], src[i + nx])));
}

__global__ void init_k(float* a, size_t cnt, unsigned long long seed) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < cnt; i += (size_t)gridDim.x * blockDim.x)
    a[i] = (float)(splitmix64(seed ^ i) >> 40) * (1.0f / 16777216.0f);
}

int main(int argc, char** argv) {
  const int nx = argc > 1 ? atoi(argv[1]) : 16384, n = argc > 2 ? atoi(argv[2]) : 16384;
  const int warps = argc > 3 ? atoi(argv[3]) : (PROTO_G == 2 ? 7 : 8);  // consumer warps per block
  const int NS = argc > 4 ? atoi(argv[4]) : 8;
  int chunks = argc > 5 ? atoi(argv[5]) : 0;
  const int T = PROTO_T, G = PROTO_G;
  const size_t cnt = (size_t)(n + 2) * nx;
  float *A, *B, *R1, *R2;
  CK(cudaMalloc(&A, cnt * 4));
  CK(cudaMalloc(&B, cnt * 4));
  CK(cudaMalloc(&R1, cnt * 4));
  CK(cudaMalloc(&R2, cnt * 4));
  init_k<<<1184, 256>>>(A, cnt, 0x5EEDull);
  CK(cudaMemcpy(B, A, cnt * 4, cudaMemcpyDeviceToDevice));
  CK(cudaMemcpy(R1, A, cnt * 4, cudaMemcpyDeviceToDevice));
  CK(cudaMemcpy(R2, A, cnt * 4, cudaMemcpyDeviceToDevice));
  const int nx4 = nx / 4, own = 32 - 2 * G;
  const int st = (nx4 + own * warps - 1) / (own * warps);
  const int strip4 = (nx4 + st - 1) / st;
  const int nc = 32 * ((strip4 + own - 1) / own);
  const int strips = (nx4 + strip4 - 1) / strip4;
#if UC_MARCH_GROUPED
  const size_t smem = (size_t)((32 * NS + 127) / 128) * 128 + (size_t)NS * kStageFloats<PROTO_G> * sizeof(float);
#else
  const size_t smem = (size_t)((32 * NS + 127) / 128) * 128 + (size_t)NS * (4 * nc + 8 * G) * sizeof(float);
#endif
  auto kern = proto_kernel<PROTO_T, PROTO_G>;
  CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int bps = 0;
  const int XT = 32;  // the producer warp
  CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, kern, nc + XT, smem));
  cudaFuncAttributes fa;
  CK(cudaFuncGetAttributes(&fa, kern));
  if (chunks <= 0) chunks = (148 * bps) / strips;
  JacobiParams p{};
  p.slab[0] = A;
  p.slab[1] = B;
  p.nx = nx;
  p.n = n;
  p.nx4 = nx4;
  p.strip4 = strip4;
  p.strips = strips;
  p.chunks = chunks;
  p.consumers = nc;
  p.stages = NS;
  p.ghosts = G;
  const int grid = strips * chunks;
  float *s = R1, *d = R2;
  for (int t = 0; t < T; ++t) {
    ref_iter<<<dim3((nx + 255) / 256, n), 256>>>(s, d, nx, n);
    float* x = s;
    s = d;
    d = x;
  }
#ifdef PROTO_FULL
  // the product kernel itself, P = 1 dirichlet chain (boundary rounds with fixed halo rows, no
  // waits, no puts), the product's chunk shrink
  unsigned long long *k_dev, *hist;
  unsigned int* done;
  double *parts, *rsum, *nh;
  CK(cudaMalloc(&k_dev, 64));
  CK(cudaMemset(k_dev, 0, 64));
  CK(cudaMalloc(&hist, 128));
  CK(cudaMemset(hist, 0, 128));
  CK(cudaMalloc(&done, 64));
  CK(cudaMemset(done, 0, 64));
  CK(cudaMalloc(&parts, 8 * 4096));
  CK(cudaMalloc(&rsum, 64));
  CK(cudaMalloc(&nh, 8 * 4096));
  p.k_dev = k_dev;
  p.launch_hist = hist;
  p.done = done;
  p.work = done + 1;
  p.nbar = done + 2;
  p.partials = parts;
  p.rank_sum = rsum;
  p.norm_hist = nh;
  p.norm_cap = 4096;
  p.device_mode = 1;
  p.size = 1;
  p.flag_half = strips;
  int shrink = getenv("PROTO_SHRINK") ? atoi(getenv("PROTO_SHRINK")) : (T > 4 ? 80 * (T - 2) : 40 * T);
  while (shrink > 0 && (n + 2 * shrink) / chunks - shrink < T + 1) --shrink;
  p.chunk_shrink = shrink;
  auto fk = jacobi_t_kernel<PROTO_T, PROTO_G>;
  CK(cudaFuncSetAttribute(fk, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  CK(cudaFuncGetAttributes(&fa, fk));
#define KLAUNCH fk<<<grid, nc + XT, smem>>>(p)
#else
#define KLAUNCH kern<<<grid, nc + XT, smem>>>(p)
#endif
  KLAUNCH;
  CK(cudaGetLastError());
  CK(cudaDeviceSynchronize());
  std::vector<unsigned> hb(cnt), hr(cnt);
  CK(cudaMemcpy(hb.data(), B, cnt * 4, cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(hr.data(), s, cnt * 4, cudaMemcpyDeviceToHost));
  size_t bad = 0;
  for (int y = T + 1; y <= n - T; ++y)
    for (int x = 0; x < nx; ++x) {
      const size_t i = (size_t)y * nx + x;
      bad += hb[i] != hr[i];
    }
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  for (int w = 0; w < 3; ++w) KLAUNCH;
  const int reps = 20;
  cudaEventRecord(e0);
  for (int r = 0; r < reps; ++r) KLAUNCH;
  cudaEventRecord(e1);
  CK(cudaEventSynchronize(e1));
  float ms = 0;
  cudaEventElapsedTime(&ms, e0, e1);
  ms /= reps;
  const double pts = (double)n * (nx - 2);
  printf("{\"tag\": \"%s\", \"T\": %d, \"G\": %d, \"warps\": %d, \"NS\": %d, \"regs\": %d, \"spill\": %d, \"bps\": %d, "
         "\"grid\": %d, \"strips\": %d, \"chunks\": %d, \"shrink\": \"%s\", \"ms\": %.5f, \"GBs\": %.1f, \"glups\": %.1f, \"bad\": %zu}\n",
         argc > 6 ? argv[6] : "", T, G, warps, NS, fa.numRegs, (int)fa.localSizeBytes, bps, grid, strips, chunks, getenv("PROTO_SHRINK") ? getenv("PROTO_SHRINK") : "-", ms,
         8.0 * pts / (ms * 1e-3) / 1e9, pts * T / (ms * 1e-3) / 1e9, bad);
  return bad ? 2 : 0;
}
