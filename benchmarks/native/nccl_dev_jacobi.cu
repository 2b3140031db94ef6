// nccl_dev_jacobi.cu -- the Listing-3 structure on NCCL 2.28's device API:
// the in-box "native" comparator of SURVEY §8 f4.  See nccl_dev_jacobi.h.
#include <cuda_runtime.h>
#include <nccl.h>
#include <nccl_device.h>

#include <algorithm>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <string>

#include "nccl_dev_jacobi.h"

namespace {

thread_local std::string g_err;
int fail(int code, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_err = buf;
  return code;
}
#define UCN_CUDA(x)                                                                          \
  do {                                                                                       \
    cudaError_t e_ = (x);                                                                    \
    if (e_ != cudaSuccess) return fail(2, "%s: %s (%s:%d)", #x, cudaGetErrorString(e_), __FILE__, __LINE__); \
  } while (0)
#define UCN_NCCL(x)                                                                          \
  do {                                                                                       \
    ncclResult_t r_ = (x);                                                                   \
    if (r_ != ncclSuccess) return fail(3, "%s: %s (%s:%d)", #x, ncclGetErrorString(r_), __FILE__, __LINE__); \
  } while (0)

constexpr int kThreads = 256;  // one float4 column per thread: a strip is 1024 columns

// Reading G1: 0.25f*((l+r)+(t+b)), round-to-nearest, never contracted, no FTZ.
__device__ __forceinline__ float upd(float l, float r, float t, float b) {
  return __fmul_rn(0.25f, __fadd_rn(__fadd_rn(l, r), __fadd_rn(t, b)));
}

// New values of the 4 columns of float4 column x4 of row y (columns 0 and nx-1 fixed).
__device__ __forceinline__ float4 row_update(const float* src, size_t nx, int y, int x4, int nx4) {
  const float* c = src + (size_t)y * nx;
  const float4 u = reinterpret_cast<const float4*>(c - nx)[x4];
  const float4 m = reinterpret_cast<const float4*>(c)[x4];
  const float4 d = reinterpret_cast<const float4*>(c + nx)[x4];
  const float L = x4 > 0 ? c[4 * x4 - 1] : 0.f;
  const float R = x4 + 1 < nx4 ? c[4 * x4 + 4] : 0.f;
  float4 o;
  o.x = x4 == 0 ? m.x : upd(L, m.y, u.x, d.x);
  o.y = upd(m.x, m.z, u.y, d.y);
  o.z = upd(m.y, m.w, u.z, d.z);
  o.w = x4 == nx4 - 1 ? m.w : upd(m.z, R, u.w, d.w);
  return o;
}

// Blocks [0, strips): the boundary block of strip s (Listing 3's last two blocks): rows 1
// and n, stored locally and into the neighbours' halo rows of the output slab through LSA peer
// pointers, then an LSA barrier (index s) across the ranks, so the next launch's boundary block
// sees its halos (release/acquire) and no rank overwrites a halo row a neighbour still reads.
// Blocks [strips, strips * (1 + chunks)): rows 2..n-1 of (strip, chunk).
__global__ void __launch_bounds__(kThreads) ucn_jacobi_kernel(ncclDevComm dc, ncclWindow_t win, float* base,
                                                              size_t slab_elems, int par, int nx, int n, int top,
                                                              int bottom, int strips, int chunks) {
  const int nx4 = nx / 4;
  const size_t pitch = (size_t)nx;
  const float* src = base + (size_t)par * slab_elems;
  float* dst = base + (size_t)(par ^ 1) * slab_elems;
  const int s = blockIdx.x % strips;
  const int x4 = s * kThreads + (int)threadIdx.x;
  const bool valid = x4 < nx4;
  if ((int)blockIdx.x < strips) {
    if (valid) {
      const float4 o1 = row_update(src, pitch, 1, x4, nx4);
      reinterpret_cast<float4*>(dst + pitch)[x4] = o1;
      float4 on = o1;
      if (n > 1) {
        on = row_update(src, pitch, n, x4, nx4);
        reinterpret_cast<float4*>(dst + (size_t)n * pitch)[x4] = on;
      }
      const size_t out_off = (size_t)(par ^ 1) * slab_elems * sizeof(float);
      if (top >= 0) {  // our row 1 -> top's halo row n+1
        float* p = (float*)ncclGetLsaPointer(win, out_off + (size_t)(n + 1) * pitch * sizeof(float), top);
        reinterpret_cast<float4*>(p)[x4] = o1;
      }
      if (bottom >= 0) {  // our row n -> bottom's halo row 0
        float* p = (float*)ncclGetLsaPointer(win, out_off, bottom);
        reinterpret_cast<float4*>(p)[x4] = on;
      }
    }
    ncclLsaBarrierSession<ncclCoopCta> bar(ncclCoopCta(), dc, ncclTeamTagLsa(), (uint32_t)s);
    bar.sync(ncclCoopCta(), cuda::memory_order_acq_rel);
    return;
  }
  const int q = (int)blockIdx.x / strips - 1;
  const int inner = n - 2;  // rows 2..n-1
  const int y0 = 2 + (int)((long long)q * inner / chunks);
  const int y1 = 2 + (int)((long long)(q + 1) * inner / chunks);
  if (!valid) return;
  for (int y = y0; y < y1; ++y) reinterpret_cast<float4*>(dst + (size_t)y * pitch)[x4] = row_update(src, pitch, y, x4, nx4);
}

}  // namespace

struct ucn_jacobi {
  ncclComm_t comm = nullptr;
  ncclDevComm dev{};
  bool dev_made = false;
  ncclWindow_t win = nullptr;
  float* buf = nullptr;
  int nx = 0, n = 0, top = -1, bottom = -1, rank = 0, nranks = 1;
  size_t slab_elems = 0;
  int strips = 0, chunks = 0;
  long long k = 0;
};

extern "C" {

const char* ucn_last_error(void) { return g_err.c_str(); }

int ucn_unique_id(void* out) {
  if (!out) return fail(1, "null output");
  ncclUniqueId id;
  UCN_NCCL(ncclGetUniqueId(&id));
  std::memcpy(out, &id, sizeof id);
  return 0;
}

int ucn_create(int rank, int nranks, const void* unique_id, int nx, int n, int top, int bottom, ucn_jacobi** out) {
  if (!out || !unique_id || nranks < 1 || rank < 0 || rank >= nranks || nx < 8 || nx % 4 || n < 1 ||
      top < -1 || top >= nranks || bottom < -1 || bottom >= nranks)
    return fail(1, "ucn_create: rank %d of %d, nx %d, n %d, top %d, bottom %d", rank, nranks, nx, n, top, bottom);
  ucn_jacobi* J = new ucn_jacobi;
  J->nx = nx;
  J->n = n;
  J->top = top;
  J->bottom = bottom;
  J->rank = rank;
  J->nranks = nranks;
  J->slab_elems = (size_t)(n + 2) * nx;
  J->strips = (nx / 4 + kThreads - 1) / kThreads;
  J->chunks = n > 2 ? std::max(1, std::min(n - 2, (148 * 8 + J->strips - 1) / J->strips)) : 1;
  ncclUniqueId id;
  std::memcpy(&id, unique_id, sizeof id);
  auto bail = [&](int code) {
    if (J->dev_made) ncclDevCommDestroy(J->comm, &J->dev);
    if (J->win) ncclCommWindowDeregister(J->comm, J->win);
    if (J->buf) ncclMemFree(J->buf);
    if (J->comm) ncclCommDestroy(J->comm);
    delete J;
    return code;
  };
  {
    ncclResult_t r = ncclCommInitRank(&J->comm, nranks, id, rank);
    if (r != ncclSuccess) return bail(fail(3, "ncclCommInitRank: %s", ncclGetErrorString(r)));
    size_t bytes = 2 * J->slab_elems * sizeof(float);
    bytes = (bytes + NCCL_WIN_REQUIRED_ALIGNMENT - 1) / NCCL_WIN_REQUIRED_ALIGNMENT * NCCL_WIN_REQUIRED_ALIGNMENT;
    r = ncclMemAlloc((void**)&J->buf, bytes);
    if (r != ncclSuccess) return bail(fail(3, "ncclMemAlloc(%zu): %s", bytes, ncclGetErrorString(r)));
    r = ncclCommWindowRegister(J->comm, J->buf, bytes, &J->win, NCCL_WIN_COLL_SYMMETRIC);
    if (r != ncclSuccess) return bail(fail(3, "ncclCommWindowRegister: %s", ncclGetErrorString(r)));
    ncclDevCommRequirements reqs;
    std::memset(&reqs, 0, sizeof reqs);
    reqs.lsaBarrierCount = J->strips;
    r = ncclDevCommCreate(J->comm, &reqs, &J->dev);
    if (r != ncclSuccess) return bail(fail(3, "ncclDevCommCreate: %s", ncclGetErrorString(r)));
    J->dev_made = true;
  }
  *out = J;
  return 0;
}

int ucn_copy_in(ucn_jacobi* J, const float* host_slab) {
  if (!J || !host_slab) return fail(1, "null argument");
  for (int b = 0; b < 2; ++b)
    UCN_CUDA(cudaMemcpy(J->buf + b * J->slab_elems, host_slab, J->slab_elems * sizeof(float), cudaMemcpyHostToDevice));
  J->k = 0;
  return 0;
}

int ucn_copy_out(ucn_jacobi* J, float* host_slab) {
  if (!J || !host_slab) return fail(1, "null argument");
  UCN_CUDA(cudaDeviceSynchronize());
  UCN_CUDA(cudaMemcpy(host_slab, J->buf + (size_t)(J->k & 1) * J->slab_elems, J->slab_elems * sizeof(float),
                      cudaMemcpyDeviceToHost));
  return 0;
}

int ucn_run(ucn_jacobi* J, int iters, void* stream) {
  if (!J || iters < 0) return fail(1, "bad argument");
  cudaStream_t s = (cudaStream_t)stream;
  const int grid = J->strips * (1 + (J->n > 2 ? J->chunks : 0));
  for (int i = 0; i < iters; ++i) {
    ucn_jacobi_kernel<<<grid, kThreads, 0, s>>>(J->dev, J->win, J->buf, J->slab_elems, (int)(J->k & 1), J->nx, J->n,
                                                J->top, J->bottom, J->strips, J->n > 2 ? J->chunks : 1);
    UCN_CUDA(cudaGetLastError());
    ++J->k;
  }
  return 0;
}

int ucn_destroy(ucn_jacobi* J) {
  if (!J) return 0;
  cudaDeviceSynchronize();
  if (J->dev_made) UCN_NCCL(ncclDevCommDestroy(J->comm, &J->dev));
  if (J->win) UCN_NCCL(ncclCommWindowDeregister(J->comm, J->win));
  if (J->buf) UCN_NCCL(ncclMemFree(J->buf));
  if (J->comm) UCN_NCCL(ncclCommDestroy(J->comm));
  delete J;
  return 0;
}

}  // extern "C"
