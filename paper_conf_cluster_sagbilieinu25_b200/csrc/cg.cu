// cg.cu -- the paper's second workload: Conjugate Gradient (§VI-D, P:416-436;
// SURVEY §8 f3) on the synthetic 3-D SPD stencil matrices of inputs/cg_gen.py.
//
// Each iteration (textbook CG, oracle/cg.py) needs the whole search direction p for the SpMV --
// the paper gathers it with AllGatherv -- and two dot products reduced over all ranks
// (P:430).  Three kernels per iteration, all scalars on the device (no host round trip, so a
// CUDA graph of many iterations replays exactly):
//   K1 cg_spmv:     q = A p (sub-warp of 4 lanes per CSR row by default, uc_cg_set_launch) fused with the partial p.q; the
//                   last block (ticket) reduces the block partials in order and, in device mode,
//                   runs the one-shot cross-rank allreduce and sets alpha = rr / p.q.
//   K2 cg_update:   x += alpha p, r -= alpha q fused with the partial r.r; the last block
//                   allreduces it, beta = rr_new / rr, rr = rr_new, history[k] = rr_new.
//   K3 cg_pupdate:  p = r + beta p for the local block, stored into the local full-length p AND,
//                   in device mode, straight into every peer's full-length p over NVLink (the
//                   AllGatherv fused into the producer of p); the last block releases "p(k+1)
//                   delivered" flags to every peer.  K1 of the next iteration waits for them.
// Host and partial modes run the same kernels without the peer stores / in-kernel allreduces:
// ncclAllReduce + a 1-thread scalar kernel after K1 and K2, ncclAllGather of p after K3.
// Write-after-read on a peer's p is safe: a rank reaches K3(k) only after K2(k)'s allreduce,
// which needs every rank's r.r partial, computed after that rank's K1(k) finished reading p.
#include <cmath>
#include <vector>

#include "device_api.cuh"
#include "uc_internal.h"

namespace uc {
using namespace dev;

struct CGState {
  double rr, alpha, beta, part;
  unsigned long long k, m;  // iteration, allreduce round
};

struct CGParams {
  const long long* rowptr;
  const int* cols;
  const double* vals;
  long long nloc, row0;
  double *x, *r, *q, *pfull;
  double* peer_pfull[UC_MAX_RANKS];
  uint64_t* pflag_peer[UC_MAX_RANKS];  // peer q's "p delivered" flags [P] (we set index rank)
  uint64_t* pflag_mine;
  double* slot[UC_MAX_RANKS];          // peer q's allreduce slots [2][P]
  uint64_t* sflag[UC_MAX_RANKS];       // peer q's allreduce flags [2][P]
  CGState* st;
  double* partials;
  unsigned int* done;
  double* hist;
  int hist_cap;
  int rank, size, device_mode;
  unsigned long long timeout_ns;
  unsigned int* err;
};

__device__ __forceinline__ double cg_block_sum(double v, double* smem) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5;
  __syncthreads();
  if (lane == 0) smem[w] = v;
  __syncthreads();
  double t = 0.0;
  if (w == 0) {
    t = lane < nw ? smem[lane] : 0.0;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) t += __shfl_xor_sync(0xffffffffu, t, o);
  }
  return t;
}

// one-shot allreduce of one double among all ranks (thread 0 of the last block), rank order
__device__ double cg_allreduce(const CGParams& p, double v) {
  const unsigned long long m = p.st->m;
  const int par = (int)(m & 1);
  for (int q = 0; q < p.size; ++q) st_relaxed_sys_f64(p.slot[q] + par * p.size + p.rank, v);
  __threadfence_system();
  for (int q = 0; q < p.size; ++q) st_release_sys(p.sflag[q] + (size_t)(par * p.size + p.rank) * kFlagStride, m + 1);
  double s = 0.0;
  for (int q = 0; q < p.size; ++q) {
    wait_ge(p.sflag[p.rank] + (size_t)(par * p.size + q) * kFlagStride, m + 1, p.timeout_ns, p.err);
    s += ld_relaxed_sys_f64(p.slot[p.rank] + par * p.size + q);
  }
  p.st->m = m + 1;
  return s;
}

// block partial -> ordered rank sum in the last block (all threads call); returns true in the
// last block's thread 0 with *tot set
__device__ bool cg_finish(const CGParams& p, double acc, double* smem, int* s_last, double* tot) {
  const double t = cg_block_sum(acc, smem);
  if (threadIdx.x == 0) {
    p.partials[blockIdx.x] = t;
    __threadfence();
    *s_last = atomicAdd(p.done, 1u) == gridDim.x - 1;
  }
  __syncthreads();
  if (!*s_last) return false;
  __threadfence();
  double v = 0.0;
  for (int i = threadIdx.x; i < (int)gridDim.x; i += blockDim.x) v += p.partials[i];
  const double s = cg_block_sum(v, smem);
  if (threadIdx.x != 0) return false;
  *p.done = 0;
  *tot = s;
  return true;
}

// CSR SpMV with TPR lanes per row and U rows in flight per lane group (memory-level
// parallelism for the dependent col -> p gathers); row sums reduced by shuffles in lane order.
template <int TPR, int U>
__global__ void __launch_bounds__(256) cg_spmv_kernel(const CGParams p) {
  __shared__ double smem[32];
  __shared__ int s_last;
  const unsigned long long k = p.st->k;
  if (p.device_mode == 1) {  // every rank's block of p(k) must have landed in our full p
    if (threadIdx.x == 0)
      for (int q = 0; q < p.size; ++q) wait_ge(p.pflag_mine + (size_t)q * kFlagStride, k, p.timeout_ns, p.err);
    __syncthreads();
  }
  const int sub = threadIdx.x % TPR;
  const unsigned mask = (TPR == 32 ? 0xffffffffu : ((1u << TPR) - 1u)) << ((threadIdx.x & 31) & ~(TPR - 1));
  const long long groups = (long long)gridDim.x * blockDim.x / TPR;
  const double* __restrict__ pf = p.pfull;
  double acc = 0.0;
  for (long long base = (blockIdx.x * (long long)blockDim.x + threadIdx.x) / TPR; base < p.nloc;
       base += groups * U) {
    long long a[U], b[U];
    double s[U];
    long long len = 0;
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const long long row = base + u * groups;
      a[u] = b[u] = 0;
      if (row < p.nloc) {
        a[u] = __ldg(p.rowptr + row);
        b[u] = __ldg(p.rowptr + row + 1);
      }
      s[u] = 0.0;
      len = max(len, b[u] - a[u]);
    }
    // Rows of up to 32 nonzeros (every stencil row here) in one unrolled sweep: all the
    // (value, column) loads first, then all the p gathers, so each lane has PASSES*U
    // independent load chains in flight instead of one per pass.  Read-only path with L1
    // allocation: a lane group's passes walk consecutive pieces of the same 128-byte lines
    // (L1::no_allocate measured 40 % slower).  Longer rows fall through to the general loop.
    constexpr int PASSES = 32 / TPR;
    double v[PASSES][U];
    int c[PASSES][U];
#pragma unroll
    for (int t = 0; t < PASSES; ++t)
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const long long j = a[u] + sub + t * TPR;
        const bool in = j < b[u];
        v[t][u] = in ? __ldg(p.vals + j) : 0.0;
        c[t][u] = in ? __ldg(p.cols + j) : -1;
      }
#pragma unroll
    for (int t = 0; t < PASSES; ++t)
#pragma unroll
      for (int u = 0; u < U; ++u)
        if (c[t][u] >= 0) s[u] += v[t][u] * __ldg(pf + c[t][u]);
    for (long long off = sub + PASSES * TPR; off < len; off += TPR) {
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const long long j = a[u] + off;
        if (j < b[u]) s[u] += __ldg(p.vals + j) * __ldg(pf + __ldg(p.cols + j));
      }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
#pragma unroll
      for (int o = TPR / 2; o > 0; o >>= 1) s[u] += __shfl_down_sync(mask, s[u], o, TPR);
      const long long row = base + u * groups;
      if (sub == 0 && row < p.nloc) {
        p.q[row] = s[u];
        acc += pf[p.row0 + row] * s[u];
      }
    }
  }
  double tot;
  if (cg_finish(p, acc, smem, &s_last, &tot)) {
    if (p.device_mode == 1) {
      const double pq = cg_allreduce(p, tot);
      p.st->alpha = p.st->rr / pq;
    } else {
      p.st->part = tot;  // host/partial: ncclAllReduce + cg_scalar_kernel(1)
    }
  }
}

__global__ void __launch_bounds__(256) cg_update_kernel(const CGParams p) {
  __shared__ double smem[32];
  __shared__ int s_last;
  const double alpha = p.st->alpha;
  const double* pl = p.pfull + p.row0;
  double acc = 0.0;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < p.nloc;
       i += (long long)gridDim.x * blockDim.x) {
    p.x[i] += alpha * pl[i];
    const double ri = p.r[i] - alpha * p.q[i];
    p.r[i] = ri;
    acc += ri * ri;
  }
  double tot;
  if (cg_finish(p, acc, smem, &s_last, &tot)) {
    if (p.device_mode == 1) {
      const double rr = cg_allreduce(p, tot);
      p.st->beta = rr / p.st->rr;
      p.st->rr = rr;
      p.hist[p.st->k % (unsigned long long)p.hist_cap] = rr;
    } else {
      p.st->part = tot;  // ncclAllReduce + cg_scalar_kernel(2)
    }
  }
}

__global__ void __launch_bounds__(256) cg_pupdate_kernel(const CGParams p) {
  __shared__ int s_last;
  const double beta = p.st->beta;
  double* pl = p.pfull + p.row0;
  const bool put = p.device_mode == 1;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < p.nloc;
       i += (long long)gridDim.x * blockDim.x) {
    const double v = p.r[i] + beta * pl[i];
    pl[i] = v;
    if (put)
      for (int q = 0; q < p.size; ++q)
        if (q != p.rank) p.peer_pfull[q][p.row0 + i] = v;  // AllGatherv fused: NVLink stores
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence_system();
    s_last = atomicAdd(p.done, 1u) == gridDim.x - 1;
  }
  __syncthreads();
  if (s_last && threadIdx.x == 0) {
    __threadfence_system();
    const unsigned long long k1 = p.st->k + 1;
    if (put)
      for (int q = 0; q < p.size; ++q) st_release_sys(p.pflag_peer[q] + (size_t)p.rank * kFlagStride, k1);
    p.st->k = k1;
    *p.done = 0;
  }
}

typedef void (*SpmvKernel)(const CGParams);

template <int TPR>
SpmvKernel spmv_for_unroll(int u) {
  return u == 4 ? cg_spmv_kernel<TPR, 4> : u == 2 ? cg_spmv_kernel<TPR, 2> : cg_spmv_kernel<TPR, 1>;
}
// nullptr for unsupported (lanes_per_row in {4, 8, 16, 32}, rows_in_flight in {1, 2, 4})
SpmvKernel spmv_kernel(int tpr, int u) {
  if (u != 1 && u != 2 && u != 4) return nullptr;
  switch (tpr) {
    case 1: return spmv_for_unroll<1>(u);
    case 2: return spmv_for_unroll<2>(u);
    case 4: return spmv_for_unroll<4>(u);
    case 8: return spmv_for_unroll<8>(u);
    case 16: return spmv_for_unroll<16>(u);
    case 32: return spmv_for_unroll<32>(u);
    default: return nullptr;
  }
}

// host/partial mode: finish alpha (which = 1) or beta/rr (which = 2) from the NCCL-reduced part
__global__ void cg_scalar_kernel(CGState* st, double* hist, int hist_cap, int which) {
  if (which == 1) {
    st->alpha = st->rr / st->part;
  } else {
    const double rr = st->part;
    st->beta = rr / st->rr;
    st->rr = rr;
    hist[st->k % (unsigned long long)hist_cap] = rr;
  }
}

}  // namespace uc

// ================================================================================ host side
using namespace uc;

struct uc_cg {
  uc_comm* comm = nullptr;
  int nx = 0, ny = 0, nz = 0, stencil = 27;
  long long N = 0, nloc = 0, row0 = 0, nnz = 0;
  long long* rowptr = nullptr;
  int* cols = nullptr;
  double* vals = nullptr;
  double *x = nullptr, *r = nullptr, *q = nullptr;
  uc_mem* pfull = nullptr;  // symmetric, N doubles
  uc_mem* ctrl = nullptr;   // symmetric: p flags [P] + allreduce flags [2][P] + slots [2][P]
  CGState* st = nullptr;
  double* partials = nullptr;
  unsigned int* done = nullptr;
  double* hist = nullptr;
  double* hist_stage = nullptr;  // page-locked mirror of hist for pageable outputs
  int hist_cap = 65536;
  int grid = 0, spmv_grid = 0, partials_cap = 0;
  // SpMV: lanes per row, rows in flight per lane group.  Round-1 sweep at 160^3, 27-point
  // (profiles/r1_cg_sweep.txt, unrolled-sweep SpMV): 4 x 1 -> 0.318 ms / iteration,
  // 2 x 1 -> 0.370, 8 x 1 -> 0.363, 4 x 2 -> 0.355, 1 x 1 -> 0.523.
  int tpr = 4, unroll = 1;
  long long k = 0;
  int mode = -1;  // launch mode that drives this solver (fixed after the first run)
  cudaStream_t aux = nullptr;
  GraphCache graphs;  // (iters, mode, stream, coordinator, timeout) -> exec
};

namespace {

size_t cg_ctrl_bytes(int P) { return ((size_t)P * kFlagStride + 2 * (size_t)P * kFlagStride + 2 * (size_t)P) * 8; }

CGParams cg_params(const uc_coord* k, const uc_cg* cg) {
  CGParams p{};
  const uc_comm* c = cg->comm;
  const int P = c->size;
  p.rowptr = cg->rowptr;
  p.cols = cg->cols;
  p.vals = cg->vals;
  p.nloc = cg->nloc;
  p.row0 = cg->row0;
  p.x = cg->x;
  p.r = cg->r;
  p.q = cg->q;
  p.pfull = (double*)cg->pfull->local;
  p.device_mode = k->mode == UC_MODE_DEVICE ? 1 : 0;
  for (int q = 0; q < P; ++q) {
    p.peer_pfull[q] = (double*)uc_mem_ptr(cg->pfull, q);
    uint64_t* base = (uint64_t*)uc_mem_ptr(cg->ctrl, q);
    p.pflag_peer[q] = base;
    p.sflag[q] = base ? base + (size_t)P * kFlagStride : nullptr;
    p.slot[q] = base ? (double*)(base + 3 * (size_t)P * kFlagStride) : nullptr;
  }
  p.pflag_mine = (uint64_t*)cg->ctrl->local;
  p.st = cg->st;
  p.partials = cg->partials;
  p.done = cg->done;
  p.hist = cg->hist;
  p.hist_cap = cg->hist_cap;
  p.rank = c->rank;
  p.size = P;
  p.timeout_ns = k->timeout_ns;
  p.err = k->err;
  return p;
}

int cg_enqueue(uc_coord* k, uc_cg* cg) {
  const CGParams p = cg_params(k, cg);
  const bool dev = k->mode == UC_MODE_DEVICE;
  spmv_kernel(cg->tpr, cg->unroll)<<<cg->spmv_grid, 256, 0, k->stream>>>(p);
  UC_CUDA(cudaGetLastError());
  if (!dev) {
    UC_NCCL(ncclAllReduce(&cg->st->part, &cg->st->part, 1, ncclFloat64, ncclSum, k->nccl, k->stream));
    cg_scalar_kernel<<<1, 1, 0, k->stream>>>(cg->st, cg->hist, cg->hist_cap, 1);
    UC_CUDA(cudaGetLastError());
  }
  cg_update_kernel<<<cg->grid, 256, 0, k->stream>>>(p);
  UC_CUDA(cudaGetLastError());
  if (!dev) {
    UC_NCCL(ncclAllReduce(&cg->st->part, &cg->st->part, 1, ncclFloat64, ncclSum, k->nccl, k->stream));
    cg_scalar_kernel<<<1, 1, 0, k->stream>>>(cg->st, cg->hist, cg->hist_cap, 2);
    UC_CUDA(cudaGetLastError());
  }
  cg_pupdate_kernel<<<cg->grid, 256, 0, k->stream>>>(p);
  UC_CUDA(cudaGetLastError());
  if (!dev) {  // AllGatherv of p (equal blocks: ncclAllGather, in place)
    double* pf = (double*)cg->pfull->local;
    UC_NCCL(ncclAllGather(pf + cg->row0, pf, (size_t)cg->nloc, ncclFloat64, k->nccl, k->stream));
  }
  return UC_OK;
}

// Launch geometry: the SpMV variant (lanes per row, rows in flight) and one wave of blocks for
// every kernel; the block-partials buffer is sized for the larger grid.
int cg_configure(uc_cg* cg, int tpr, int unroll) {
  const SpmvKernel f = spmv_kernel(tpr, unroll);
  if (!f)
    return fail(UC_ERR_ARG, "SpMV lanes_per_row %d (1, 2, 4, 8, 16, 32) / rows_in_flight %d (1, 2, 4)", tpr, unroll);
  int sms = 148, bps = 0, bpv = 0;
  UC_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, cg->comm->env->device));
  UC_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, f, 256, 0));
  UC_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bpv, cg_update_kernel, 256, 0));
  const long long groups_needed = (cg->nloc + unroll - 1) / unroll;
  const int sg = (int)std::min<long long>((long long)sms * std::max(1, bps),
                                          std::max<long long>(1, (groups_needed * tpr + 255) / 256));
  const int vg = (int)std::min<long long>((long long)sms * std::max(1, bpv), std::max<long long>(1, (cg->nloc + 255) / 256));
  const int need = std::max(sg, vg);
  if (need > cg->partials_cap) {
    if (cg->partials) cudaFree(cg->partials);
    cg->partials = nullptr;
    UC_CUDA(cudaMalloc(&cg->partials, sizeof(double) * need));
    cg->partials_cap = need;
  }
  cg->tpr = tpr;
  cg->unroll = unroll;
  cg->spmv_grid = sg;
  cg->grid = vg;
  cg->graphs.clear();
  return UC_OK;
}

uint64_t splitmix(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

}  // namespace

extern "C" {

int uc_cg_create(uc_comm* c, int nx, int ny, int nz, int stencil, uint64_t seed, uc_cg** out) {
  if (!c || !out) return fail(UC_ERR_ARG, "NULL argument");
  *out = nullptr;
  if (nx < 1 || ny < 1 || nz < 1) return fail(UC_ERR_ARG, "grid %dx%dx%d", nx, ny, nz);
  if (stencil != 7 && stencil != 27) return fail(UC_ERR_ARG, "stencil must be 7 or 27");
  const long long N = (long long)nx * ny * nz;
  const int P = c->size;
  if (N % P) return fail(UC_ERR_ARG, "N=%lld rows must split equally over %d ranks (P:432)", N, P);
  if (N > 0x7fffffffLL) return fail(UC_ERR_ARG, "N=%lld exceeds 32-bit column indices", N);
  if (c->env->device < 0) return fail(UC_ERR_STATE, "bootstrap-only environment has no device");
  UC_CUDA(cudaSetDevice(c->env->device));
  uc_cg* cg = new uc_cg;
  cg->comm = c;
  cg->nx = nx;
  cg->ny = ny;
  cg->nz = nz;
  cg->stencil = stencil;
  cg->N = N;
  cg->nloc = N / P;
  cg->row0 = (long long)c->rank * cg->nloc;
  auto bail = [&](int rc) {
    if (cg->pfull) uc_mem_free_symmetric(cg->pfull);
    if (cg->ctrl) uc_mem_free_symmetric(cg->ctrl);
    cudaFree(cg->rowptr);
    cudaFree(cg->cols);
    cudaFree(cg->vals);
    cudaFree(cg->x);
    cudaFree(cg->r);
    cudaFree(cg->q);
    cudaFree(cg->st);
    cudaFree(cg->partials);
    cudaFree(cg->done);
    cudaFree(cg->hist);
    if (cg->hist_stage) cudaFreeHost(cg->hist_stage);
    if (cg->aux) cudaStreamDestroy(cg->aux);
    delete cg;
    return rc;
  };
  cudaError_t e = cudaStreamCreateWithFlags(&cg->aux, cudaStreamNonBlocking);
  if (e != cudaSuccess) return bail(fail(UC_ERR_CUDA, "aux stream: %s", cudaGetErrorString(e)));
  // ---- matrix rows of this rank (inputs/cg_gen.py definition), CSR with sorted columns
  std::vector<long long> rowptr(cg->nloc + 1);
  std::vector<int> cols;
  std::vector<double> vals;
  cols.reserve((size_t)cg->nloc * stencil);
  vals.reserve((size_t)cg->nloc * stencil);
  const double diag = stencil == 27 ? 26.0 : 6.0;
  rowptr[0] = 0;
  for (long long i = 0; i < cg->nloc; ++i) {
    const long long g = cg->row0 + i;
    const int x = (int)(g % nx), y = (int)((g / nx) % ny), z = (int)(g / ((long long)nx * ny));
    for (int dz = -1; dz <= 1; ++dz)
      for (int dy = -1; dy <= 1; ++dy)
        for (int dx = -1; dx <= 1; ++dx) {
          const int taxi = (dx != 0) + (dy != 0) + (dz != 0);
          if (stencil == 7 && taxi > 1) continue;
          const int xx = x + dx, yy = y + dy, zz = z + dz;
          if (xx < 0 || xx >= nx || yy < 0 || yy >= ny || zz < 0 || zz >= nz) continue;
          cols.push_back((int)(xx + (long long)nx * (yy + (long long)ny * zz)));
          vals.push_back(taxi == 0 ? diag : -1.0);
        }
    rowptr[i + 1] = (long long)cols.size();
  }
  cg->nnz = (long long)cols.size();
  // ---- b (53-bit splitmix64 values), x0 = 0, r0 = p0 = b (full-length p on every rank)
  std::vector<double> b((size_t)N);
  for (long long g = 0; g < N; ++g) b[g] = (double)(splitmix(seed ^ (uint64_t)g) >> 11) * 0x1p-53;
  double rr0 = 0.0;
  for (long long g = 0; g < N; ++g) rr0 += b[g] * b[g];
  int rc = uc_mem_alloc_symmetric(c, (size_t)N * 8, &cg->pfull);
  if (rc != UC_OK) return bail(rc);
  rc = uc_mem_alloc_symmetric(c, cg_ctrl_bytes(P), &cg->ctrl);
  if (rc != UC_OK) return bail(rc);
  rc = cg_configure(cg, cg->tpr, cg->unroll);
  if (rc != UC_OK) return bail(rc);
  e = cudaMalloc(&cg->rowptr, sizeof(long long) * rowptr.size());
  if (e == cudaSuccess) e = cudaMalloc(&cg->cols, sizeof(int) * std::max<size_t>(1, cols.size()));
  if (e == cudaSuccess) e = cudaMalloc(&cg->vals, sizeof(double) * std::max<size_t>(1, vals.size()));
  if (e == cudaSuccess) e = cudaMalloc(&cg->x, sizeof(double) * cg->nloc);
  if (e == cudaSuccess) e = cudaMalloc(&cg->r, sizeof(double) * cg->nloc);
  if (e == cudaSuccess) e = cudaMalloc(&cg->q, sizeof(double) * cg->nloc);
  if (e == cudaSuccess) e = cudaMalloc(&cg->st, sizeof(CGState));
  if (e == cudaSuccess) e = cudaMalloc(&cg->done, sizeof(unsigned int));
  if (e == cudaSuccess) e = cudaMalloc(&cg->hist, sizeof(double) * cg->hist_cap);
  if (e == cudaSuccess) e = cudaHostAlloc((void**)&cg->hist_stage, sizeof(double) * cg->hist_cap, cudaHostAllocDefault);
  if (e != cudaSuccess) return bail(fail(UC_ERR_OOM, "CG state: %s", cudaGetErrorString(e)));
  CGState st0{rr0, 0.0, 0.0, 0.0, 0ull, 0ull};
  cudaStream_t s = cg->aux;
  e = cudaMemcpyAsync(cg->rowptr, rowptr.data(), sizeof(long long) * rowptr.size(), cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess && !cols.empty())
    e = cudaMemcpyAsync(cg->cols, cols.data(), sizeof(int) * cols.size(), cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess && !vals.empty())
    e = cudaMemcpyAsync(cg->vals, vals.data(), sizeof(double) * vals.size(), cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess) e = cudaMemsetAsync(cg->x, 0, sizeof(double) * cg->nloc, s);
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(cg->r, b.data() + cg->row0, sizeof(double) * cg->nloc, cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess) e = cudaMemcpyAsync(cg->pfull->local, b.data(), sizeof(double) * N, cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess) e = cudaMemcpyAsync(cg->st, &st0, sizeof st0, cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess) e = cudaMemsetAsync(cg->done, 0, sizeof(unsigned int), s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return bail(fail(UC_ERR_CUDA, "CG upload: %s", cudaGetErrorString(e)));
  rc = uc_comm_barrier(c, nullptr);  // every rank's p is in place before anyone puts into it
  if (rc != UC_OK) return bail(rc);
  c->live_objects++;
  *out = cg;
  return UC_OK;
}

int uc_cg_run(uc_coord* k, uc_cg* cg, int iters, double* rr_out, int use_graph) {
  if (!k || !cg) return fail(UC_ERR_ARG, "NULL argument");
  if (k->comm != cg->comm) return fail(UC_ERR_ARG, "coordinator and solver belong to different communicators");
  if (iters < 0 || iters > cg->hist_cap) return fail(UC_ERR_ARG, "iters %d not in [0, %d]", iters, cg->hist_cap);
  UC_CUDA(cudaSetDevice(cg->comm->env->device));
  if (iters == 0) return UC_OK;
  // the "p delivered" flags only advance in device mode: one solver, one launch mode
  if (cg->mode >= 0 && (cg->mode == UC_MODE_DEVICE) != (k->mode == UC_MODE_DEVICE))
    return fail(UC_ERR_STATE, "a CG solver cannot switch between device and host/partial launch modes");
  cg->mode = (int)k->mode;
  if (k->mode != UC_MODE_DEVICE) UC_TRY(ensure_nccl(k));
  if (use_graph && k->stream) {
    JacobiGraph* g = nullptr;
    for (auto& x : cg->graphs.graphs)
      if (x.iters == iters && x.mode == (int)k->mode && x.stream == k->stream && x.coord == k &&
          x.timeout_ns == k->timeout_ns)
        g = &x;
    if (!g) {
      UC_CUDA(cudaStreamBeginCapture(k->stream, cudaStreamCaptureModeThreadLocal));
      int rc = UC_OK;
      for (int i = 0; i < iters && rc == UC_OK; ++i) rc = cg_enqueue(k, cg);
      cudaGraph_t graph = nullptr;
      cudaError_t e = cudaStreamEndCapture(k->stream, &graph);
      if (rc != UC_OK) {
        if (graph) cudaGraphDestroy(graph);
        return rc;
      }
      if (e != cudaSuccess) return fail(UC_ERR_CUDA, "graph capture: %s", cudaGetErrorString(e));
      JacobiGraph ng;
      ng.iters = iters;
      ng.mode = (int)k->mode;
      ng.stream = k->stream;
      ng.coord = k;
      ng.timeout_ns = k->timeout_ns;
      e = cudaGraphInstantiate(&ng.exec, graph, 0);
      cudaGraphDestroy(graph);
      if (e == cudaSuccess) e = cudaGraphUpload(ng.exec, k->stream);
      if (e == cudaSuccess) e = cudaStreamSynchronize(k->stream);
      if (e != cudaSuccess) return fail(UC_ERR_CUDA, "graph build: %s", cudaGetErrorString(e));
      cg->graphs.add(k, ng);
      g = &cg->graphs.graphs.back();
      UC_TRY(uc_comm_barrier(cg->comm, k->stream));  // building a graph is collective (see Jacobi)
    }
    UC_CUDA(cudaGraphLaunch(g->exec, k->stream));
  } else {
    for (int i = 0; i < iters; ++i) UC_TRY(cg_enqueue(k, cg));
  }
  if (rr_out) {
    const long long k0 = cg->k;
    int done = 0;
    while (done < iters) {
      const int idx = (int)((k0 + done) % cg->hist_cap);
      const int len = std::min(iters - done, cg->hist_cap - idx);
      UC_TRY(enqueue_d2h_f64(k, rr_out + done, cg->hist + idx, cg->hist_stage + idx, (size_t)len));
      done += len;
    }
  }
  cg->k += iters;
  return UC_OK;
}

int uc_cg_copy_x(uc_coord* k, uc_cg* cg, double* host_x) {
  if (!k || !cg || !host_x) return fail(UC_ERR_ARG, "NULL argument");
  UC_CUDA(cudaSetDevice(cg->comm->env->device));
  UC_CUDA(cudaMemcpyAsync(host_x, cg->x, sizeof(double) * cg->nloc, cudaMemcpyDeviceToHost, k->stream));
  UC_CUDA(cudaStreamSynchronize(k->stream));
  return UC_OK;
}

int uc_cg_info(const uc_cg* cg, int64_t* n_global, int64_t* n_local, int64_t* row0, int64_t* nnz_local,
               int64_t* iteration) {
  if (!cg) return fail(UC_ERR_ARG, "solver is NULL");
  if (n_global) *n_global = cg->N;
  if (n_local) *n_local = cg->nloc;
  if (row0) *row0 = cg->row0;
  if (nnz_local) *nnz_local = cg->nnz;
  if (iteration) *iteration = cg->k;
  return UC_OK;
}

int uc_cg_set_launch(uc_cg* cg, int lanes_per_row, int rows_in_flight) {
  if (!cg) return fail(UC_ERR_ARG, "solver is NULL");
  UC_CUDA(cudaSetDevice(cg->comm->env->device));
  UC_CUDA(cudaDeviceSynchronize());
  return cg_configure(cg, lanes_per_row > 0 ? lanes_per_row : 4, rows_in_flight > 0 ? rows_in_flight : 1);
}

int uc_cg_destroy(uc_cg* cg) {
  if (!cg) return fail(UC_ERR_ARG, "solver is NULL");
  uc_comm* c = cg->comm;
  UC_CUDA(cudaSetDevice(c->env->device));
  UC_CUDA(cudaStreamSynchronize(cg->aux));
  cg->graphs.release();
  UC_TRY(uc_mem_free_symmetric(cg->pfull));
  UC_TRY(uc_mem_free_symmetric(cg->ctrl));
  cudaFree(cg->rowptr);
  cudaFree(cg->cols);
  cudaFree(cg->vals);
  cudaFree(cg->x);
  cudaFree(cg->r);
  cudaFree(cg->q);
  cudaFree(cg->st);
  cudaFree(cg->partials);
  cudaFree(cg->done);
  cudaFree(cg->hist);
  if (cg->hist_stage) cudaFreeHost(cg->hist_stage);
  cudaStreamDestroy(cg->aux);
  c->live_objects--;
  delete cg;
  return UC_OK;
}

}  // extern "C"

namespace uc {
int preload_cg_kernels() {
  std::vector<const void*> fns = {(const void*)cg_update_kernel, (const void*)cg_pupdate_kernel,
                                  (const void*)cg_scalar_kernel};
  for (int tpr : {1, 2, 4, 8, 16, 32})
    for (int u : {1, 2, 4}) fns.push_back((const void*)spmv_kernel(tpr, u));
  for (const void* f : fns) {
    cudaFuncAttributes a;
    UC_CUDA(cudaFuncGetAttributes(&a, f));
  }
  return UC_OK;
}
}  // namespace uc
