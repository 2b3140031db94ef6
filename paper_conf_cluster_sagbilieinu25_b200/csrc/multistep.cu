// multistep.cu -- kernel variant 5 of libuniconn_b200, G = 1 ghost lane per warp side (T = 1..4
// iterations per launch), and the host-side dispatch of both ghost layouts (multistep_g2.cu:
// G = 2, T = 1..8).  (§VI-C stencil; Listing 3 P:52-74 halo exchange.)
#include "multistep.cuh"

namespace uc {

size_t multistep_smem_bytes(int consumers, int stages, int ghosts) {
  // [full mbarriers][empty mbarriers] padded to 128 B, then the row ring (4G halo floats per side)
#if UC_MARCH_GROUPED
  (void)consumers;  // compile-time ring stride: the widest row the launch bounds allow
  const size_t row = ghosts == 2 ? kStageFloats<2> : kStageFloats<1>;
#else
  const size_t row = (size_t)(4 * consumers + 8 * ghosts);
#endif
  return (size_t)((32 * stages + 127) / 128) * 128 + (size_t)stages * row * sizeof(float);
}

// Host-overlap split launch (part 1 = edge chunks, part 2 = the rest): after the join, one block
// sums the block partials of both parts in index order (norm launches) and advances the
// iteration counter, as the last block of an unsplit launch does (finish_iteration).
__global__ void overlap_finish_kernel(const JacobiParams p, int T, int nparts) {
  __shared__ double smem[32];
  const uint64_t k = p.k_dev[0];
  bool nl = false;
  if (p.norm_every > 0) {
    const uint64_t ne = (uint64_t)p.norm_every;
    nl = ((k + ne - 1) / ne) * ne < k + (uint64_t)T;
  }
  double v = 0.0;
  if (nl)
    for (int i = threadIdx.x; i < nparts; i += blockDim.x) v += p.partials[i];
  const double tot = block_sum(v, smem);
  if (threadIdx.x == 0) {
    if (nl) *p.rank_sum = tot;
    p.k_dev[0] = k + (unsigned long long)T;
    if ((T & 1) == 0) p.k_dev[2] = p.k_dev[2] ^ 1ull;
    p.launch_hist[T < 15 ? T : 15] += 1ull;
    __threadfence();
  }
}

// CPU-free convergence loop (uc_jacobi_solve): the last node of the WHILE body.  The period just
// run had its norm round on its first iteration (norm_hist[m-1], identical on every rank: the
// cross-rank sums are rank-ordered); continue while !(norm < tol) and fewer than kmax iterations.
__global__ void solve_check_kernel(const double* norm_hist, int norm_cap, const unsigned long long* k_dev, double tol,
                                   unsigned long long kmax, cudaGraphConditionalHandle h, double* last) {
  const unsigned long long m = k_dev[1];
  const double nrm = m > 0 ? norm_hist[(m - 1) % (unsigned long long)norm_cap] : 0.0;
  *last = nrm;
  cudaGraphSetConditional(h, (!(nrm < tol) && k_dev[0] < kmax) ? 1u : 0u);
}

int launch_solve_check(const double* norm_hist, int norm_cap, const unsigned long long* k_dev, double tol,
                       unsigned long long kmax, cudaGraphConditionalHandle h, double* last, cudaStream_t s) {
  solve_check_kernel<<<1, 1, 0, s>>>(norm_hist, norm_cap, k_dev, tol, kmax, h, last);
  UC_CUDA(cudaGetLastError());
  return UC_OK;
}

int launch_overlap_finish(const JacobiParams& p, int T, int nparts, cudaStream_t s) {
  overlap_finish_kernel<<<1, 256, 0, s>>>(p, T, nparts);
  UC_CUDA(cudaGetLastError());
  return UC_OK;
}

int launch_jacobi_t(const JacobiParams& p, int grid, int block, int T, cudaStream_t s) {
  const size_t smem = multistep_smem_bytes(p.consumers, p.stages, p.ghosts);
  if (p.ghosts == 2) return launch_jacobi_t_g2(p, grid, block, T, smem, s);
  if (p.ghosts != 1) return fail(UC_ERR_ARG, "%d ghost lanes per warp side not in 1..2", p.ghosts);
  switch (T) {
    case 1: jacobi_t_kernel<1, 1><<<grid, block, smem, s>>>(p); break;
    case 2: jacobi_t_kernel<2, 1><<<grid, block, smem, s>>>(p); break;
    case 3: jacobi_t_kernel<3, 1><<<grid, block, smem, s>>>(p); break;
    case 4: jacobi_t_kernel<4, 1><<<grid, block, smem, s>>>(p); break;
    default: return fail(UC_ERR_ARG, "T = %d iterations per launch not in 1..4 (one ghost lane)", T);
  }
  UC_CUDA(cudaGetLastError());
  return UC_OK;
}

int preload_multistep() {
  const void* fns[] = {(const void*)jacobi_t_kernel<1, 1>, (const void*)jacobi_t_kernel<2, 1>,
                       (const void*)jacobi_t_kernel<3, 1>, (const void*)jacobi_t_kernel<4, 1>};
  for (const void* f : fns) {
    UC_CUDA(cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
    cudaFuncAttributes a;
    UC_CUDA(cudaFuncGetAttributes(&a, f));
  }
  return preload_multistep_g2();
}

// ring stages of variant 5 must be a multiple of this (the grouped march), 1 = any
int multistep_stage_group() { return UC_MARCH_GROUPED ? kGroup : 1; }

int multistep_max_consumers(int ghosts) { return ghosts == 2 ? kMaxBlockG2 : kMaxBlock; }

int multistep_occupancy(int block, size_t smem, int ghosts, int* blocks_per_sm) {
  if (ghosts == 2) return multistep_occupancy_g2(block, smem, blocks_per_sm);
  UC_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, jacobi_t_kernel<4, 1>, block, smem));
  return UC_OK;
}

}  // namespace uc
