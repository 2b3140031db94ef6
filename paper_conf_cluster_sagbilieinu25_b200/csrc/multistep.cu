// multistep.cu -- kernel variant 5 of libuniconn_b200, G = 1 ghost lane per warp side (T = 1..4
// iterations per launch), and the host-side dispatch of both ghost layouts (multistep_g2.cu:
// G = 2, T = 1..8).  (§VI-C stencil; Listing 3 P:52-74 halo exchange.)
#include "multistep.cuh"

namespace uc {

size_t multistep_smem_bytes(int consumers, int stages, int ghosts) {
  // [full mbarriers][empty mbarriers] padded to 128 B, then the row ring (4G halo floats per side)
  return (size_t)((32 * stages + 127) / 128) * 128 + (size_t)stages * (4 * consumers + 8 * ghosts) * sizeof(float);
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

int multistep_max_consumers(int ghosts) { return ghosts == 2 ? kMaxBlockG2 : kMaxBlock; }

int multistep_occupancy(int block, size_t smem, int ghosts, int* blocks_per_sm) {
  if (ghosts == 2) return multistep_occupancy_g2(block, smem, blocks_per_sm);
  UC_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, jacobi_t_kernel<4, 1>, block, smem));
  return UC_OK;
}

}  // namespace uc
