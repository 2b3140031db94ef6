// multistep_g2b.cu -- kernel variant 5 of libuniconn_b200 with G = 2 ghost lanes per warp side,
// the deep instances T = 6, 7 (multistep.cuh; T = 1..5 in multistep_g2.cu, T = 8 in multistep_g2c.cu).
#include "multistep.cuh"

namespace uc {

int launch_jacobi_t_g2b(const JacobiParams& p, int grid, int block, int T, size_t smem, cudaStream_t s) {
  switch (T) {
    case 6: jacobi_t_kernel<6, 2><<<grid, block, smem, s>>>(p); break;
    case 7: jacobi_t_kernel<7, 2><<<grid, block, smem, s>>>(p); break;
    case 8: return launch_jacobi_t_g2c(p, grid, block, smem, s);
    default: return fail(UC_ERR_ARG, "T = %d iterations per launch not in 6..8", T);
  }
  UC_CUDA(cudaGetLastError());
  return UC_OK;
}

int preload_multistep_g2b() {
  const void* fns[] = {(const void*)jacobi_t_kernel<6, 2>, (const void*)jacobi_t_kernel<7, 2>};
  for (const void* f : fns) {
    UC_CUDA(cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
    cudaFuncAttributes a;
    UC_CUDA(cudaFuncGetAttributes(&a, f));
  }
  return preload_multistep_g2c();
}

}  // namespace uc
