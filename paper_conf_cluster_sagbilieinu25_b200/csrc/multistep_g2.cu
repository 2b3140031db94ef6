// multistep_g2.cu -- kernel variant 5 of libuniconn_b200 with G = 2 ghost lanes per warp side:
// T = 1..8 Jacobi iterations per launch, 28 owned float4 columns per warp (multistep.cuh).
// T = 1..5 here, T = 6..8 in multistep_g2b.cu: own translation units so the deep instances
// compile in parallel with the rest.
#include "multistep.cuh"

namespace uc {

int launch_jacobi_t_g2(const JacobiParams& p, int grid, int block, int T, size_t smem, cudaStream_t s) {
  switch (T) {
    case 1: jacobi_t_kernel<1, 2><<<grid, block, smem, s>>>(p); break;
    case 2: jacobi_t_kernel<2, 2><<<grid, block, smem, s>>>(p); break;
    case 3: jacobi_t_kernel<3, 2><<<grid, block, smem, s>>>(p); break;
    case 4: jacobi_t_kernel<4, 2><<<grid, block, smem, s>>>(p); break;
    case 5: jacobi_t_kernel<5, 2><<<grid, block, smem, s>>>(p); break;
    case 6:
    case 7:
    case 8: return launch_jacobi_t_g2b(p, grid, block, T, smem, s);
    default: return fail(UC_ERR_ARG, "T = %d iterations per launch not in 1..8 (two ghost lanes)", T);
  }
  UC_CUDA(cudaGetLastError());
  return UC_OK;
}

int preload_multistep_g2() {
  const void* fns[] = {(const void*)jacobi_t_kernel<1, 2>, (const void*)jacobi_t_kernel<2, 2>,
                       (const void*)jacobi_t_kernel<3, 2>, (const void*)jacobi_t_kernel<4, 2>,
                       (const void*)jacobi_t_kernel<5, 2>};
  for (const void* f : fns) {
    UC_CUDA(cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
    cudaFuncAttributes a;
    UC_CUDA(cudaFuncGetAttributes(&a, f));
  }
  return preload_multistep_g2b();
}

}  // namespace uc
