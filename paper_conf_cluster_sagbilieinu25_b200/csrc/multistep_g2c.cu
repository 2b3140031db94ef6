// multistep_g2c.cu -- kernel variant 5 of libuniconn_b200 with G = 2 ghost lanes per warp side,
// the deepest instance T = 8 (multistep.cuh), alone in its translation unit (the longest compile).
#include "multistep.cuh"

namespace uc {

#if UC_TRACE
// every translation unit has its own copy of the trace pointer (multistep.cuh): set this one too
int set_trace_g2c(unsigned long long* buf) {
  UC_CUDA(cudaMemcpyToSymbol(uc_trace_ptr, &buf, sizeof buf));
  return UC_OK;
}
#endif

int launch_jacobi_t_g2c(const JacobiParams& p, int grid, int block, size_t smem, cudaStream_t s) {
  jacobi_t_kernel<8, 2><<<grid, block, smem, s>>>(p);
  UC_CUDA(cudaGetLastError());
  return UC_OK;
}

int preload_multistep_g2c() {
  UC_CUDA(cudaFuncSetAttribute(jacobi_t_kernel<8, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
  cudaFuncAttributes a;
  UC_CUDA(cudaFuncGetAttributes(&a, jacobi_t_kernel<8, 2>));
  return UC_OK;
}

// the deepest instance bounds the geometry of every T of the two-ghost-lane layout
int multistep_occupancy_g2(int block, size_t smem, int* blocks_per_sm) {
  UC_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, jacobi_t_kernel<8, 2>, block, smem));
  return UC_OK;
}

}  // namespace uc
