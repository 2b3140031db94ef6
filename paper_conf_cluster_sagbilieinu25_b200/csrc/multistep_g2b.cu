// multistep_g2b.cu -- kernel variant 5 of libuniconn_b200 with G = 2 ghost lanes per warp side,
// the deep instances T = 6, 7 (multistep.cuh; T = 1..5 in multistep_g2.cu, T = 8 in multistep_g2c.cu).
#include <cstring>

#include "multistep.cuh"

namespace uc {

#if UC_TRACE
int set_trace_g2c(unsigned long long* buf);
static unsigned long long* g_trace = nullptr;
}  // namespace uc
extern "C" unsigned long long* uc_debug_trace_buffer() { return uc::g_trace; }
namespace uc {
#endif

int launch_jacobi_t_g2b(const JacobiParams& p, int grid, int block, int T, size_t smem, cudaStream_t s) {
#if UC_TRACE
  if (!g_trace) {
    UC_CUDA(cudaMallocManaged(&g_trace, sizeof(unsigned long long) * 16 * 4096));
    memset(g_trace, 0, sizeof(unsigned long long) * 16 * 4096);
    UC_CUDA(cudaMemcpyToSymbol(uc_trace_ptr, &g_trace, sizeof g_trace));
    if (int e = set_trace_g2c(g_trace)) return e;
  }
#endif
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
