// device_api_ring.cu -- a USER kernel written against the header-only device API
// (include/uniconn_device.cuh) and launched through uc_launch: the paper's point that device-side
// communication is inlined into application kernels with a chosen ThreadGroup
// granularity.
//
// Every rank puts `n` floats (its rank-tagged data, computed in the kernel) into the symmetric
// buffer of its bottom neighbour, signals it, and waits for the data from its top neighbour.
// Built as libuc_device_example.so by build(); uc_example_ring_kernel(g) returns the CUfunction
// of the THREAD (g = 0), WARP (1) or BLOCK (2) variant for uc_launch.
#include <cuda_runtime.h>

#include "uniconn_device.cuh"

// args: float* scratch (local, n), float* dst_bottom (bottom's symmetric buffer), uint64_t*
// sig_bottom (bottom's signal), const uint64_t* sig_mine, int n, int rank, uint64_t round,
// unsigned long long timeout_ns, unsigned int* err
template <int G>
__global__ void ring_kernel(float* scratch, float* dst_bottom, uint64_t* sig_bottom, const uint64_t* sig_mine, int n,
                            int rank, uint64_t round, unsigned long long timeout_ns, unsigned int* err) {
  // one group moves the whole message: THREAD -> thread 0 of block 0, WARP -> warp 0, BLOCK -> block 0
  if (blockIdx.x != 0) return;
  if (G == UC_DEV_THREAD && threadIdx.x != 0) return;
  if (G == UC_DEV_WARP && threadIdx.x >= 32) return;
  for (int i = uc_dev_group_rank<G>(); i < n; i += uc_dev_group_size<G>())
    scratch[i] = (float)(rank * 1000 + (int)round) + 0.5f * (float)i;
  uc_dev_group_sync<G>();
  uc_dev_put_signal<G>(dst_bottom, scratch, (size_t)n * sizeof(float), sig_bottom, round, UC_DEV_SIGNAL_SET);
  if (uc_dev_group_rank<G>() == 0) uc_dev_wait_ge(sig_mine, round, timeout_ns, err);
  uc_dev_group_sync<G>();
}

extern "C" const void* uc_example_ring_kernel(int group) {
  cudaFunction_t f = nullptr;
  const void* sym = group == 0 ? (const void*)ring_kernel<UC_DEV_THREAD>
                  : group == 1 ? (const void*)ring_kernel<UC_DEV_WARP>
                               : (const void*)ring_kernel<UC_DEV_BLOCK>;
  if (cudaGetFuncBySymbol(&f, sym) != cudaSuccess) return nullptr;
  return (const void*)f;
}
