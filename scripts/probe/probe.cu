// One-shot environment probe for the B200 box (not product code).
// Measures: device properties, float4 copy bandwidth, CUDA IPC between two
// processes on the SAME device, whether a spinning kernel in one process sees
// a flag written by a kernel of another process on the same GPU (time-slicing
// vs concurrency), and NCCL single-rank self send/recv inside a group.
#include <cuda_runtime.h>
#include <nccl.h>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <unistd.h>
#include <sys/wait.h>
#include <chrono>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { \
  printf("CUDA error %s at %s:%d: %s\n", #x, __FILE__, __LINE__, cudaGetErrorString(e)); exit(1);} } while (0)
#define NK(x) do { ncclResult_t e = (x); if (e != ncclSuccess) { \
  printf("NCCL error %s at %s:%d: %s\n", #x, __FILE__, __LINE__, ncclGetErrorString(e)); exit(1);} } while (0)

__global__ void copy4(const float4* __restrict__ a, float4* __restrict__ b, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    b[i] = a[i];
}

__device__ __forceinline__ unsigned long long gtime() {
  unsigned long long t; asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t)); return t;
}
__device__ __forceinline__ unsigned long long ld_acq(const unsigned long long* p) {
  unsigned long long v; asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory"); return v;
}
__device__ __forceinline__ void st_rel(unsigned long long* p, unsigned long long v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" :: "l"(p), "l"(v) : "memory");
}
__global__ void spin_until(const unsigned long long* flag, unsigned long long v, unsigned long long timeout_ns,
                           unsigned long long* out_ns) {
  unsigned long long t0 = gtime();
  while (ld_acq(flag) < v) { if (gtime() - t0 > timeout_ns) { *out_ns = ~0ull; return; } }
  *out_ns = gtime() - t0;
}
__global__ void set_flag(unsigned long long* flag, unsigned long long v) { st_rel(flag, v); }

int main(int argc, char** argv) {
  setvbuf(stdout, NULL, _IONBF, 0);
  bool do_ipc = argc > 1 && !strcmp(argv[1], "ipc");
  int p2c[2], c2p[2];
  if (do_ipc) {
  if (pipe(p2c) || pipe(c2p)) return 1;
  pid_t pid = fork();
  if (pid == 0) {
    cudaIpcMemHandle_t h;
    if (read(p2c[0], &h, sizeof h) != sizeof h) return 2;
    CK(cudaSetDevice(0));
    void* p = nullptr;
    cudaError_t e = cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess);
    int ok = (e == cudaSuccess);
    if (!ok) printf("[child] cudaIpcOpenMemHandle failed: %s\n", cudaGetErrorString(e));
    if (write(c2p[1], &ok, sizeof ok) != sizeof ok) return 3;
    if (ok) {
      int go; if (read(p2c[0], &go, sizeof go) != sizeof go) return 4;
      usleep(200000);
      set_flag<<<1, 1>>>((unsigned long long*)p, 7);
      CK(cudaDeviceSynchronize());
      CK(cudaIpcCloseMemHandle(p));
    }
    return 0;
  }
  CK(cudaSetDevice(0));
  cudaDeviceProp prop; CK(cudaGetDeviceProperties(&prop, 0));
  printf("device %s sm_%d%d SMs=%d L2=%d MB smemPerBlockOptin=%zu KB regsPerSM=%d memBusWidth=%d\n",
         prop.name, prop.major, prop.minor, prop.multiProcessorCount, prop.l2CacheSize >> 20,
         prop.sharedMemPerBlockOptin >> 10, prop.regsPerMultiprocessor, prop.memoryBusWidth);
  unsigned long long *flag, *out;
  CK(cudaMalloc(&flag, 256)); CK(cudaMemset(flag, 0, 256));
  CK(cudaMallocManaged(&out, 8));
  cudaIpcMemHandle_t h; CK(cudaIpcGetMemHandle(&h, flag));
  if (write(p2c[1], &h, sizeof h) != sizeof h) return 5;
  int ok = 0; if (read(c2p[0], &ok, sizeof ok) != sizeof ok) return 6;
  printf("IPC open in second process on same device: %s\n", ok ? "OK" : "FAILED");
  if (ok) {
    spin_until<<<1, 1>>>(flag, 7, 5000000000ull, out);
    int go = 1; if (write(p2c[1], &go, sizeof go) != sizeof go) return 7;
    CK(cudaDeviceSynchronize());
    if (*out == ~0ull) printf("cross-process spin: TIMEOUT after 5 s (no concurrency)\n");
    else printf("cross-process spin: saw flag after %.3f ms (child sleeps 200 ms first)\n", *out / 1e6);
  }
  int st; waitpid(pid, &st, 0);
  return 0;
  }
  CK(cudaSetDevice(0));
  { cudaDeviceProp prop; CK(cudaGetDeviceProperties(&prop, 0));
  printf("device %s SMs=%d L2=%d MB\n", prop.name, prop.multiProcessorCount, prop.l2CacheSize >> 20); }

  // ---------------- copy bandwidth
  size_t n = (size_t)1 << 28;  // 1 GiB of floats
  float4 *a, *b; CK(cudaMalloc(&a, n * 4)); CK(cudaMalloc(&b, n * 4));
  CK(cudaMemset(a, 0, n * 4));
  cudaEvent_t e0, e1; CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
  for (int blocks : {148 * 4, 148 * 8, 148 * 16, 148 * 64}) {
    float best = 1e9;
    for (int r = 0; r < 10; ++r) {
      CK(cudaEventRecord(e0)); copy4<<<blocks, 256>>>(a, b, n / 4); CK(cudaEventRecord(e1));
      CK(cudaEventSynchronize(e1)); float ms; CK(cudaEventElapsedTime(&ms, e0, e1)); if (ms < best) best = ms;
    }
    printf("float4 copy 1 GiB grid=%d: %.3f ms -> %.1f GB/s (read+write)\n", blocks, best, 2.0 * n * 4 / best / 1e6);
  }
  {
    float best = 1e9;
    for (int r = 0; r < 10; ++r) {
      CK(cudaEventRecord(e0)); CK(cudaMemcpyAsync(b, a, n * 4, cudaMemcpyDeviceToDevice)); CK(cudaEventRecord(e1));
      CK(cudaEventSynchronize(e1)); float ms; CK(cudaEventElapsedTime(&ms, e0, e1)); if (ms < best) best = ms;
    }
    printf("cudaMemcpy D2D 1 GiB: %.3f ms -> %.1f GB/s (read+write)\n", best, 2.0 * n * 4 / best / 1e6);
  }

  // ---------------- NCCL single-rank self send/recv
  int ver; NK(ncclGetVersion(&ver)); printf("NCCL runtime version %d\n", ver);
  ncclComm_t comm; int dev = 0; NK(ncclCommInitAll(&comm, 1, &dev));
  float *s, *r; CK(cudaMalloc(&s, 1 << 20)); CK(cudaMalloc(&r, 1 << 20));
  CK(cudaMemset(s, 0x3f, 1 << 20)); CK(cudaMemset(r, 0, 1 << 20));
  cudaStream_t stream; CK(cudaStreamCreate(&stream));
  NK(ncclGroupStart());
  NK(ncclSend(s, 1 << 18, ncclFloat, 0, comm, stream));
  NK(ncclRecv(r, 1 << 18, ncclFloat, 0, comm, stream));
  NK(ncclGroupEnd());
  CK(cudaStreamSynchronize(stream));
  float hv; CK(cudaMemcpy(&hv, r + 1000, 4, cudaMemcpyDeviceToHost));
  printf("NCCL self send/recv value check: %s\n", hv == *(float*)"\x3f\x3f\x3f\x3f" ? "OK" : "BAD");
  // graph capture of NCCL self send/recv
  cudaGraph_t g; cudaGraphExec_t ge2;
  CK(cudaStreamBeginCapture(stream, cudaStreamCaptureModeThreadLocal));
  NK(ncclGroupStart());
  NK(ncclSend(s, 1 << 18, ncclFloat, 0, comm, stream));
  NK(ncclRecv(r, 1 << 18, ncclFloat, 0, comm, stream));
  NK(ncclGroupEnd());
  CK(cudaStreamEndCapture(stream, &g));
  CK(cudaGraphInstantiate(&ge2, g, 0));
  CK(cudaGraphLaunch(ge2, stream)); CK(cudaStreamSynchronize(stream));
  printf("NCCL graph capture: OK\n");
  ncclCommDestroy(comm);
  return 0;
}
