// Pipe-rate probe (A/B measurement, not product code): issue cost per warp instruction of the
// FP32 forms the T-level march uses (FADD, FADD2, FMUL2, FMUL-imm, SHFL) alone and mixed, with
// 8 independent chains per thread and W warps per SM.  Prints SMSP-cycles per warp instruction.
#include <cstdio>
#include <cuda_runtime.h>

#define ITERS 4096
template <int OP>
__global__ void __launch_bounds__(1024, 1) k(float* out, float seed, long long* cyc) {
  float a[8], b[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) { a[i] = seed * (threadIdx.x + i); b[i] = seed + i; }
  long long t0 = clock64();
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int i = 0; i < 8; i += 2) {
      if (OP == 0) {  // 2 x FADD r,r
        asm volatile("add.rn.f32 %0, %0, %1;" : "+f"(a[i]) : "f"(b[i]));
        asm volatile("add.rn.f32 %0, %0, %1;" : "+f"(a[i + 1]) : "f"(b[i + 1]));
      } else if (OP == 1) {  // 1 x FADD2
        asm volatile("{.reg .b64 x, y; mov.b64 x, {%0, %1}; mov.b64 y, {%2, %3}; add.rn.f32x2 x, x, y; mov.b64 {%0, %1}, x;}"
                     : "+f"(a[i]), "+f"(a[i + 1]) : "f"(b[i]), "f"(b[i + 1]));
      } else if (OP == 2) {  // 1 x FMUL2 by a pair
        asm volatile("{.reg .b64 x, y; mov.b64 x, {%0, %1}; mov.b64 y, {%2, %2}; mul.rn.f32x2 x, x, y; mov.b64 {%0, %1}, x;}"
                     : "+f"(a[i]), "+f"(a[i + 1]) : "f"(0.999f));
      } else if (OP == 3) {  // 2 x FMUL imm
        asm volatile("mul.rn.f32 %0, %0, 0f3F7FBE77;" : "+f"(a[i]));
        asm volatile("mul.rn.f32 %0, %0, 0f3F7FBE77;" : "+f"(a[i + 1]));
      } else if (OP == 4) {  // 2 x SHFL
        asm volatile("shfl.sync.up.b32 %0, %0, 1, 0, -1;" : "+f"(a[i]));
        asm volatile("shfl.sync.down.b32 %0, %0, 1, 31, -1;" : "+f"(a[i + 1]));
      } else if (OP == 5) {  // FADD2 + 2 FADD (per pair of chains: 1 packed + 2 scalar)
        asm volatile("{.reg .b64 x, y; mov.b64 x, {%0, %1}; mov.b64 y, {%2, %3}; add.rn.f32x2 x, x, y; mov.b64 {%0, %1}, x;}"
                     : "+f"(a[i]), "+f"(a[i + 1]) : "f"(b[i]), "f"(b[i + 1]));
        asm volatile("add.rn.f32 %0, %0, %1;" : "+f"(b[i]) : "f"(a[i + 1]));
        asm volatile("add.rn.f32 %0, %0, %1;" : "+f"(b[i + 1]) : "f"(a[i]));
      } else if (OP == 6) {  // FADD2 + FMUL2
        asm volatile("{.reg .b64 x, y; mov.b64 x, {%0, %1}; mov.b64 y, {%2, %3}; add.rn.f32x2 x, x, y; mov.b64 {%0, %1}, x;}"
                     : "+f"(a[i]), "+f"(a[i + 1]) : "f"(b[i]), "f"(b[i + 1]));
        asm volatile("{.reg .b64 x, y; mov.b64 x, {%0, %1}; mov.b64 y, {%2, %2}; mul.rn.f32x2 x, x, y; mov.b64 {%0, %1}, x;}"
                     : "+f"(b[i]), "+f"(b[i + 1]) : "f"(0.999f));
      } else if (OP == 7) {  // FADD2 + 2 SHFL
        asm volatile("{.reg .b64 x, y; mov.b64 x, {%0, %1}; mov.b64 y, {%2, %3}; add.rn.f32x2 x, x, y; mov.b64 {%0, %1}, x;}"
                     : "+f"(a[i]), "+f"(a[i + 1]) : "f"(b[i]), "f"(b[i + 1]));
        asm volatile("shfl.sync.up.b32 %0, %0, 1, 0, -1;" : "+f"(b[i]));
        asm volatile("shfl.sync.down.b32 %0, %0, 1, 31, -1;" : "+f"(b[i + 1]));
      } else if (OP == 8) {  // 2 FADD + 2 FMUL imm
        asm volatile("add.rn.f32 %0, %0, %1;" : "+f"(a[i]) : "f"(b[i]));
        asm volatile("add.rn.f32 %0, %0, %1;" : "+f"(a[i + 1]) : "f"(b[i + 1]));
        asm volatile("mul.rn.f32 %0, %0, 0f3F7FBE77;" : "+f"(b[i]));
        asm volatile("mul.rn.f32 %0, %0, 0f3F7FBE77;" : "+f"(b[i + 1]));
      } else if (OP == 9) {  // 2 FADD + 2 MOV-like (integer add on ALU pipe)
        asm volatile("add.rn.f32 %0, %0, %1;" : "+f"(a[i]) : "f"(b[i]));
        asm volatile("add.rn.f32 %0, %0, %1;" : "+f"(a[i + 1]) : "f"(b[i + 1]));
        asm volatile("{.reg .b32 t; mov.b32 t, %0; xor.b32 t, t, 1; mov.b32 %0, t;}" : "+f"(b[i]));
        asm volatile("{.reg .b32 t; mov.b32 t, %0; xor.b32 t, t, 1; mov.b32 %0, t;}" : "+f"(b[i + 1]));
      }
    }
  }
  long long t1 = clock64();
  float s = 0;
#pragma unroll
  for (int i = 0; i < 8; ++i) s += a[i] + b[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

template <int OP>
void run(const char* name, int ipp, int warps, float* out, long long* cyc) {
  // ipp: warp instructions per pair-iteration (per i step)
  k<OP><<<148, warps * 32>>>(out, 1.0001f, cyc);
  cudaDeviceSynchronize();
  long long h[148];
  cudaMemcpy(h, cyc, sizeof(h), cudaMemcpyDeviceToHost);
  double c = 0;
  for (int i = 0; i < 148; ++i) c += h[i];
  c /= 148;
  const double instr_per_smsp = (double)ITERS * 4 * ipp * warps / 4.0;
  printf("%-28s warps/SM %2d: %.3f SMSP-cycles per warp instruction\n", name, warps, c / instr_per_smsp);
}

int main() {
  float* out;
  long long* cyc;
  cudaMalloc(&out, 148 * 1024 * 4);
  cudaMalloc(&cyc, 148 * 8);
  for (int w : {8, 16, 32}) {
    run<0>("FADD r,r", 2, w, out, cyc);
    run<1>("FADD2", 1, w, out, cyc);
    run<2>("FMUL2 (pair reg)", 1, w, out, cyc);
    run<3>("FMUL imm", 2, w, out, cyc);
    run<4>("SHFL", 2, w, out, cyc);
    run<5>("FADD2 + 2 FADD", 3, w, out, cyc);
    run<6>("FADD2 + FMUL2", 2, w, out, cyc);
    run<7>("FADD2 + 2 SHFL", 3, w, out, cyc);
    run<8>("2 FADD + 2 FMUL imm", 4, w, out, cyc);
    run<9>("2 FADD + 2 LOP3", 4, w, out, cyc);
  }
  printf("%s\n", cudaGetErrorString(cudaGetLastError()));
}
