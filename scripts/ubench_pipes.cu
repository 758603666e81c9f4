// ubench_pipes.cu — which integer / float ops share an issue pipe on sm_100a?  One warp per SM
// sub-partition runs 8 independent chains of op A interleaved with 8 independent chains of op B;
// cycles per (A, B) pair ~ 2 if they use different pipes at 2 cycles each, ~4 if they share one.
//   nvcc -std=c++17 -O3 -gencode arch=compute_100a,code=sm_100a -o scripts/ubench_pipes scripts/ubench_pipes.cu
#include <cstdio>
#include <cuda_runtime.h>

constexpr int ITER = 2048;

template <int OP>
__device__ __forceinline__ void op(int& v, int b, int c) {
  if constexpr (OP == 0) asm volatile("max.s32 %0, %0, %1;" : "+r"(v) : "r"(b));
  if constexpr (OP == 1) asm volatile("mad.lo.s32 %0, %0, %1, %2;" : "+r"(v) : "r"(b), "r"(c));
  if constexpr (OP == 2) { v = __viaddmax_s32(v, b, c); asm volatile("" : "+r"(v)); }
  if constexpr (OP == 3) { v = __vimax3_s32(v, b, c); asm volatile("" : "+r"(v)); }
  if constexpr (OP == 4) asm volatile("add.s32 %0, %0, %1;" : "+r"(v) : "r"(b));
  if constexpr (OP == 5) asm volatile("fma.rn.f32 %0, %0, %1, %2;" : "+r"(v) : "r"(b), "r"(c));
  if constexpr (OP == 6) asm volatile("max.f32 %0, %0, %1;" : "+r"(v) : "r"(b));
  if constexpr (OP == 7) asm volatile("max.f16x2 %0, %0, %1;" : "+r"(v) : "r"(b));
  if constexpr (OP == 8) asm volatile("fma.rn.f16x2 %0, %0, %1, %2;" : "+r"(v) : "r"(b), "r"(c));
  if constexpr (OP == 9) asm volatile("add.f32 %0, %0, %1;" : "+r"(v) : "r"(b));
  if constexpr (OP == 10) asm volatile("max.s16x2 %0, %0, %1;" : "+r"(v) : "r"(b));
  if constexpr (OP == 11) asm volatile("{ .reg .pred q; setp.ne.s32 q, %2, 0; selp.b32 %0, %0, %1, q; }" : "+r"(v) : "r"(b), "r"(c));
  if constexpr (OP == 12) asm volatile("add.s32 %0, %0, 7;" : "+r"(v));
  if constexpr (OP == 13) asm volatile("max.s32 %0, %0, 7;" : "+r"(v));
  if constexpr (OP == 14) asm volatile("mad.lo.s32 %0, %0, 3, %1;" : "+r"(v) : "r"(b));
}

// NA chains of A and NB chains of B, interleaved
template <int A, int B, int NA, int NB>
__global__ void k(int* out, long long* cyc, int s) {
  int va[8], vb[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) va[i] = threadIdx.x + i * s, vb[i] = threadIdx.x * 3 + i;
  int b = s | 1, c = s * 5;
  asm volatile("" : "+r"(b), "+r"(c));
  __syncwarp();
  long long t0 = clock64();
#pragma unroll 2
  for (int it = 0; it < ITER; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      if (i < NA) op<A>(va[i], b, c);
      if (i < NB) op<B>(vb[i], b, c);
    }
  }
  long long t1 = clock64();
  int acc = 0;
#pragma unroll
  for (int i = 0; i < 8; ++i) acc += va[i] + vb[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  if ((threadIdx.x & 31) == 0) cyc[blockIdx.x * 4 + threadIdx.x / 32] = t1 - t0;
}

template <int A, int B, int NA, int NB>
double run1(int* out, long long* cyc) {
  long long h[4];
  k<A, B, NA, NB><<<148, 128>>>(out, cyc, 3);
  k<A, B, NA, NB><<<148, 128>>>(out, cyc, 3);
  cudaDeviceSynchronize();
  cudaMemcpy(h, cyc, 32, cudaMemcpyDeviceToHost);
  return static_cast<double>(h[0]) / (ITER * 8.0);  // cycles per chain-slot (8 slots per iteration)
}

template <int A, int B>
void run(const char* na, const char* nb, int* out, long long* cyc) {
  const double a = run1<A, A, 8, 0>(out, cyc), b = run1<B, B, 8, 0>(out, cyc), ab = run1<A, B, 8, 8>(out, cyc);
  printf("%-10s alone %5.2f | %-10s alone %5.2f | A+B interleaved %5.2f cyc per pair (%s)\n", na, a, nb, b, ab,
         ab < 0.75 * (a + b) ? "separate pipes" : "same pipe / issue bound");
}

int main() {
  int* out;
  long long* cyc;
  cudaMalloc(&out, 148 * 128 * 4);
  cudaMalloc(&cyc, 148 * 4 * 8);
  run<0, 1>("IMNMX", "IMAD", out, cyc);
  run<2, 1>("VIADDMNMX", "IMAD", out, cyc);
  run<3, 1>("VIMNMX3", "IMAD", out, cyc);
  run<0, 4>("IMNMX", "IADD", out, cyc);
  run<0, 5>("IMNMX", "FFMA", out, cyc);
  run<6, 5>("FMNMX", "FFMA", out, cyc);
  run<0, 7>("IMNMX", "HMNMX2", out, cyc);
  run<7, 8>("HMNMX2", "HFMA2", out, cyc);
  run<0, 9>("IMNMX", "FADD", out, cyc);
  run<0, 10>("IMNMX", "VIMNMX16x2", out, cyc);
  run<0, 11>("IMNMX", "SEL", out, cyc);
  run<0, 12>("IMNMX", "IADD imm", out, cyc);
  run<13, 14>("IMNMX imm", "IMAD imm", out, cyc);
  run<0, 6>("IMNMX", "FMNMX", out, cyc);
  return 0;
}
