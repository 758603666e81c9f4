// ubench_ops.cu — issue interval (8 independent chains) and dependent latency (1 chain) of the
// integer ops the wavefront step can be built from, one warp per SM sub-partition.
//   nvcc -std=c++17 -O3 -gencode arch=compute_100a,code=sm_100a -o scripts/ubench_ops scripts/ubench_ops.cu
#include <cstdio>
#include <cuda_runtime.h>

constexpr int ITER = 4096;

template <int OP>
__device__ __forceinline__ int op(int a, int b, int c) {
  int d;
  if constexpr (OP == 0) asm volatile("max.s32 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(b));                     // IMNMX
  if constexpr (OP == 1) d = __vimax3_s32(a, b, c);                                                           // VIMNMX3
  if constexpr (OP == 2) d = __viaddmax_s32(a, b, c);                                                         // VIADDMNMX
  if constexpr (OP == 3) asm volatile("add.s32 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(b));                     // IADD
  if constexpr (OP == 4) asm volatile("{ .reg .s32 t; add.s32 t, %1, %2; add.s32 %0, t, %3; }" : "=r"(d) : "r"(a), "r"(b), "r"(c));  // IADD3
  if constexpr (OP == 5) asm volatile("mad.lo.s32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));      // IMAD
  if constexpr (OP == 6) asm volatile("max.f32 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(b));                     // FMNMX
  if constexpr (OP == 7) asm volatile("add.f32 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(b));                     // FADD
  if constexpr (OP == 8) asm volatile("max.s16x2 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(b));                   // VHMNMX / 16x2
  if constexpr (OP == 9) d = __vimax3_s16x2(a, b, c);                                                         // 16x2 3-input
  if constexpr (OP == 10) d = __viaddmax_s16x2(a, b, c);                                                      // 16x2 add-max
  if constexpr (OP == 11) asm volatile("max.f32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));       // FMNMX3 (if any)
  if constexpr (OP == 12) asm volatile("{ .reg .pred q; setp.ne.s32 q, %3, 0; selp.b32 %0, %1, %2, q; }" : "=r"(d) : "r"(a), "r"(b), "r"(c));  // SEL
  return d;
}

template <int OP, int CH>
__global__ void k(int* out, long long* cyc, int s) {
  int v[CH];
#pragma unroll
  for (int i = 0; i < CH; ++i) v[i] = threadIdx.x * 7 + i * s;
  const int b = s + 1, c = s - 3;
  __syncwarp();
  long long t0 = clock64();
#pragma unroll 4
  for (int it = 0; it < ITER; ++it) {
#pragma unroll
    for (int i = 0; i < CH; ++i) v[i] = op<OP>(v[i], b ^ it, c + i);
  }
  long long t1 = clock64();
  int acc = 0;
#pragma unroll
  for (int i = 0; i < CH; ++i) acc += v[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  if ((threadIdx.x & 31) == 0) cyc[blockIdx.x * 4 + threadIdx.x / 32] = t1 - t0;
}

template <int OP>
void run(const char* name, int* out, long long* cyc) {
  long long h[4];
  k<OP, 8><<<148, 128>>>(out, cyc, 3);
  k<OP, 8><<<148, 128>>>(out, cyc, 3);
  cudaDeviceSynchronize();
  cudaMemcpy(h, cyc, 32, cudaMemcpyDeviceToHost);
  const double thr = static_cast<double>(h[0]) / (ITER * 8.0);
  k<OP, 1><<<148, 128>>>(out, cyc, 3);
  cudaError_t e = cudaDeviceSynchronize();
  cudaMemcpy(h, cyc, 32, cudaMemcpyDeviceToHost);
  const double lat = static_cast<double>(h[0]) / ITER;
  printf("%-34s issue interval %5.2f cyc/warp-instr   dependent latency %5.2f cyc  %s\n", name, thr, lat,
         e == cudaSuccess ? "" : cudaGetErrorString(e));
}

int main() {
  int* out;
  long long* cyc;
  cudaMalloc(&out, 148 * 128 * 4);
  cudaMalloc(&cyc, 148 * 4 * 8);
  run<0>("IMNMX (max.s32)", out, cyc);
  run<1>("VIMNMX3 (__vimax3_s32)", out, cyc);
  run<2>("VIADDMNMX (__viaddmax_s32)", out, cyc);
  run<3>("IADD (add.s32)", out, cyc);
  run<4>("IADD3 (add+add)", out, cyc);
  run<5>("IMAD (mad.lo.s32)", out, cyc);
  run<6>("FMNMX (max.f32)", out, cyc);
  run<7>("FADD (add.f32)", out, cyc);
  run<8>("max.s16x2", out, cyc);
  run<9>("__vimax3_s16x2", out, cyc);
  run<10>("__viaddmax_s16x2", out, cyc);
  run<11>("max.f32 3-input", out, cyc);
  run<12>("selp", out, cyc);
  return 0;
}
