// ubench.cu — single-warp latency microbenchmarks of the primitives on the strip kernel's
// critical path (SHFL.UP, SEL, VIADDMNMX, LDS) on the target GPU.  Build + run:
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ubench scripts/ubench.cu && /tmp/ubench
#include <cstdio>
#include <cuda_runtime.h>

constexpr int N = 4096;

__global__ void k_shfl(int* out, long long* cyc, int seed) {
  int x = threadIdx.x + seed;
  long long t0 = clock64();
#pragma unroll 16
  for (int i = 0; i < N; ++i) x = __shfl_up_sync(0xffffffffu, x, 1);
  long long t1 = clock64();
  out[threadIdx.x] = x;
  if (threadIdx.x == 0) cyc[0] = t1 - t0;
}
__global__ void k_shfl_add(int* out, long long* cyc, int seed) {
  int x = threadIdx.x + seed;
  long long t0 = clock64();
#pragma unroll 16
  for (int i = 0; i < N; ++i) x = __shfl_up_sync(0xffffffffu, x, 1) + 1;
  long long t1 = clock64();
  out[threadIdx.x] = x;
  if (threadIdx.x == 0) cyc[0] = t1 - t0;
}
__global__ void k_viadd(int* out, long long* cyc, int seed) {
  int x = threadIdx.x + seed, y = seed * 3;
  long long t0 = clock64();
#pragma unroll 16
  for (int i = 0; i < N; ++i) x = __viaddmax_s32(x, -seed, y + i);
  long long t1 = clock64();
  out[threadIdx.x] = x;
  if (threadIdx.x == 0) cyc[0] = t1 - t0;
}
__global__ void k_sel(int* out, long long* cyc, int seed) {
  int x = threadIdx.x + seed, y = seed;
  const bool p = threadIdx.x == 0;
  long long t0 = clock64();
#pragma unroll 16
  for (int i = 0; i < N; ++i) {
    x = p ? y : x;
    asm volatile("" : "+r"(x));
    x = x + 1;
  }
  long long t1 = clock64();
  out[threadIdx.x] = x;
  if (threadIdx.x == 0) cyc[0] = t1 - t0;
}
__global__ void k_lds(int* out, long long* cyc, int seed) {
  __shared__ int sm[1024];
  for (int i = threadIdx.x; i < 1024; i += 32) sm[i] = (i + 1 + seed) & 1023;
  __syncwarp();
  int x = threadIdx.x;
  long long t0 = clock64();
#pragma unroll 16
  for (int i = 0; i < N; ++i) x = sm[x];
  long long t1 = clock64();
  out[threadIdx.x] = x;
  if (threadIdx.x == 0) cyc[0] = t1 - t0;
}
// step-like recurrence: SHFL.UP -> SEL -> VIADDMNMX -> next
__global__ void k_step(int* out, long long* cyc, int seed) {
  int v = threadIdx.x + seed, b = seed;
  const bool l0 = threadIdx.x == 0;
  long long t0 = clock64();
#pragma unroll 16
  for (int i = 0; i < N; ++i) {
    const int f = __shfl_up_sync(0xffffffffu, v, 1);
    const int L = l0 ? b + i : f;
    v = __viaddmax_s32(L, -seed, v);
  }
  long long t1 = clock64();
  out[threadIdx.x] = v;
  if (threadIdx.x == 0) cyc[0] = t1 - t0;
}

int main() {
  int* out;
  long long* cyc;
  cudaMalloc(&out, 4096);
  cudaMalloc(&cyc, 64);
  auto run = [&](const char* name, void (*k)(int*, long long*, int), int per) {
    long long h = 0;
    for (int rep = 0; rep < 3; ++rep) {
      k<<<1, 32>>>(out, cyc, 1);
      cudaDeviceSynchronize();
      cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
    }
    printf("%-28s %8.2f cycles/iter\n", name, double(h) / N / per);
  };
  run("SHFL.UP dependent", k_shfl, 1);
  run("SHFL.UP + IADD dependent", k_shfl_add, 1);
  run("VIADDMNMX dependent", k_viadd, 1);
  run("SEL + IADD dependent", k_sel, 1);
  run("LDS pointer chase", k_lds, 1);
  run("step: SHFL->SEL->VIADDMNMX", k_step, 1);
  printf("%s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
