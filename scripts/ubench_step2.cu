// ubench_step2.cu — the compute warp's step of nw_wave.cuh (K=8) in isolation: ring LDS.128 /
// STS.128, SHFL.UP chain, SHFL.IDX border value, DPX cells, publish STS.64; one warp per SM.
// Variants of the cell arithmetic are timed in cycles per step.
//   nvcc -std=c++20 -gencode arch=compute_100a,code=sm_100a -O3 -o scripts/ubench_step2 scripts/ubench_step2.cu
#include <cstdio>
#include <cuda_runtime.h>

constexpr int NSTEP = 8192;
constexpr int K = 8, R = 64, RS = 32 * K + 4;

__device__ __forceinline__ int4 lds128(unsigned a) {
  int4 v;
  asm volatile("ld.shared.v4.b32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a));
  return v;
}
__device__ __forceinline__ void sts128(unsigned a, int x, int y, int z, int w) {
  asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(x), "r"(y), "r"(z), "r"(w));
}
__device__ __forceinline__ unsigned opaque(unsigned x) {
  asm volatile("mov.b32 %0, %0;" : "+r"(x));
  return x;
}

// V: 0 = as in the kernel (sequential Y chain, Pv = max(L + negp, Y)), 1 = positive pk with the
// negation modifier, 2 = 1 + Y chain split in two halves, 3 = 2 + Pv[K-1] first
template <int V>
__global__ void k_step(int* out, long long* cyc, int p, int seed) {
  extern __shared__ __align__(16) int sm[];
  const int t = threadIdx.x & 31;
  const unsigned base = static_cast<unsigned>(__cvta_generic_to_shared(sm));
  const unsigned refR = base, scR = base + 4u * R * RS, bring = scR + 4u * R * RS;
  for (int i = t; i < R * RS; i += 32) sm[i] = (i * 7 + seed) % 13 - 4;
  __syncwarp();
  int Pv[K], rvn[K], negp[K], pk[K];
#pragma unroll
  for (int m = 0; m < K; ++m) {
    Pv[m] = -t * 10 - m;
    rvn[m] = 0;
    negp[m] = static_cast<int>(opaque(static_cast<unsigned>(-(m + 1) * p)));
    pk[m] = static_cast<int>(opaque(static_cast<unsigned>((m + 1) * p)));
  }
  int Lprev = 0, vlast = Pv[K - 1];
  const unsigned long long cur = static_cast<unsigned long long>(seed + t);
  const unsigned laneR = refR + 32u * t, laneS = scR + 32u * t;
  long long t0 = clock64();
#pragma unroll 8
  for (int s = 0; s < NSTEP; ++s) {
    const int r = s + 1 - t;
    int rv[K];
#pragma unroll
    for (int m = 0; m < K; ++m) rv[m] = rvn[m];
    const unsigned an = laneR + static_cast<unsigned>(r & (R - 1)) * (4u * RS);
    const int4 u = lds128(an), w4 = lds128(an + 16);
    rvn[0] = u.x, rvn[1] = u.y, rvn[2] = u.z, rvn[3] = u.w, rvn[4] = w4.x, rvn[5] = w4.y, rvn[6] = w4.z, rvn[7] = w4.w;
    const int bval = __shfl_sync(0xffffffffu, static_cast<int>(cur), s & 7);
    const int from_left = __shfl_up_sync(0xffffffffu, vlast, 1);
    const int L = (t == 0) ? bval : from_left;
    int Y[K];
    if (V >= 2) {
      int x[K];
      int d = Lprev;
#pragma unroll
      for (int m = 0; m < K; ++m) {
        x[m] = __viaddmax_s32(Pv[m], -p, d + rv[m]);
        d = Pv[m];
      }
      Y[0] = x[0];
      Y[4] = x[4];
#pragma unroll
      for (int m = 1; m < 4; ++m) {
        Y[m] = __viaddmax_s32(Y[m - 1], -p, x[m]);
        Y[4 + m] = __viaddmax_s32(Y[3 + m], -p, x[4 + m]);
      }
#pragma unroll
      for (int m = 4; m < 8; ++m) Y[m] = __viaddmax_s32(Y[3], -pk[m - 4], Y[m]);
    } else {
      int d = Lprev;
#pragma unroll
      for (int m = 0; m < K; ++m) {
        const int x = __viaddmax_s32(Pv[m], -p, d + rv[m]);
        Y[m] = m == 0 ? x : __viaddmax_s32(Y[m - 1], -p, x);
        d = Pv[m];
      }
    }
    if (V == 0) {
#pragma unroll
      for (int m = 0; m < K; ++m) Pv[m] = __viaddmax_s32(L, negp[m], Y[m]);
    } else if (V == 3) {
      Pv[K - 1] = __viaddmax_s32(L, -pk[K - 1], Y[K - 1]);
      vlast = Pv[K - 1];
#pragma unroll
      for (int m = 0; m < K - 1; ++m) Pv[m] = __viaddmax_s32(L, -pk[m], Y[m]);
    } else {
#pragma unroll
      for (int m = 0; m < K; ++m) Pv[m] = __viaddmax_s32(L, -pk[m], Y[m]);
    }
    Lprev = L;
    const unsigned aS = laneS + static_cast<unsigned>((r - 1) & (R - 1)) * (4u * RS);
    sts128(aS, Pv[0], Pv[1], Pv[2], Pv[3]);
    sts128(aS + 16, Pv[4], Pv[5], Pv[6], Pv[7]);
    if (t == 31) {
      asm volatile("{ .reg .b64 e; mov.b64 e, {%1, %2}; st.volatile.shared.b64 [%0], e; }" ::"r"(bring + 8u * (r & 255)), "r"(Pv[K - 1]), "r"(r) : "memory");
    }
    vlast = Pv[K - 1];
  }
  long long t1 = clock64();
  int acc = 0;
#pragma unroll
  for (int m = 0; m < K; ++m) acc += Pv[m];
  out[blockIdx.x * 32 + t] = acc;
  if (t == 0 && blockIdx.x == 0) cyc[0] = t1 - t0;
}

template <int V>
void run(int* out, long long* cyc) {
  const size_t smem = 2ull * R * RS * 4 + 256 * 8;
  cudaFuncSetAttribute(k_step<V>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  long long h = 0;
  for (int rep = 0; rep < 2; ++rep) {
    k_step<V><<<148, 32, smem>>>(out, cyc, 10, rep);
    cudaDeviceSynchronize();
  }
  cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
  printf("variant %d: %7.1f cycles/step\n", V, double(h) / NSTEP);
}

int main() {
  int* out;
  long long* cyc;
  cudaMalloc(&out, 148 * 32 * 4);
  cudaMalloc(&cyc, 64);
  run<0>(out, cyc);
  run<1>(out, cyc);
  run<2>(out, cyc);
  run<3>(out, cyc);
  printf("%s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
