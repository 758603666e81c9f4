// ubench_sp.cu — cycles per wavefront step of the gap-normalised NW cell (nw_wave.cuh) in
// isolation: K cells per lane, ref row from a shared ring (LDS.128), score row to a shared ring
// (STS.128), SHFL.UP left chain; NWARP independent warps per CTA (one CTA per SM).
//   nvcc -std=c++20 -O3 -gencode arch=compute_100a,code=sm_100a -o scripts/ubench_sp scripts/ubench_sp.cu
#include <cstdio>
#include <cuda_runtime.h>

constexpr int NSTEP = 16384, R = 32;

template <int K>
__device__ __forceinline__ void ldsK(unsigned a, int* v) {
  if constexpr (K == 2) {
    asm volatile("ld.shared.v2.b32 {%0, %1}, [%2];" : "=r"(v[0]), "=r"(v[1]) : "r"(a));
  } else {
#pragma unroll
    for (int q = 0; q < K / 4; ++q)
      asm volatile("ld.shared.v4.b32 {%0, %1, %2, %3}, [%4];" : "=r"(v[4 * q]), "=r"(v[4 * q + 1]), "=r"(v[4 * q + 2]), "=r"(v[4 * q + 3]) : "r"(a + 16 * q));
  }
}
template <int K>
__device__ __forceinline__ void stsK(unsigned a, const int* v) {
  if constexpr (K == 2) {
    asm volatile("st.shared.v2.b32 [%0], {%1, %2};" ::"r"(a), "r"(v[0]), "r"(v[1]));
  } else {
#pragma unroll
    for (int q = 0; q < K / 4; ++q)
      asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(a + 16 * q), "r"(v[4 * q]), "r"(v[4 * q + 1]), "r"(v[4 * q + 2]), "r"(v[4 * q + 3]));
  }
}
__device__ __forceinline__ int iaddfma(int a, int one, int b) {  // a * one + b: IMAD (FMA pipe)
  int d;
  asm("mad.lo.s32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(one), "r"(b));
  return d;
}

// V=0: x = max(d + (r + 2p), up) as the kernel writes it; V=1: r + 2p forced onto the FMA pipe
// (IMAD) so x is one VIADDMNMX; V=2: like 1 with a sequential prefix (no 3-input max)
template <int K, int V>
__global__ void k_sp(int* out, long long* cyc, int p2, int one, unsigned long long* gbuf) {
  unsigned long long* gout = gbuf + static_cast<size_t>(blockIdx.x * 8 + (threadIdx.x >> 5)) * NSTEP;
  const int tag = blockIdx.x + 1;
  const int curv = threadIdx.x * 3 + p2;
  extern __shared__ __align__(16) int sm[];
  const int t = threadIdx.x & 31, w = threadIdx.x >> 5;
  constexpr int RS = 32 * K + 4;
  int* ring = sm + w * 2 * R * RS;
  const unsigned base = static_cast<unsigned>(__cvta_generic_to_shared(ring));
  for (int i = t; i < 2 * R * RS; i += 32) ring[i] = (i * 7) % 13 - 4;
  __syncwarp();
  int Pv[K], rvn[K];
#pragma unroll
  for (int m = 0; m < K; ++m) Pv[m] = t * K + m, rvn[m] = 0;
  int Lprev = 0, vlast = Pv[K - 1];
  const unsigned laneR = base + 4u * K * t, laneS = base + 4u * R * RS + 4u * K * t;
  long long t0 = clock64();
#pragma unroll 8
  for (int s = 0; s < NSTEP; ++s) {
    int rv[K];
#pragma unroll
    for (int m = 0; m < K; ++m) rv[m] = (V == 1 || V == 3) ? iaddfma(rvn[m], one, p2) : rvn[m] + p2;
    ldsK<K>(laneR + ((s + 1) & (R - 1)) * 4u * RS, rvn);
    int L;
    if constexpr (V == 6 || V == 8) {
      const int bval = __shfl_sync(0xffffffffu, curv, s & 15);
      const int from_left = __shfl_up_sync(0xffffffffu, vlast, 1);
      L = t == 0 ? bval : from_left;
    } else if constexpr (V == 5) {
      L = __shfl_sync(0xffffffffu, vlast, (t + 31) & 31);  // lane 31 carries the border value
    } else {
      const int from_left = __shfl_up_sync(0xffffffffu, vlast, 1);
      L = t == 0 ? s : from_left;
    }
    int x[K], Y[K];
    if constexpr (V != 1 && V != 3) {
      x[0] = __viaddmax_s32(Lprev, rv[0], Pv[0]);
#pragma unroll
      for (int m = 1; m < K; ++m) x[m] = __viaddmax_s32(Pv[m - 1], rv[m], Pv[m]);
    } else {  // the diagonal sum on the FMA pipe too
      x[0] = max(iaddfma(Lprev, one, rv[0]), Pv[0]);
#pragma unroll
      for (int m = 1; m < K; ++m) x[m] = max(iaddfma(Pv[m - 1], one, rv[m]), Pv[m]);
    }
    Y[0] = x[0];
    if constexpr (V >= 2) {
#pragma unroll
      for (int m = 1; m < K; ++m) Y[m] = max(Y[m - 1], x[m]);
    } else {
      Y[1] = max(x[0], x[1]);
      if constexpr (K >= 4) {
        Y[2] = __vimax3_s32(x[0], x[1], x[2]);
        Y[3] = __vimax3_s32(Y[1], x[2], x[3]);
      }
      if constexpr (K == 8) {
        Y[4] = __vimax3_s32(Y[2], x[3], x[4]);
        Y[5] = __vimax3_s32(Y[3], x[4], x[5]);
        Y[6] = __vimax3_s32(Y[4], x[5], x[6]);
        Y[7] = __vimax3_s32(Y[5], x[6], x[7]);
      }
    }
#pragma unroll
    for (int m = 0; m < K; ++m) Pv[m] = max(L, Y[m]);
    Lprev = L;
    stsK<K>(laneS + (s & (R - 1)) * 4u * RS, Pv);
    if constexpr (V == 7 || V == 8) {
      asm volatile("{ .reg .pred q; setp.ne.b32 q, %0, 0; @q st.relaxed.gpu.global.v2.b32 [%1], {%2, %3}; }" ::"r"(static_cast<int>(t == 31)),
                   "l"(gout + s), "r"(Pv[K - 1]), "r"(tag)
                   : "memory");
    }
    vlast = Pv[K - 1];
    if constexpr (V == 5) {
      if (t == 31) vlast = s ^ rvn[0];  // (stand-in for the next row's border value)
    }
  }
  long long t1 = clock64();
  int acc = 0;
#pragma unroll
  for (int m = 0; m < K; ++m) acc ^= Pv[m];
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  if (t == 0) cyc[blockIdx.x * 32 + w] = t1 - t0;
}

template <int K, int V>
void run(int nw, int sms) {
  int *out;
  long long* cyc;
  cudaMalloc(&out, sms * 32 * nw * 4);
  cudaMalloc(&cyc, sms * 32 * 8);
  unsigned long long* gbuf;
  cudaMalloc(&gbuf, static_cast<size_t>(sms) * 8 * NSTEP * 8);
  const int smem = nw * 2 * R * (32 * K + 4) * 4;
  cudaFuncSetAttribute(k_sp<K, V>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  k_sp<K, V><<<sms, 32 * nw, smem>>>(out, cyc, 20, 1, gbuf);
  k_sp<K, V><<<sms, 32 * nw, smem>>>(out, cyc, 20, 1, gbuf);
  cudaError_t e = cudaDeviceSynchronize();
  long long h[32];
  cudaMemcpy(h, cyc, 32 * 8, cudaMemcpyDeviceToHost);
  double mx = 0;
  for (int i = 0; i < nw; ++i) mx = h[i] > mx ? h[i] : mx;
  const double cps = mx / NSTEP;
  printf("K=%d V=%d warps/SM=%d: %6.1f cyc/step  %5.2f cells/cyc/warp  %5.2f cells/cyc/SM %s\n", K, V, nw, cps,
         32.0 * K / cps, 32.0 * K * nw / cps, e == cudaSuccess ? "" : cudaGetErrorString(e));
  cudaFree(out);
  cudaFree(cyc);
  cudaFree(gbuf);
}

int main() {
  int sms = 148;
  for (int nw : {1}) {
    run<8, 2>(nw, sms);
    run<8, 6>(nw, sms);
    run<8, 7>(nw, sms);
    run<8, 8>(nw, sms);
    run<4, 0>(nw, sms);
    run<4, 2>(nw, sms);
    run<4, 8>(nw, sms);
  }
  return 0;
}
