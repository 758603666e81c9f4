// ubench_mw.cu — cycles per wavefront step with NC compute warps per SM (one per sub-partition),
// each sweeping its own band (no cross-warp dependency), with or without staging warps moving
// representative traffic (ref rows in by 4-byte cp.async, score rows out by LDS + STG).
// Decides the round-2 kernel geometry (K columns per lane, compute warps per SM, cell form).
//   nvcc -std=c++20 -O3 -gencode arch=compute_100a,code=sm_100a -o scripts/ubench_mw scripts/ubench_mw.cu
//
// Forms: F=0 gap-normalised (round-1 kernel: ref+2p, VIADDMNMX, prefix IMNMX, IMNMX with L);
//        F=1 plain S form: d = diag + ref on the FMA pipe (IMAD), x = max(up - p, d),
//            Y = max(Y - p, x), S = max(L - (m+1)p, Y) -- three VIADDMNMX per cell, no conversion.
// Border: B=0 lane 0 takes the border from a 16-row block held in lanes 0..15 (SHFL.IDX + SEL);
//         B=1 rotate: lane 31 sends the border of lane 0's next row through the same SHFL
//             (one shuffle per step; lane 31 reads the value by a broadcast LDS).
#include <cstdio>
#include <cuda_runtime.h>

constexpr int NSTEP = 8192, RR = 64;

__device__ __forceinline__ int imad1(int a, int one, int b) {
  int d;
  asm("mad.lo.s32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(one), "r"(b));
  return d;
}
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
__device__ __forceinline__ int lds32(unsigned a) {
  int v;
  asm volatile("ld.shared.b32 %0, [%1];" : "=r"(v) : "r"(a));
  return v;
}

// smem per compute warp: ref ring RR rows x W, score ring RR rows x W (row stride W + pad)
template <int K>
struct G {
  static constexpr int W = 32 * K;
  static constexpr int RS = K == 8 ? W + 4 : W;  // K = 8 needs the bank-group shift
  static constexpr int WARP_WORDS = 2 * RR * RS + 64;
};

template <int K, int NC, int F, int B, int NS>
__global__ void __launch_bounds__(32 * (NC + NS), 1) k_mw(int* out, long long* cyc, const int* gref, int* gsc, int p) {
  extern __shared__ __align__(16) int sm[];
  constexpr int W = G<K>::W, RS = G<K>::RS;
  const int t = threadIdx.x & 31, w = threadIdx.x >> 5;
  volatile int* prog = sm;  // [0]: compute warp 0's step
  if (threadIdx.x == 0) prog[0] = 0;
  for (int i = threadIdx.x; i < NC * G<K>::WARP_WORDS; i += blockDim.x) sm[64 + i] = (i * 7) % 13 - 4;
  __syncthreads();
  if (w >= NC) {
    // staging warp: NS = 2 -> warp NC: ref rows in (cp.async 4 B), warp NC+1: score rows out
    const bool is_ref = w == NC;
    const int* src = gref + blockIdx.x * 4096;
    int* dst = gsc + blockIdx.x * 4096;
    unsigned ring = static_cast<unsigned>(__cvta_generic_to_shared(sm + 64));
    int done = 0;
    while (done < NSTEP) {
      const int cur = prog[0];
      if (cur >= NSTEP - 8) break;
      if (done + 8 > cur + 32) continue;  // pace: about the compute warps' rate
      for (int c = 0; c < NC; ++c) {
        const unsigned wr = ring + 4u * (c * G<K>::WARP_WORDS);
        for (int r = 0; r < 8; ++r) {
          const int row = (done + r) & (RR - 1);
          if (is_ref) {
#pragma unroll
            for (int i = 0; i < K; ++i)
              asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(wr + 4u * (row * RS + 32 * i + t)), "l"(src + ((r * W + 32 * i + t) & 4095)) : "memory");
          } else {
#pragma unroll
            for (int i = 0; i < K; ++i) dst[(r * W + 32 * i + t) & 4095] = lds32(wr + 4u * (RR * RS + row * RS + 32 * i + t)) + r;
          }
        }
      }
      if (is_ref) asm volatile("cp.async.commit_group; cp.async.wait_group 2;" ::: "memory");
      done += 8;
    }
    asm volatile("cp.async.wait_all;" ::: "memory");
    return;
  }
  const unsigned base = static_cast<unsigned>(__cvta_generic_to_shared(sm + 64 + w * G<K>::WARP_WORDS));
  const unsigned laneR = base + 4u * K * t, laneS = base + 4u * (RR * RS) + 4u * K * t;
  const unsigned bring = base;  // border values (stand-in)
  int up[K], rvn[K], cm[K];
#pragma unroll
  for (int m = 0; m < K; ++m) up[m] = t * K + m, rvn[m] = 0, cm[m] = -(m + 1) * p;
  const int negp = -p, p2 = 2 * p, one = 1;
  int Lprev = 0, vlast = up[K - 1], curv = t * 3, bnext = 0;
  long long t0 = clock64();
  for (int s0 = 0; s0 < NSTEP; s0 += 16) {
    // event: publish, read a progress word, new border block
    __syncwarp();
    if (w == 0 && t == 0) prog[0] = s0;
    curv = lds32(bring + 4u * ((s0 + t) & 63)) + s0;
    int chk = prog[0];
    if (chk < 0) out[0] = chk;
#pragma unroll
    for (int jj = 0; jj < 16; ++jj) {
      const int s = s0 + jj;
      int rv[K];
#pragma unroll
      for (int m = 0; m < K; ++m) rv[m] = F == 0 ? rvn[m] + p2 : rvn[m];
      ldsK<K>(laneR + ((s + 1) & (RR - 1)) * 4u * RS, rvn);
      int L;
      if constexpr (B == 0) {
        const int bval = __shfl_sync(0xffffffffu, curv, jj);
        const int fl = __shfl_up_sync(0xffffffffu, vlast, 1);
        L = t == 0 ? bval : fl;
      } else {
        L = __shfl_sync(0xffffffffu, vlast, (t + 31) & 31);
      }
      int S[K];
      if constexpr (F == 0) {
        int x[K], Y[K];
        x[0] = __viaddmax_s32(Lprev, rv[0], up[0]);
#pragma unroll
        for (int m = 1; m < K; ++m) x[m] = __viaddmax_s32(up[m - 1], rv[m], up[m]);
        Y[0] = x[0];
#pragma unroll
        for (int m = 1; m < K; ++m) Y[m] = max(Y[m - 1], x[m]);
#pragma unroll
        for (int m = 0; m < K; ++m) S[m] = max(L, Y[m]);
      } else {
        int Y[K];
#pragma unroll
        for (int m = 0; m < K; ++m) {
          const int d = imad1(m == 0 ? Lprev : up[m - 1], one, rv[m]);
          const int x = __viaddmax_s32(up[m], negp, d);
          Y[m] = m == 0 ? x : __viaddmax_s32(Y[m - 1], negp, x);
        }
#pragma unroll
        for (int m = 0; m < K; ++m) S[m] = __viaddmax_s32(L, cm[m], Y[m]);
      }
#pragma unroll
      for (int m = 0; m < K; ++m) up[m] = S[m];
      Lprev = L;
      stsK<K>(laneS + (s & (RR - 1)) * 4u * RS, S);
      vlast = S[K - 1];
      if constexpr (B == 1) {
        vlast = t == 31 ? bnext : vlast;
        bnext = lds32(bring + 4u * ((s + 2) & 63));
      }
    }
  }
  long long t1 = clock64();
  if (w == 0 && t == 0) prog[0] = NSTEP;
  int acc = 0;
#pragma unroll
  for (int m = 0; m < K; ++m) acc ^= up[m];
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  if (t == 0) cyc[blockIdx.x * 8 + w] = t1 - t0;
}

template <int K, int NC, int F, int B, int NS>
void run(int sms, const int* gref, int* gsc) {
  int* out;
  long long* cyc;
  cudaMalloc(&out, sms * 32 * 8 * 4);
  cudaMalloc(&cyc, sms * 8 * 8);
  const int smem = 4 * (64 + NC * G<K>::WARP_WORDS);
  auto k = k_mw<K, NC, F, B, NS>;
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  k<<<sms, 32 * (NC + NS), smem>>>(out, cyc, gref, gsc, 10);
  k<<<sms, 32 * (NC + NS), smem>>>(out, cyc, gref, gsc, 10);
  cudaError_t e = cudaDeviceSynchronize();
  long long h[8];
  cudaMemcpy(h, cyc, 8 * 8, cudaMemcpyDeviceToHost);
  double mx = 0;
  for (int i = 0; i < NC; ++i) mx = h[i] > mx ? h[i] : mx;
  const double cps = mx / NSTEP;
  printf("K=%d NC=%d F=%d B=%d NS=%d: %6.1f cyc/step  %6.2f cells/cyc/SM  (smem %d B) %s\n", K, NC, F, B, NS, cps, 32.0 * K * NC / cps, smem,
         e == cudaSuccess ? "" : cudaGetErrorString(e));
  cudaFree(out);
  cudaFree(cyc);
}

int main() {
  const int sms = 148;
  int *gref, *gsc;
  cudaMalloc(&gref, sms * 4096 * 4);
  cudaMalloc(&gsc, sms * 4096 * 4);
  cudaMemset(gref, 0, sms * 4096 * 4);
#define R5(K, NC, F, B, NS) run<K, NC, F, B, NS>(sms, gref, gsc)
  R5(8, 1, 0, 0, 0); R5(8, 1, 1, 0, 0); R5(8, 1, 0, 1, 0); R5(8, 1, 1, 1, 0);
  R5(8, 1, 0, 0, 2); R5(8, 1, 1, 1, 2);
  R5(8, 2, 0, 0, 0); R5(8, 2, 1, 1, 0); R5(8, 2, 1, 1, 2);
  R5(4, 1, 0, 0, 0); R5(4, 1, 1, 0, 0); R5(4, 1, 1, 1, 0);
  R5(4, 2, 0, 0, 0); R5(4, 2, 1, 0, 0); R5(4, 2, 1, 1, 0); R5(4, 2, 0, 0, 2); R5(4, 2, 1, 1, 2);
  R5(4, 4, 0, 0, 0); R5(4, 4, 1, 1, 0); R5(4, 4, 1, 1, 2);
  R5(2, 1, 0, 0, 0); R5(2, 1, 1, 0, 0); R5(2, 1, 1, 1, 0);
  R5(2, 4, 0, 0, 0); R5(2, 4, 1, 0, 0); R5(2, 4, 1, 1, 0); R5(2, 4, 0, 0, 2); R5(2, 4, 1, 1, 2);
  R5(2, 8, 1, 1, 0);
  R5(4, 8, 1, 1, 0);
  return 0;
}
