// ubench_step3.cu — cycles per wavefront step of ONE compute warp (K = 8: 256 cells), the step
// in isolation (ref ring LDS.128, score ring STS.128, SHFL.UP left value, SHFL.IDX border value),
// for several formulations of the cell arithmetic (round 2: which form does the SM issue fastest?)
//   nvcc -std=c++20 -O3 -gencode arch=compute_100a,code=sm_100a -o scripts/ubench_step3 scripts/ubench_step3.cu
#include <cstdio>
#include <cuda_runtime.h>

constexpr int NSTEP = 8192, RR = 64, K = 8, W = 256, RS = W + 4;

struct Prm {
  int one, p2;
  int z[8];
};

__device__ __forceinline__ int imad(int a, int b, int c) {
  int d;
  asm("mad.lo.s32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
  return d;
}

template <int F, int POLL = 0>
__global__ void __launch_bounds__(128, 1) k(int* out, long long* cyc, const __grid_constant__ Prm P) {
  extern __shared__ __align__(16) int sm[];
  const int t = threadIdx.x & 31;
  if (threadIdx.x >= 32) {  // POLL warps: spin on a shared word until the compute warp is done
    if (threadIdx.x / 32 > POLL) return;
    volatile int* flag = sm + 2 * RR * RS + 64;
    int acc = 0;
    while (flag[0] == 0) acc += flag[1];
    if (acc == 12345) out[0] = acc;
    return;
  }
  if (t == 0) sm[2 * RR * RS + 64] = 0;
  for (int i = t; i < 2 * RR * RS + 64; i += 32) sm[i] = (i * 7) % 13 - 4;
  __syncwarp();
  const unsigned base = static_cast<unsigned>(__cvta_generic_to_shared(sm + 64));
  const unsigned laneR = base + 4u * K * t, laneS = base + 4u * (RR * RS) + 4u * K * t;
  int Pv[K], rvn[K], z[K];
#pragma unroll
  for (int m = 0; m < K; ++m) Pv[m] = t * K + m, rvn[m] = 0, z[m] = P.z[m];
  const int one = P.one, p2 = P.p2;
  int Lprev = 0, vlast = Pv[K - 1], curv = t * 3;
  long long t0 = clock64();
  for (int s0 = 0; s0 < NSTEP; s0 += 16) {
    __syncwarp();
    curv = sm[(s0 + t) & 63] + s0;
#pragma unroll
    for (int jj = 0; jj < 16; ++jj) {
      const int s = s0 + jj, r = s + 1 - t;
      int rv[K];
#pragma unroll
      for (int m = 0; m < K; ++m) rv[m] = rvn[m];
      const unsigned aR = laneR + static_cast<unsigned>(r & (RR - 1)) * 4u * RS;
      {
        int4 u, v;
        asm volatile("ld.shared.v4.b32 {%0,%1,%2,%3}, [%4];" : "=r"(u.x), "=r"(u.y), "=r"(u.z), "=r"(u.w) : "r"(aR));
        asm volatile("ld.shared.v4.b32 {%0,%1,%2,%3}, [%4+16];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(aR));
        rvn[0] = u.x, rvn[1] = u.y, rvn[2] = u.z, rvn[3] = u.w, rvn[4] = v.x, rvn[5] = v.y, rvn[6] = v.z, rvn[7] = v.w;
      }
      int bval, fl;
      if constexpr (F == 7) {  // no SHFL.IDX
        bval = curv + jj;
        fl = __shfl_up_sync(0xffffffffu, vlast, 1);
      } else if constexpr (F == 8 || F == 15 || F == 16) {  // no shuffle at all
        bval = curv + jj;
        fl = vlast + 1;
      } else if constexpr (F == 9) {  // two SHFL.UP, no SHFL.IDX
        bval = __shfl_up_sync(0xffffffffu, curv + jj, 2);
        fl = __shfl_up_sync(0xffffffffu, vlast, 1);
      } else {
        bval = __shfl_sync(0xffffffffu, curv, jj);
        fl = __shfl_up_sync(0xffffffffu, vlast, 1);
      }
      const int L = t == 0 ? bval : fl;
      if constexpr (F == 0) {  // kernel round-2 form: IMAD(one) adds, VIMNMX3 prefix, VIADDMNMX(L + z)
        int Yk[K];
        Yk[0] = max(imad(imad(rv[0], one, p2), one, Lprev), Pv[0]);
#pragma unroll
        for (int m = 1; m < K; ++m) Yk[m] = __vimax3_s32(Yk[m - 1], imad(imad(rv[m], one, p2), one, Pv[m - 1]), Pv[m]);
#pragma unroll
        for (int m = 0; m < K; ++m) Pv[m] = __viaddmax_s32(L, z[m], Yk[m]);
      } else if constexpr (F == 1) {  // round-1 form (ptxas: IADD3 + serial VIMNMX3 chain through L)
        int x[K], Y[K];
        x[0] = __viaddmax_s32(Lprev, rv[0] + p2, Pv[0]);
#pragma unroll
        for (int m = 1; m < K; ++m) x[m] = __viaddmax_s32(Pv[m - 1], rv[m] + p2, Pv[m]);
        Y[0] = x[0];
#pragma unroll
        for (int m = 1; m < K; ++m) Y[m] = max(Y[m - 1], x[m]);
#pragma unroll
        for (int m = 0; m < K; ++m) Pv[m] = max(L, Y[m]);
      } else if constexpr (F == 2) {  // ref' (= ref + 2p) from the ring, x = VIADDMNMX, S chained from L
        int S = L, D = Lprev;
#pragma unroll
        for (int m = 0; m < K; ++m) {
          const int x = __viaddmax_s32(D, rv[m], Pv[m]);
          D = Pv[m];
          S = max(S, x);
          Pv[m] = S;
        }
      } else if constexpr (F == 3 || F >= 7) {  // ref' from the ring, x = VIADDMNMX, Y chain, S = max(L + z, Y)
        int Y = -0x40000000, D = Lprev;
#pragma unroll
        for (int m = 0; m < K; ++m) {
          const int x = __viaddmax_s32(D, rv[m], Pv[m]);
          D = Pv[m];
          Y = max(Y, x);
          Pv[m] = __viaddmax_s32(L, z[m], Y);
        }
      } else if constexpr (F == 10) {  // fp32: d = FADD(diag, ref'), Y = FMNMX3 chain, S = FMNMX(L + z, Y) (FADD z)
        float Y = -1e30f, D = __int_as_float(Lprev);
#pragma unroll
        for (int m = 0; m < K; ++m) {
          const float up = __int_as_float(Pv[m]);
          const float d = D + __int_as_float(rv[m]);
          float y;
          asm("max.f32 %0, %1, %2, %3;" : "=f"(y) : "f"(Y), "f"(d), "f"(up));
          Y = y;
          D = up;
          Pv[m] = __float_as_int(fmaxf(__int_as_float(L) + __int_as_float(z[m]), Y));
        }
      } else if constexpr (F == 11) {  // fp32 chained: S = FMNMX3(S, d, up)
        float S = __int_as_float(L), D = __int_as_float(Lprev);
#pragma unroll
        for (int m = 0; m < K; ++m) {
          const float up = __int_as_float(Pv[m]);
          const float d = D + __int_as_float(rv[m]);
          float y;
          asm("max.f32 %0, %1, %2, %3;" : "=f"(y) : "f"(S), "f"(d), "f"(up));
          S = y;
          D = up;
          Pv[m] = __float_as_int(S);
        }
      } else if constexpr (F == 12) {  // fp32: Y = FMNMX(FMNMX(d, up), Y) 2-input, S = FMNMX(L + z, Y)
        float Y = -1e30f, D = __int_as_float(Lprev);
#pragma unroll
        for (int m = 0; m < K; ++m) {
          const float up = __int_as_float(Pv[m]);
          const float d = D + __int_as_float(rv[m]);
          Y = fmaxf(Y, fmaxf(d, up));
          D = up;
          Pv[m] = __float_as_int(fmaxf(__int_as_float(L) + __int_as_float(z[m]), Y));
        }
      } else if constexpr (F == 13 || F == 15) {  // tree prefix (z on level-2/3 nodes), x = VIADDMNMX(diag, ref+p2, up), S = max(L, Y)
        int x[K], Y[K];
        const int p2 = P.p2;
        x[0] = __viaddmax_s32(Lprev, rv[0] + p2, Pv[0]);
#pragma unroll
        for (int m = 1; m < K; ++m) x[m] = __viaddmax_s32(Pv[m - 1], rv[m] + p2, Pv[m]);
        const int m01 = max(x[0], x[1]), m23 = max(x[2], x[3]), m45 = max(x[4], x[5]), m67 = max(x[6], x[7]);
        Y[0] = x[0];
        Y[1] = m01;
        Y[2] = __viaddmax_s32(m01, z[0], x[2]);
        Y[3] = __viaddmax_s32(m01, z[1], m23);
        const int m46 = __viaddmax_s32(m45, z[2], x[6]), m47 = __viaddmax_s32(m45, z[3], m67);
        Y[4] = __viaddmax_s32(Y[3], z[4], x[4]);
        Y[5] = __viaddmax_s32(Y[3], z[5], m45);
        Y[6] = __viaddmax_s32(Y[3], z[6], m46);
        Y[7] = __viaddmax_s32(Y[3], z[7], m47);
        const int LL = F == 15 ? fl : L;
#pragma unroll
        for (int m = 0; m < K; ++m) Pv[m] = max(LL, Y[m]);
      } else if constexpr (F == 14 || F == 16) {  // two half chains + combine
        int x[K], Y[K];
        const int p2 = P.p2;
        x[0] = __viaddmax_s32(Lprev, rv[0] + p2, Pv[0]);
#pragma unroll
        for (int m = 1; m < K; ++m) x[m] = __viaddmax_s32(Pv[m - 1], rv[m] + p2, Pv[m]);
        Y[0] = x[0];
        for (int m = 1; m < 4; ++m) Y[m] = max(Y[m - 1], x[m]);
        int Z = x[4];
        Y[4] = __viaddmax_s32(Y[3], z[4], Z);
        for (int m = 5; m < 8; ++m) { Z = max(Z, x[m]); Y[m] = __viaddmax_s32(Y[3], z[m], Z); }
        const int LL = F == 16 ? fl : L;
#pragma unroll
        for (int m = 0; m < K; ++m) Pv[m] = max(LL, Y[m]);
      } else if constexpr (F == 4) {  // raw ref: x = max(IADD3(diag, ref, 2p), up), S chained
        int S = L, D = Lprev;
#pragma unroll
        for (int m = 0; m < K; ++m) {
          const int x = max(D + rv[m] + p2, Pv[m]);
          D = Pv[m];
          S = max(S, x);
          Pv[m] = S;
        }
      } else if constexpr (F == 5) {  // F2 without SEL: L straight from SHFL.UP (border ignored)
        int S = fl, D = Lprev;
#pragma unroll
        for (int m = 0; m < K; ++m) {
          const int x = __viaddmax_s32(D, rv[m], Pv[m]);
          D = Pv[m];
          S = max(S, x);
          Pv[m] = S;
        }
      } else if constexpr (F == 6) {  // F2 arithmetic only: no LDS / STS (rv reused)
        int S = L, D = Lprev;
#pragma unroll
        for (int m = 0; m < K; ++m) {
          const int x = __viaddmax_s32(D, rv[m], Pv[m]);
          D = Pv[m];
          S = max(S, x);
          Pv[m] = S;
        }
      }
      Lprev = L;
      if constexpr (F != 6) {
        const unsigned aS = laneS + static_cast<unsigned>((r - 1) & (RR - 1)) * 4u * RS;
        asm volatile("st.shared.v4.b32 [%0], {%1,%2,%3,%4};" ::"r"(aS), "r"(Pv[0]), "r"(Pv[1]), "r"(Pv[2]), "r"(Pv[3]));
        asm volatile("st.shared.v4.b32 [%0+16], {%1,%2,%3,%4};" ::"r"(aS), "r"(Pv[4]), "r"(Pv[5]), "r"(Pv[6]), "r"(Pv[7]));
      } else {
#pragma unroll
        for (int m = 0; m < K; ++m) rvn[m] ^= Pv[m] & 1;
      }
      vlast = Pv[K - 1];
    }
  }
  long long t1 = clock64();
  if (t == 0) sm[2 * RR * RS + 64] = 1;
  int acc = 0;
#pragma unroll
  for (int m = 0; m < K; ++m) acc ^= Pv[m];
  out[blockIdx.x * 32 + t] = acc;
  if (t == 0) cyc[blockIdx.x] = t1 - t0;
}

template <int F, int POLL = 0>
void run(const char* name, int* out, long long* cyc) {
  Prm P{};
  P.one = 1;
  P.p2 = 20;
  for (int i = 0; i < 8; ++i) P.z[i] = 0;
  const int smem = 4 * (2 * RR * RS + 64 + 4);
  cudaFuncSetAttribute(k<F, POLL>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  k<F, POLL><<<148, 32 * (1 + POLL), smem>>>(out, cyc, P);
  k<F, POLL><<<148, 32 * (1 + POLL), smem>>>(out, cyc, P);
  cudaError_t e = cudaDeviceSynchronize();
  long long h = 0;
  cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
  printf("F=%d P=%d %-60s %6.1f cyc/step %s\n", F, POLL, name, static_cast<double>(h) / NSTEP, e == cudaSuccess ? "" : cudaGetErrorString(e));
}

int main() {
  int* out;
  long long* cyc;
  cudaMalloc(&out, 148 * 32 * 4);
  cudaMalloc(&cyc, 148 * 8);
  run<0>("IMAD(one) adds + VIMNMX3 prefix + VIADDMNMX(L+z)", out, cyc);
  run<1>("round-1: ref+2p, VIADDMNMX x, prefix, max(L,Y) (ptxas chain)", out, cyc);
  run<2>("ref' from ring: VIADDMNMX x, S = max(S, x) chained from L", out, cyc);
  run<3>("ref' from ring: VIADDMNMX x, Y chain, S = VIADDMNMX(L,z,Y)", out, cyc);
  run<4>("raw ref: max(IADD3(d, ref, 2p), up), S chained", out, cyc);
  run<5>("F2 without the border SEL", out, cyc);
  run<6>("F2 without LDS / STS", out, cyc);
  run<7>("F3 without the SHFL.IDX", out, cyc);
  run<8>("F3 without any shuffle", out, cyc);
  run<9>("F3 with two SHFL.UP", out, cyc);
  run<10>("fp32: FADD d, FMNMX3 Y chain, FMNMX(L+z, Y)", out, cyc);
  run<11>("fp32 chained: S = FMNMX3(S, d, up)", out, cyc);
  run<12>("fp32: 2-input FMNMX Y, FMNMX(L+z, Y)", out, cyc);
  run<13>("tree prefix (z on L2/L3 nodes), S = max(L, Y)", out, cyc);
  run<14>("two half chains + combine, S = max(L, Y)", out, cyc);
  run<15>("tree prefix, no shuffles", out, cyc);
  run<16>("two half chains, no shuffles", out, cyc);
  run<1, 1>("round-1 form + 1 warp polling a shared word", out, cyc);
  run<1, 3>("round-1 form + 3 warps polling a shared word", out, cyc);
  run<8, 3>("no shuffles + 3 polling warps", out, cyc);
  return 0;
}
