// ubench_step.cu — idealised NW band step (no HBM, no events): the ceiling of the
// one-warp-per-band skewed sweep.  Each warp runs NSTEP steps of a K-column-per-lane band:
// ref from a shared ring (per-lane skewed rows), results to a shared ring, SHFL.UP chain,
// DPX cells.  Reports cycles/step per warp and cells/cycle/SM for 1..16 warps per SM.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o scripts/ubench_step scripts/ubench_step.cu
#include <cstdio>
#include <cuda_runtime.h>

constexpr int NSTEP = 8192;
constexpr int RING = 32;

template <int K, int RPS, int PF>
__global__ void k_band(int* out, long long* cyc, int p) {
  extern __shared__ int sm[];
  const int t = threadIdx.x & 31, w = threadIdx.x >> 5;
  constexpr int RS = 32 * K + 33;  // odd: the 32 skewed rows fall in distinct banks
  int* ref = sm + w * 2 * RING * RS;
  int* sc = ref + RING * RS;
  for (int i = t; i < RING * RS; i += 32) ref[i] = (i * 7) % 13 - 4;
  __syncwarp();
  int Pv[K];  // the row above (the lane's previous row)
#pragma unroll
  for (int m = 0; m < K; ++m) Pv[m] = -t * 10 - m;
  int Lprev = 0;
  int vlast[RPS];
#pragma unroll
  for (int r = 0; r < RPS; ++r) vlast[r] = Pv[K - 1] + r;
  int row = (RING - t) & (RING - 1);
  const int negp = -p;
  int rvn[RPS][K];
#pragma unroll
  for (int r = 0; r < RPS; ++r)
#pragma unroll
    for (int m = 0; m < K; ++m) rvn[r][m] = ref[((row + r) & (RING - 1)) * RS + t * K + m];
  long long t0 = clock64();
#pragma unroll 4
  for (int s = 0; s < NSTEP; ++s) {
    const int* rr = ref + row * RS + t * K;
    int* ss = sc + row * RS + t * K;
    int fl[RPS];
#pragma unroll
    for (int r = 0; r < RPS; ++r) fl[r] = __shfl_up_sync(0xffffffffu, vlast[r], 1);
#pragma unroll
    for (int r = 0; r < RPS; ++r) {
      int rv[K];
#pragma unroll
      for (int m = 0; m < K; ++m) {
        if (PF) {
          rv[m] = rvn[r][m];
          rvn[r][m] = rr[((row + RPS + r) & (RING - 1)) * RS - row * RS + m];
        } else {
          rv[m] = rr[((row + r) & (RING - 1)) * RS - row * RS + m];
        }
      }
      const int L = t == 0 ? s + r : fl[r];
      int Y[K];
      int d = Lprev;
#pragma unroll
      for (int m = 0; m < K; ++m) {
        const int up = Pv[m];
        const int x = __viaddmax_s32(up, negp, d + rv[m]);
        Y[m] = m == 0 ? x : __viaddmax_s32(Y[m - 1], negp, x);
        d = up;
      }
#pragma unroll
      for (int m = 0; m < K; ++m) Pv[m] = __viaddmax_s32(L, -(m + 1) * p, Y[m]);
      Lprev = L;
      vlast[r] = Pv[K - 1];
#pragma unroll
      for (int m = 0; m < K; ++m) ss[((row + r) & (RING - 1)) * RS - row * RS + m] = Pv[m];
    }
    row = (row + RPS) & (RING - 1);
  }
  long long t1 = clock64();
  int acc = 0;
#pragma unroll
  for (int m = 0; m < K; ++m) acc += Pv[m];
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  if (t == 0 && blockIdx.x == 0) cyc[w] = t1 - t0;
}

template <int K, int RPS, int PF>
void run(int* out, long long* cyc, int nw) {
  constexpr int RS = 32 * K + 33;  // odd: the 32 skewed rows fall in distinct banks
  const size_t smem = (size_t)nw * 2 * RING * RS * 4;
  if (smem > 227 * 1024) { printf("K=%2d RPS=%d warps/SM=%2d  (smem too large)\n", K, RPS, nw); return; }
  cudaFuncSetAttribute(k_band<K, RPS, PF>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  long long h[32] = {0};
  for (int rep = 0; rep < 2; ++rep) {
    k_band<K, RPS, PF><<<148, 32 * nw, smem>>>(out, cyc, 10);
    cudaDeviceSynchronize();
  }
  cudaMemcpy(h, cyc, 8 * nw, cudaMemcpyDeviceToHost);
  double mx = 0;
  for (int i = 0; i < nw; ++i) mx = h[i] > mx ? h[i] : mx;
  const double cps = mx / NSTEP;  // cycles per step
  printf("K=%2d RPS=%d PF=%d warps/SM=%2d  %7.1f cycles/step  %6.2f cells/cycle/SM\n", K, RPS, PF, nw, cps,
         32.0 * K * RPS * nw / cps);
}

int main() {
  int* out;
  long long* cyc;
  cudaMalloc(&out, 148 * 1024 * 4);
  cudaMalloc(&cyc, 8 * 32);
  for (int nw : {1, 4}) {
    run<1, 1, 0>(out, cyc, nw);
    run<2, 1, 0>(out, cyc, nw);
    run<2, 1, 1>(out, cyc, nw);
    run<4, 1, 0>(out, cyc, nw);
    run<4, 1, 1>(out, cyc, nw);
    run<8, 1, 1>(out, cyc, nw);
    run<2, 2, 1>(out, cyc, nw);
    run<4, 2, 1>(out, cyc, nw);
  }
  printf("%s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
