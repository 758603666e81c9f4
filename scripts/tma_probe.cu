// tma_probe.cu — does a TMA tiled copy of one unaligned row segment (Rodinia pitch ld = n+1, odd)
// work through the "4-row fold" tensor map, and may its shared-memory destination be only 16-byte
// aligned (ring rows at a 1040-byte stride) or must it be 128-byte aligned?
//   nvcc -std=c++17 -O3 -gencode arch=compute_100a,code=sm_100a -o scripts/tma_probe scripts/tma_probe.cu
//   ./scripts/tma_probe <dst stride bytes> <c0>
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>

constexpr int ROWS = 64;
#ifndef BOXW
#define BOXW 256
#endif
constexpr int BOX = BOXW;

// MODE 0: tensor map as a __grid_constant__ parameter; 1: tensor map in global memory (tmg);
// 2: plain 1-D bulk copy (cp.async.bulk, 16-byte aligned source: c0 rounded down)
__global__ void k(const __grid_constant__ CUtensorMap tm, const CUtensorMap* tmg, int mode, int stride_b, int c0, int ld, int* bad, long long* cyc, const int* gsrc) {
  extern __shared__ __align__(1024) unsigned char sm[];
  __shared__ __align__(8) unsigned long long bar;
  const unsigned b = static_cast<unsigned>(__cvta_generic_to_shared(&bar));
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(b));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  long long t0 = clock64();
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(b), "r"(ROWS * BOX * 4) : "memory");
    for (int r = 0; r < ROWS; ++r) {
      const unsigned dst = static_cast<unsigned>(__cvta_generic_to_shared(sm + r * stride_b));
      const int x = (r & 3) * ld + c0, y = r >> 2;
      if (mode == 2) {
        const int* src = gsrc + (static_cast<long long>(r) * ld + c0) / 4 * 4;
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst), "l"(src), "r"(BOX * 4), "r"(b) : "memory");
      } else {
        const unsigned long long tmap = mode == 0 ? reinterpret_cast<unsigned long long>(&tm) : reinterpret_cast<unsigned long long>(tmg);
        asm volatile(
            "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(dst),
            "l"(tmap), "r"(x), "r"(y), "r"(b)
            : "memory");
      }
    }
  }
  long long t1 = clock64();
  {
    unsigned ok = 0;
    while (!ok)
      asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0; selp.u32 %0, 1, 0, p; }" : "=r"(ok) : "r"(b) : "memory");
  }
  long long t2 = clock64();
  int nb = 0;
  for (int r = 0; r < ROWS; ++r)
    for (int c = threadIdx.x; c < BOX; c += blockDim.x) {
      const int v = reinterpret_cast<const int*>(sm + r * stride_b)[c];
      const int cc = mode == 2 ? (r * ld + c0) / 4 * 4 - r * ld + c : c0 + c;  // (bulk: aligned-down start)
      const int want = (cc >= 0 && cc < ld) ? r * 100000 + cc : -1;  // beyond the row: ignore
      if (want >= 0 && v != want) ++nb;
    }
  atomicAdd(bad, nb);
  if (threadIdx.x == 0) cyc[0] = t1 - t0, cyc[1] = t2 - t0;
}

int main(int argc, char** argv) {
  const int stride_b = argc > 1 ? atoi(argv[1]) : 1024;
  const int c0 = argc > 2 ? atoi(argv[2]) : 1;
  const int mode = argc > 3 ? atoi(argv[3]) : 0;
  const int n = 1024, ld = n + 1;  // odd pitch: rows start at every 4-byte phase
  int* h = (int*)malloc(sizeof(int) * (n + 1) * ld);
  for (int r = 0; r <= n; ++r)
    for (int c = 0; c < ld; ++c) h[r * ld + c] = r * 100000 + c;
  int *d, *bad;
  long long* cyc;
  cudaMalloc(&d, sizeof(int) * (n + 1) * ld);
  cudaMalloc(&bad, 4);
  cudaMalloc(&cyc, 16);
  cudaMemset(bad, 0, 4);
  cudaMemcpy(d, h, sizeof(int) * (n + 1) * ld, cudaMemcpyHostToDevice);
  PFN_cuTensorMapEncodeTiled_v12000 enc = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", reinterpret_cast<void**>(&enc), cudaEnableDefault, &q);
  if (!enc) { printf("no cuTensorMapEncodeTiled\n"); return 1; }
  CUtensorMap tm;
  const int F = 4;
  cuuint64_t dims[2] = {static_cast<cuuint64_t>(F) * ld, static_cast<cuuint64_t>((n + 1) / F)};
  cuuint64_t strides[1] = {static_cast<cuuint64_t>(F) * ld * 4};
  cuuint32_t box[2] = {BOX, 1}, es[2] = {1, 1};
  CUresult cr = enc(&tm, CU_TENSOR_MAP_DATA_TYPE_INT32, 2, d, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                    CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (cr != CUDA_SUCCESS) { printf("encode failed %d\n", (int)cr); return 1; }
  const int smem = ROWS * stride_b + 1024;
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  CUtensorMap* tmg = nullptr;
  cudaMalloc(&tmg, sizeof(CUtensorMap));
  cudaMemcpy(tmg, &tm, sizeof(CUtensorMap), cudaMemcpyHostToDevice);
  k<<<1, 128, smem>>>(tm, tmg, mode, stride_b, c0, ld, bad, cyc, d);
  cudaError_t e = cudaDeviceSynchronize();
  int hb = -1;
  long long hc[2] = {0, 0};
  cudaMemcpy(&hb, bad, 4, cudaMemcpyDeviceToHost);
  cudaMemcpy(hc, cyc, 16, cudaMemcpyDeviceToHost);
  printf("mode %d stride %d B, c0 %d: %s, mismatches %d, issue %lld cyc for %d TMA, landed after %lld cyc\n", mode, stride_b, c0,
         e == cudaSuccess ? "ok" : cudaGetErrorString(e), hb, hc[0], ROWS, hc[1]);
  return 0;
}
