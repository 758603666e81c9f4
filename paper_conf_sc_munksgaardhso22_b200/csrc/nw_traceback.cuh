// nw_traceback.cuh — traceback of a filled score matrix (the step after
// the paper's path: Rodinia / the paper stop at the matrix, Fig. 2).
//
// From (n, n), each interior cell takes the first move, diagonal > up > left (DESIGN.md reading
// R12), whose predecessor reproduces its value under the Fig. 2 cell function
//     diagonal  S[i][j] == S[i-1][j-1] + ref[i][j]   op 0
//     up        S[i][j] == S[i-1][j] - p             op 1
//     left      S[i][j] == S[i][j-1] - p             op 2
// and on row 0 / column 0 the path follows the border to the origin.
//
// The walk is one dependent chain of up to 2n steps, so a pair is one warp and the design is
// about latency, not bandwidth (the matrix is read once along a ~33-cell-wide strip around the
// path: ~2n * 33 * 8 B, negligible next to the fill's 8n^2 B):
//   * window: the 33-row x 32-column block of S (and ref) whose bottom-right corner is the
//     current cell; lane c loads column c, all 66 loads of a lane issued before the first use
//     (one memory round trip per window);
//   * the warp classifies the window's 32 x 31 interior cells in registers (left / diagonal
//     neighbours by __shfl_up; int32 differences with an overflow test, exact like the oracle's
//     int64) into one move code per cell (3 = no move matches) in shared memory;
//   * lane 0 walks the codes (one LDS per step) until the path leaves the window, which takes
//     at least 31 steps, collecting the ops in shared memory; the warp then stores them to
//     global memory in traceback order;
//   * the border tail (all ups or all lefts) is written by the whole warp.
// A second kernel reverses each pair's ops in place into forward order (one thread per swapped
// byte pair, grid over the worst case n), so the result matches the oracle's layout.
#pragma once
#include <cstdint>

namespace nwb200 {

constexpr int kTbWarps = 4;   // pairs per CTA
constexpr int kTbRows = 33;   // window rows i-32 .. i (row 0 of the window = predecessor row)
constexpr int kTbLd = 33;     // move-code pitch (bytes)

struct TbParams {
  const int32_t* score;
  long long lds, pss;  // pitch, pair stride (elements)
  const int32_t* ref;
  long long ldr, psr;
  long long batch, n;
  int p;
  uint8_t* ops;
  long long ops_stride;  // bytes between pairs' op buffers (>= 2n)
  int32_t* len;          // per pair: path length, or -1 (a cell matches no move)
};

// x - y == want, exactly (as integers): the int32 difference plus its signed-overflow test
__device__ __forceinline__ bool diff_is(int32_t x, int32_t y, int32_t want) {
  const int32_t d = static_cast<int32_t>(static_cast<uint32_t>(x) - static_cast<uint32_t>(y));
  return d == want && ((x ^ y) & (x ^ d)) >= 0;
}

__global__ void __launch_bounds__(32 * kTbWarps) nw_traceback_kernel(TbParams P) {
  __shared__ uint8_t sM[kTbWarps][kTbRows * kTbLd];
  __shared__ uint8_t sO[kTbWarps][2 * kTbRows];
  const int wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const long long pair = static_cast<long long>(blockIdx.x) * kTbWarps + wid;
  if (pair >= P.batch) return;
  const int32_t* __restrict__ S = P.score + pair * P.pss;
  const int32_t* __restrict__ R = P.ref + pair * P.psr;
  uint8_t* __restrict__ ops = P.ops + pair * P.ops_stride;
  uint8_t* wm = sM[wid];
  uint8_t* wo = sO[wid];
  const int32_t p = P.p;

  long long i = P.n, j = P.n, L = 0;
  int bad = 0;
  while (i > 0 && j > 0) {
    // window: rows i0..i (<= 33), columns j0..j (<= 32, lane c holds column j0 + c).  Rows and
    // columns past the window are clamped to it (valid addresses; their codes are never read).
    const long long i0 = i > kTbRows - 1 ? i - (kTbRows - 1) : 0, j0 = j > 31 ? j - 31 : 0;
    const int h = static_cast<int>(i - i0) + 1, w = static_cast<int>(j - j0) + 1;
    const int c = lane < w ? lane : w - 1;
    const int32_t* sp = S + i0 * P.lds + j0 + c;
    const int32_t* rp = R + i0 * P.ldr + j0 + c;
    // one round of independent loads (all issued before the first use)
    int32_t vs[kTbRows], vr[kTbRows];
#pragma unroll
    for (int r = 0; r < kTbRows; ++r) {
      const int rr = r < h ? r : h - 1;
      vs[r] = __ldg(sp + rr * P.lds);
      if (r >= 1) vr[r] = __ldg(rp + rr * P.ldr);
    }
    // move code of every cell (row r >= 1, column lane >= 1): left / diagonal neighbours from
    // lane - 1 by shuffle
    int32_t diag = __shfl_up_sync(0xffffffffu, vs[0], 1);
#pragma unroll
    for (int r = 1; r < kTbRows; ++r) {
      const int32_t left = __shfl_up_sync(0xffffffffu, vs[r], 1);
      const int32_t v = vs[r];
      const uint8_t m = diff_is(v, diag, vr[r]) ? 0 : diff_is(vs[r - 1], v, p) ? 1 : diff_is(left, v, p) ? 2 : 3;
      wm[r * kTbLd + lane] = m;
      diag = left;
    }
    __syncwarp();
    int k = 0;
    if (lane == 0) {
      int ci = h - 1, cj = w - 1;
      while (ci > 0 && cj > 0) {
        const uint8_t m = wm[ci * kTbLd + cj];
        if (m == 3) {
          bad = 1;
          break;
        }
        wo[k++] = m;
        ci -= (m != 2);
        cj -= (m != 1);
      }
      i = i0 + ci;
      j = j0 + cj;
    }
    i = __shfl_sync(0xffffffffu, i, 0);
    j = __shfl_sync(0xffffffffu, j, 0);
    k = __shfl_sync(0xffffffffu, k, 0);
    bad = __shfl_sync(0xffffffffu, bad, 0);
    __syncwarp();
    for (int e = lane; e < k; e += 32) ops[L + e] = wo[e];
    L += k;
    __syncwarp();
    if (bad) break;
  }
  if (bad) {
    if (lane == 0) P.len[pair] = -1;
    return;
  }
  // border tail, traceback order: i ups (column 0), then j lefts (row 0); one of them is 0
  for (long long e = lane; e < i + j; e += 32) ops[L + e] = e < i ? 1 : 2;
  if (lane == 0) P.len[pair] = static_cast<int32_t>(L + i + j);
}

// ops[0..len) of each pair: traceback order -> forward order (thread t swaps t <-> len-1-t).
__global__ void nw_traceback_reverse_kernel(uint8_t* __restrict__ ops, long long ops_stride,
                                            const int32_t* __restrict__ len, long long batch) {
  for (long long pair = blockIdx.y; pair < batch; pair += gridDim.y) {
    const int32_t L = len[pair];
    uint8_t* o = ops + pair * ops_stride;
    for (long long t = static_cast<long long>(blockIdx.x) * blockDim.x + threadIdx.x; t < L / 2;
         t += static_cast<long long>(gridDim.x) * blockDim.x) {
      const uint8_t x = o[t], y = o[L - 1 - t];
      o[t] = y;
      o[L - 1 - t] = x;
    }
  }
}

}  // namespace nwb200
