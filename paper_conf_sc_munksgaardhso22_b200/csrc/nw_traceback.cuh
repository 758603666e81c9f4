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
//   * window: the 33 x 33 block of S (and ref) whose bottom-right corner is the current cell is
//     loaded by the warp in one round of independent coalesced loads;
//   * the warp then classifies all 32 x 32 interior cells of the window in parallel (one move
//     code per cell, 3 = no move matches) into shared memory;
//   * lane 0 walks the codes (one LDS per step) until the path leaves the window, which takes
//     at least 32 steps; the ops go to global memory in traceback order;
//   * the border tail (all ups or all lefts) is written by the whole warp.
// A second kernel reverses each pair's ops in place into forward order (one thread per swapped
// byte pair, grid over the worst case n), so the result matches the oracle's layout.
#pragma once
#include <cstdint>

namespace nwb200 {

constexpr int kTbWarps = 4;        // pairs per CTA
constexpr int kTbWin = 32;         // window: (kTbWin+1)^2 cells incl. the predecessor row/column
constexpr int kTbLd = kTbWin + 1;  // odd pitch: column-wise LDS are bank-conflict free

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

__global__ void __launch_bounds__(32 * kTbWarps) nw_traceback_kernel(TbParams P) {
  __shared__ int32_t sS[kTbWarps][kTbLd * kTbLd];
  __shared__ int32_t sR[kTbWarps][kTbLd * kTbLd];
  __shared__ uint8_t sM[kTbWarps][kTbLd * kTbLd];
  const int wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const long long pair = static_cast<long long>(blockIdx.x) * kTbWarps + wid;
  if (pair >= P.batch) return;
  const int32_t* __restrict__ S = P.score + pair * P.pss;
  const int32_t* __restrict__ R = P.ref + pair * P.psr;
  uint8_t* __restrict__ ops = P.ops + pair * P.ops_stride;
  int32_t* ws = sS[wid];
  int32_t* wr = sR[wid];
  uint8_t* wm = sM[wid];
  const long long p = P.p;

  long long i = P.n, j = P.n, L = 0;
  int bad = 0;
  while (i > 0 && j > 0) {
    const long long i0 = i > kTbWin ? i - kTbWin : 0, j0 = j > kTbWin ? j - kTbWin : 0;
    const int h = static_cast<int>(i - i0) + 1, w = static_cast<int>(j - j0) + 1;
    // one round of independent loads: row r of the window, lanes across the columns
    for (int e = lane; e < h * kTbLd; e += 32) {
      const int r = e / kTbLd, c = e - r * kTbLd;
      if (c < w) {
        ws[r * kTbLd + c] = __ldg(S + (i0 + r) * P.lds + j0 + c);
        wr[r * kTbLd + c] = __ldg(R + (i0 + r) * P.ldr + j0 + c);
      }
    }
    __syncwarp();
    // classify every interior cell of the window (rows/cols >= 1 of the window)
    for (int e = lane; e < (h - 1) * kTbLd; e += 32) {
      const int r = 1 + e / kTbLd, c = e - (r - 1) * kTbLd;
      if (c >= 1 && c < w) {
        const long long v = ws[r * kTbLd + c];
        uint8_t m = 3;
        if (v == static_cast<long long>(ws[(r - 1) * kTbLd + c - 1]) + wr[r * kTbLd + c]) m = 0;
        else if (v == static_cast<long long>(ws[(r - 1) * kTbLd + c]) - p) m = 1;
        else if (v == static_cast<long long>(ws[r * kTbLd + c - 1]) - p) m = 2;
        wm[r * kTbLd + c] = m;
      }
    }
    __syncwarp();
    if (lane == 0) {
      int ci = h - 1, cj = w - 1;
      long long l = L;
      while (ci > 0 && cj > 0) {
        const uint8_t m = wm[ci * kTbLd + cj];
        if (m == 3) {
          bad = 1;
          break;
        }
        ops[l++] = m;
        ci -= (m != 2);
        cj -= (m != 1);
      }
      i = i0 + ci;
      j = j0 + cj;
      L = l;
    }
    i = __shfl_sync(0xffffffffu, i, 0);
    j = __shfl_sync(0xffffffffu, j, 0);
    L = __shfl_sync(0xffffffffu, L, 0);
    bad = __shfl_sync(0xffffffffu, bad, 0);
    __syncwarp();
    if (bad) break;
  }
  if (bad) {
    if (lane == 0) P.len[pair] = -1;
    return;
  }
  // border tail, traceback order: i ups (column 0), then j lefts (row 0); one of them is 0
  for (long long k = lane; k < i + j; k += 32) ops[L + k] = k < i ? 1 : 2;
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
