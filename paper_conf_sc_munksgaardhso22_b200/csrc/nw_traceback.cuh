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
//   * lane 0 walks the codes (each code is the move's address step, so a step is one
//     LDS -> IADD chain; row/column 0 of the window hold a stop code) until the path leaves the window, which takes
//     at least 31 steps, collecting the ops in shared memory; the warp then stores them to
//     global memory in traceback order;
//   * the border tail (all ups or all lefts) is written by the whole warp.
// A second kernel reverses each pair's ops in place into forward order (one thread per swapped
// byte pair, grid over the worst case n), so the result matches the oracle's layout.
#pragma once
#include <cstdint>

namespace nwb200 {

constexpr int kTbWarps = 4;   // warps per CTA
constexpr int kTbFewPairs = 296;  // up to 2 x 148 pairs: one pair per CTA
#ifndef NW_TB_FEW_WPP
#define NW_TB_FEW_WPP 16
#endif
constexpr int kTbFewWpp = NW_TB_FEW_WPP;  // warps per pair (and per CTA) for few pairs
#ifndef NW_TB_MANY_WPP
#define NW_TB_MANY_WPP 1
#endif
constexpr int kTbManyWpp = NW_TB_MANY_WPP;  // warps per pair for many pairs
constexpr int kTbRows = 33;   // window rows i-32 .. i (row 0 of the window = predecessor row)
constexpr int kTbLd = 33;     // move-code pitch (bytes)
// move codes in shared memory = the address step of the move in the code array
constexpr uint8_t kTbDiag = kTbLd + 1, kTbUp = kTbLd, kTbLeft = 1;
constexpr uint8_t kTbBad = 0xFE;   // no move reproduces the cell
constexpr uint8_t kTbStop = 0xFF;  // window row 0 / column 0: the path leaves the window

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

// WPP warps per pair (1 for large batches: kTbWarps pairs per CTA; 4 for few pairs: the
// window's rows are loaded and classified by kTbFewWpp = 16 warps, 2 rows each, and lane 0 of the first
// warp walks).  The group synchronises with a named barrier (id = group + 1).
template <int WPP, int NW = kTbWarps>
__global__ void __launch_bounds__(32 * NW) nw_traceback_kernel(TbParams P) {
  constexpr int G = NW / WPP;                // pairs per CTA
  constexpr int RPW = (kTbRows - 1) / WPP;   // window rows classified per warp
  __shared__ uint8_t sM[G][kTbRows * kTbLd];
  __shared__ uint8_t sO[G][2 * kTbRows];
  __shared__ long long sIJ[G][2];
  __shared__ int sK[G], sBad[G];
  const int wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int g = wid / WPP, sub = wid - g * WPP;
  const long long pair = static_cast<long long>(blockIdx.x) * G + g;
  if (pair >= P.batch) return;  // the whole group (same pair) leaves together
  const int32_t* __restrict__ S = P.score + pair * P.pss;
  const int32_t* __restrict__ R = P.ref + pair * P.psr;
  uint8_t* __restrict__ ops = P.ops + pair * P.ops_stride;
  uint8_t* wm = sM[g];
  uint8_t* wo = sO[g];
  const int32_t p = P.p;
  auto group_sync = [&]() {
    if constexpr (WPP == 1) __syncwarp();
    else asm volatile("bar.sync %0, %1;" ::"r"(g + 1), "r"(32 * WPP) : "memory");
  };

  if (sub == 0) wm[lane] = kTbStop;  // window row 0 (the predecessor row) stops the walk; column 0 below
  long long i = P.n, j = P.n, L = 0;
  int bad = 0;
  while (i > 0 && j > 0) {
    // window: rows i0..i (<= 33), columns j0..j (<= 32, lane c holds column j0 + c).  Rows and
    // columns past the window are clamped to it (valid addresses; their codes are never read).
    const long long i0 = i > kTbRows - 1 ? i - (kTbRows - 1) : 0, j0 = j > 31 ? j - 31 : 0;
    const int h = static_cast<int>(i - i0) + 1, w = static_cast<int>(j - j0) + 1;
    const int c = lane < w ? lane : w - 1;
    const int rb = sub * RPW;  // this warp loads window rows rb .. rb + RPW, classifies rb+1 ..
    const int32_t* sp = S + i0 * P.lds + j0 + c;
    const int32_t* rp = R + i0 * P.ldr + j0 + c;
    // one round of independent loads (all issued before the first use)
    int32_t vs[RPW + 1], vr[RPW + 1];
#pragma unroll
    for (int q = 0; q <= RPW; ++q) {
      const int rr = rb + q < h ? rb + q : h - 1;
      vs[q] = __ldg(sp + rr * P.lds);
      if (q >= 1) vr[q] = __ldg(rp + rr * P.ldr);
    }
    // move code of every cell (row >= 1, column lane >= 1): left / diagonal neighbours from
    // lane - 1 by shuffle
    int32_t diag = __shfl_up_sync(0xffffffffu, vs[0], 1);
#pragma unroll
    for (int q = 1; q <= RPW; ++q) {
      const int32_t left = __shfl_up_sync(0xffffffffu, vs[q], 1);
      const int32_t v = vs[q];
      const uint8_t m = diff_is(v, diag, vr[q]) ? kTbDiag : diff_is(vs[q - 1], v, p) ? kTbUp
                      : diff_is(left, v, p) ? kTbLeft : kTbBad;
      wm[(rb + q) * kTbLd + lane] = lane == 0 ? kTbStop : m;
      diag = left;
    }
    group_sync();
    if (sub == 0 && lane == 0) {
      // the code is the address step: one LDS -> IADD -> LDS chain per step
      int a = (h - 1) * kTbLd + (w - 1), k = 0;
      uint8_t m;
      while ((m = wm[a]) < kTbBad) {
        wo[k++] = m;
        a -= m;
      }
      const int ci = a / kTbLd;
      sIJ[g][0] = i0 + ci;
      sIJ[g][1] = j0 + (a - ci * kTbLd);
      sK[g] = k;
      sBad[g] = m == kTbBad;
    }
    group_sync();
    i = sIJ[g][0];
    j = sIJ[g][1];
    bad = sBad[g];
    const int k = sK[g];
    if (sub == 0)
      for (int e = lane; e < k; e += 32) ops[L + e] = wo[e] == kTbDiag ? 0 : (wo[e] == kTbUp ? 1 : 2);
    L += k;
    if (bad) break;
  }
  if (sub != 0) return;
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
