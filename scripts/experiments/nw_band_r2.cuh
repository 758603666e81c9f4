// nw_band.cuh — the persistent NW wavefront kernel, round 2.
//
// What it computes (Fig. 2, with Rodinia's cell function, R1):
//     score[i][j] = max(score[i-1][j-1] + ref[i][j], score[i-1][j] - p, score[i][j-1] - p)
// for every interior cell, each value written ONCE, in place, into score (the short-circuited
// update of P:512-516 / P:616-656: no temporary array, no copy).
//
// Geometry.  A band = W = 32 K adjacent columns x all rows, swept by ONE compute warp: lane t owns
// columns c0 + tK .. c0 + tK + K - 1 and at step s computes row s + 1 - t (the intra-tile
// anti-diagonals of P:498-501, skewed one row per lane).  A CTA owns a GROUP of NC consecutive
// bands: NC compute warps, NC staging warps (one per band: ref rows in, score rows out) and one
// border warp (the group's left border column in); for NC = 2 the compute and staging warps take
// one SM sub-partition each.  CTAs claim groups through an atomic ticket in wavefront order (band
// k waits only on band k-1: deadlock free without co-residency).
//
// The cell, in plain S form (no gap normalisation, so every intermediate is a true candidate
// value and int32 cannot overflow under the nw.h range contract):
//     d_m = diag_m + ref_m                       (IMAD, FMA pipe)
//     x_m = max(up_m - p, d_m)                   (VIADDMNMX)
//     Y_0 = x_0,  Y_m = max(Y_{m-1} - p, x_m)    (VIADDMNMX: the row's left chain inside the lane)
//     S_m = max(L - (m+1) p, Y_m)                (VIADDMNMX: the left value L enters once per cell)
// L is lane t-1's last column of the same row (SHFL.UP) or, for lane 0, the band's left border.
//
// Step-indexed ("skewed") shared rings: at step s EVERY lane of a compute warp reads ref slot
// s mod RR and writes score slot s mod SR, so the compute warp's shared addresses are
// warp-uniform (no per-step address arithmetic).  Slot x holds, for lane L, ref row x + 2 - L and
// score row x + 1 - L: the staging warp applies the skew (its reads and writes stay bank-conflict
// free: the row stride is 0 mod 32 words and a warp covers 32 consecutive words of one row).
//
// Synchronisation (formal under the PTX memory model; mbarrier arrive = release at CTA scope with
// no MEMBAR, test_wait = acquire), per band:
//   cdone[c]   compute -> staging, arrived at event c+1: ref slot chunk c (slots 16c..16c+15)
//              has been read and score row chunk c-2 (rows 16c-31 .. 16c-16) is complete;
//   ready[c]   staging -> compute: ref slot chunk c landed (32 cp.async.mbarrier.arrive.noinc)
//              and score row chunk c - SR/16 stored (one arrive): the block's slots are usable;
//   entfree[b] compute -> producer of its left border: border block b read.
// Band borders travel as 64-bit entries {value, tag} (flag fused with the value; every access a
// single 8-byte relaxed operation, so single-copy atomic): into band w's shared in-ring from
// compute warp w-1 or, for band 0 of the group, from the border warp (tag = gen | row), which
// forwards the previous group's global entries (tag = launch epoch, relaxed gpu-scope stores,
// polled with relaxed sys-scope loads), a strip halo (sys scope) or the plain score column.
// A compute warp never holds a long-latency load in a register across its step loop (a pending
// load's scoreboard would alias the steps' and stall them: measured 45-75 cycles per step).
#pragma once
#include <cstdint>
#include <utility>

#include "nw_common.cuh"

namespace nwb200 {

// timing experiments only (scripts/, results invalid): bit 0 skips the ref copies, bit 1 the
// score stores, bit 2 the compute warps' ready waits, bit 3 their border waits, bit 4 runs no
// helper warps; the release build has NW_EXP = 0
#ifndef NW_EXP
#define NW_EXP 0
#endif
#ifndef NW_SPLIT
#define NW_SPLIT 0  // (experiments) NC = 1: separate ref and store warps
#endif
#ifndef NW_SPREAD
#define NW_SPREAD 0  // (experiments) staging: pause (ns) between groups of 4 rows
#endif
#ifndef NW_STAGE_SLEEP
#define NW_STAGE_SLEEP 0  // staging-warp idle back-off (ns; 0: none)
#endif

template <int K_, int NC_>
struct BandCfg {
  static constexpr int K = K_, NC = NC_;
  static constexpr int W = 32 * K;
  static constexpr int CH = 16;                        // rows per chunk = steps per event = border block
  // ring slots (multiples of 16; wraps by one unsigned-min, so not necessarily powers of two).
  // Ref: a row chunk lands in slots 16k-1 .. 16k+45, so the copy of row chunk k waits for slot
  // chunk k + 2 - NRB to be read and runs NRB - 4 blocks ahead of the compute warp.  Score: row
  // chunk k occupies slots 16k .. 16k+46 and may be stored after event k+3: NSB - 3 blocks of slack.
  static constexpr int RR = K == 8 ? 96 : ((K * NC >= 8) ? 112 : 128);
  static constexpr int SR = K == 8 ? 96 : ((K * NC >= 8) ? 96 : 128);
  static constexpr int NRB = RR / CH, NSB = SR / CH;   // chunk slots
  // cdone / ready barrier rings: an arrival for chunk c must follow the completion of the phase of
  // chunk c - NRDY (ready: copies follow cdone[c + 3 - NRB], stores follow cdone[c - NSB + 2])
  static constexpr int NRDY = 8;
  // ring row layout (words).  K <= 4: the band's W words in order (row stride 0 mod 32: a lane's
  // K-word vector loads / stores of one slot are bank-conflict free).  K = 8: lane L's words 0..3
  // at 4L, words 4..7 at HALF + 4L (HALF = 144: the second half shifted by 16 banks), so both of a
  // lane's LDS.128 / STS.128 and the staging warps' 32 consecutive words stay conflict free.
  static constexpr int HALF = K == 8 ? 144 : W;
  static constexpr int RS = K == 8 ? 2 * HALF : W;
  static constexpr int RS4 = 4 * RS;
  __host__ __device__ static constexpr int word_pos(int wd) {
    return K == 8 ? ((wd & 7) < 4 ? 4 * (wd >> 3) + (wd & 7) : HALF + 4 * (wd >> 3) + (wd & 7) - 4) : wd;
  }
  __host__ __device__ static constexpr int lane_off(int t) { return K == 8 ? 16 * t : 4 * K * t; }  // bytes
  static constexpr int BR = 256, NBB = BR / CH;        // border in-ring per band (entries / blocks)
  static constexpr int BP = 4;                         // out-ring back-pressure checked every BP events
  // warp roles (warp w runs on SM sub-partition w % 4): [0, NC) compute, [NC, 2NC) staging (ref
  // rows in and score rows out of band w - NC), 2NC the border-in warp (NC = 2: the compute and
  // staging warps take one sub-partition each; the mostly waiting border warp shares the first).
  // NC = 1: separate ref and store warps (compute, ref, store, border: one sub-partition each)
  static constexpr bool SPLIT = NW_SPLIT && NC == 1;
  static constexpr int NWARPS = SPLIT ? 4 : 2 * NC + 1;
  static constexpr int W_BORDER = SPLIT ? 3 : 2 * NC;
  // shared layout: [0] ticket, [16..] mbarriers, then per band ref ring, score ring, border in-ring
  static constexpr int NBAR_BAND = 2 * NRDY + NBB;
  static constexpr int NBAR = NC * NBAR_BAND;
  static constexpr size_t HDR = (static_cast<size_t>(16 + 8 * NBAR) + 127) / 128 * 128;
  static constexpr size_t REF_BYTES = static_cast<size_t>(RR) * RS4, SC_BYTES = static_cast<size_t>(SR) * RS4;
  static constexpr size_t LINK_BYTES = static_cast<size_t>(BR) * 8;
  static constexpr size_t BAND_BYTES = REF_BYTES + SC_BYTES + LINK_BYTES;
  static constexpr size_t kSmem = HDR + NC * BAND_BYTES;
  static_assert(K == 2 || K == 4 || K == 8, "K/4 LDS.128 or one LDS.64 per step");
  static_assert(NC >= 1 && NC <= 3 && NWARPS <= 8, "geometry");
  static_assert(kSmem <= 232448, "shared memory per CTA");
  static_assert(RR % CH == 0 && SR % CH == 0 && NRB >= 6 && NSB >= 4, "rings: lookahead and store slack of at least one block");
  static_assert(NRDY > NRB - 4 && NRDY > NSB - 3 && NRDY >= 4, "barrier rings deep enough for the arrival order");
  static_assert(NBB >= 2 * BP + 4, "border in-ring deep enough for the periodic back-pressure check");
};

// ---- small PTX helpers --------------------------------------------------------------------
__device__ __forceinline__ void bar_init(uint32_t a, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(a), "r"(count) : "memory");
}
__device__ __forceinline__ void bar_inval(uint32_t a) {
  asm volatile("mbarrier.inval.shared::cta.b64 [%0];" ::"r"(a) : "memory");
}
__device__ __forceinline__ void bar_arrive(uint32_t a) {
  asm volatile("{ .reg .b64 st; mbarrier.arrive.release.cta.shared::cta.b64 st, [%0]; }" ::"r"(a) : "memory");
}
__device__ __forceinline__ void bar_arrive_p(bool p, uint32_t a) {  // (no branch: a predicated arrive)
  asm volatile("{ .reg .pred q; .reg .b64 st; setp.ne.b32 q, %0, 0; @q mbarrier.arrive.release.cta.shared::cta.b64 st, [%1]; }" ::"r"(
                   static_cast<int>(p)),
               "r"(a)
               : "memory");
}
__device__ __forceinline__ bool bar_test(uint32_t a, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{ .reg .pred p; mbarrier.test_wait.parity.acquire.cta.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
      : "=r"(ok)
      : "r"(a), "r"(parity)
      : "memory");
  return ok != 0;
}
// bounded wait for the phase with the given parity to complete (watchdog: error word + trap)
// (sleep_ns > 0: helper warps back off instead of competing with the compute warps' issue slots)
__device__ __noinline__ void bar_spin(uint32_t a, uint32_t parity, const StripParams& P, unsigned sleep_ns) {
  const uint64_t t0 = globaltimer_ns();
  unsigned spins = 0;
  while (!bar_test(a, parity)) {
    if (sleep_ns) __nanosleep(sleep_ns);
    if ((++spins & 255u) == 0 && globaltimer_ns() - t0 > P.spin_limit_ns) watchdog_trap(P.err);
  }
}
__device__ __forceinline__ void bar_wait(uint32_t a, uint32_t parity, const StripParams& P, unsigned sleep_ns = 0) {
  if (!bar_test(a, parity)) bar_spin(a, parity, P, sleep_ns);
}
__device__ __forceinline__ void cpa_arrive_noinc(uint32_t a) {
  asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(a) : "memory");
}
__device__ __forceinline__ void cpa4(uint32_t dst, const void* src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(dst), "l"(src) : "memory");
}
__device__ __forceinline__ void cpa4_p(bool p, uint32_t dst, const void* src) {
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %0, 0; @q cp.async.ca.shared.global [%1], [%2], 4; }" ::"r"(static_cast<int>(p)), "r"(dst),
               "l"(src)
               : "memory");
}
__device__ __forceinline__ uint64_t ld_rlx_sys_p(bool p, const uint64_t* g) {
  uint64_t v = 0;
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %1, 0; @q ld.relaxed.sys.global.b64 %0, [%2]; }" : "+l"(v) : "r"(static_cast<int>(p)), "l"(g)
               : "memory");
  return v;
}
__device__ __forceinline__ uint64_t ld_rlx_gpu_p(bool p, const uint64_t* g) {
  uint64_t v = 0;
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %1, 0; @q ld.relaxed.gpu.global.b64 %0, [%2]; }" : "+l"(v) : "r"(static_cast<int>(p)), "l"(g)
               : "memory");
  return v;
}
__device__ __forceinline__ uint64_t ld_rlx_cta_smem(uint32_t a) {
  uint64_t v;
  asm volatile("ld.relaxed.cta.shared.b64 %0, [%1];" : "=l"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ uint64_t pack_entry(int v, uint32_t tag) {
  return (static_cast<uint64_t>(tag) << 32) | static_cast<uint32_t>(v);
}
__device__ __forceinline__ void st_ent_smem_p(bool p, uint32_t a, uint64_t e) {
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %0, 0; @q st.relaxed.cta.shared.b64 [%1], %2; }" ::"r"(static_cast<int>(p)), "r"(a), "l"(e)
               : "memory");
}
// two consecutive ring entries (16-byte aligned) in one store of two 8-byte elements
template <int OFF>
__device__ __forceinline__ void st_pair_smem_p(int p, uint32_t a, uint64_t e0, uint64_t e1) {
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %0, 0; @q st.relaxed.cta.shared.v2.b64 [%1+%4], {%2, %3}; }" ::"r"(p), "r"(a), "l"(e0), "l"(e1),
               "n"(OFF)
               : "memory");
}
template <int OFF, bool SYS>
__device__ __forceinline__ void st_pair_global_p(int p, uint64_t* g, uint64_t e0, uint64_t e1) {
  if constexpr (SYS)
    asm volatile("{ .reg .pred q; setp.ne.b32 q, %0, 0; @q st.relaxed.sys.global.v2.b64 [%1+%4], {%2, %3}; }" ::"r"(p), "l"(g), "l"(e0), "l"(e1),
                 "n"(OFF)
                 : "memory");
  else
    asm volatile("{ .reg .pred q; setp.ne.b32 q, %0, 0; @q st.relaxed.gpu.global.v2.b64 [%1+%4], {%2, %3}; }" ::"r"(p), "l"(g), "l"(e0), "l"(e1),
                 "n"(OFF)
                 : "memory");
}
__device__ __forceinline__ void st_ent_gpu_p(bool p, uint64_t* g, uint64_t e) {
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %0, 0; @q st.relaxed.gpu.global.b64 [%1], %2; }" ::"r"(static_cast<int>(p)), "l"(g), "l"(e)
               : "memory");
}
__device__ __forceinline__ void st_ent_sys_p(bool p, uint64_t* g, uint64_t e) {
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %0, 0; @q st.relaxed.sys.global.b64 [%1], %2; }" ::"r"(static_cast<int>(p)), "l"(g), "l"(e)
               : "memory");
}
template <int K, int HALF4 = 0>
__device__ __forceinline__ void lds_ref(uint32_t a, int* v) {
  if constexpr (K == 2) {
    asm volatile("ld.shared.v2.b32 {%0, %1}, [%2];" : "=r"(v[0]), "=r"(v[1]) : "r"(a) : "memory");
  } else {
    asm volatile("ld.shared.v4.b32 {%0, %1, %2, %3}, [%4];" : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]) : "r"(a) : "memory");
    if constexpr (K == 8)
      asm volatile("ld.shared.v4.b32 {%0, %1, %2, %3}, [%4+%5];" : "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]) : "r"(a), "n"(HALF4) : "memory");
  }
}
template <int K, int HALF4 = 0>
__device__ __forceinline__ void sts_score(uint32_t a, const int* v) {
  if constexpr (K == 2) {
    asm volatile("st.shared.v2.b32 [%0], {%1, %2};" ::"r"(a), "r"(v[0]), "r"(v[1]) : "memory");
  } else {
    asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]) : "memory");
    if constexpr (K == 8)
      asm volatile("st.shared.v4.b32 [%0+%5], {%1, %2, %3, %4};" ::"r"(a), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]), "n"(HALF4) : "memory");
  }
}
__device__ __forceinline__ int lds32(uint32_t a) {
  int v;
  asm volatile("ld.shared.b32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ int imad1(int a, int one, int b) {  // a + b on the FMA pipe
  int d;
  asm("mad.lo.s32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(one), "r"(b));
  return d;
}

// ---- one band's geometry (uniform) ------------------------------------------------------------
struct BandTask {
  int n, p, band, c0, ws, g;  // g: group within the pair
  long long pair;
  bool last_band;
  int32_t* S;
  const int32_t* R;
};

template <class C>
struct BandSmem {
  uint32_t base;  // shared window address of the dynamic smem
  __device__ __forceinline__ uint32_t bar(int i) const { return base + 16u + 8u * static_cast<uint32_t>(i); }
  __device__ __forceinline__ uint32_t cdone(int w, int c) const { return bar(w * C::NBAR_BAND + (c & (C::NRDY - 1))); }
  __device__ __forceinline__ uint32_t ready(int w, int c) const { return bar(w * C::NBAR_BAND + C::NRDY + (c & (C::NRDY - 1))); }
  // entfree(w, b): the in-ring of band w
  __device__ __forceinline__ uint32_t entfree(int w, int b) const { return bar(w * C::NBAR_BAND + 2 * C::NRDY + (b & (C::NBB - 1))); }
  __device__ __forceinline__ uint32_t refR(int w) const { return base + static_cast<uint32_t>(C::HDR + w * C::BAND_BYTES); }
  __device__ __forceinline__ uint32_t scR(int w) const { return refR(w) + static_cast<uint32_t>(C::REF_BYTES); }
  __device__ __forceinline__ uint32_t link(int w) const { return scR(w) + static_cast<uint32_t>(C::SC_BYTES); }  // band w's in-ring
};

// border-ring slot of row r: (r - 2) mod BR, so that the 16 rows a compute warp's lane 31 finishes in
// one steady block (rows 16Q - 30 .. 16Q - 15) fill 16 consecutive slots starting at a multiple of 16
template <class C>
__device__ __forceinline__ uint32_t ring_slot(int r) { return static_cast<uint32_t>(r - 2) & (C::BR - 1); }

// parity of the use of chunk k of a ring of NB slots
__device__ __forceinline__ uint32_t phase_of(int k, int nb) { return static_cast<uint32_t>((k / nb) & 1); }

// ---- the staging warp of band slot w: ref rows in, score rows out ------------------------------
// Ref, by SLOT chunks: slot chunk c = slots 16c .. 16c+15; slot x holds, for compute lane L, ref
// row x + 2 - L, so for a fixed (lane, word) the source rows of a slot chunk are 16 consecutive
// rows and the destinations 16 consecutive slots: one base pointer per word, immediates for the
// slots (a warp instruction reads 8 row segments of 16 bytes; the L1 keeps the rest of each line
// for the next slots).  Copied once its physical chunk has been read (cdone[c - NRB]); completion
// is counted on ready[c] (32 cp.async.mbarrier.arrive.noinc).
// Score, by ROW chunks: row chunk k (rows 16k+1 .. 16k+16) once complete (cdone[k+2]); word
// 32i+t of row r sits in slot (r - 1 + L) (L = (32i+t)/K): the slot's byte offset is
// (o + imm) & MASK, two ALU operations per load; the global stores are coalesced by row.  Then
// one arrive on ready[k + SR/16] (the slots the compute warp rewrites in that block are free).
// ROLE: kStageRef (ref rows in), kStageStore (score rows out) or both.
enum : int { kStageRef = 1, kStageStore = 2 };
template <class C, bool AL, int ROLE>
__device__ __forceinline__ void band_stage_warp(const StripParams& P, const BandTask& b, const BandSmem<C>& sm, const int w, const int t) {
  constexpr bool DO_REF = (ROLE & kStageRef) != 0, DO_ST = (ROLE & kStageStore) != 0;
  constexpr int K = C::K, CH = C::CH, RR = C::RR, SR = C::SR, RS4 = C::RS4;
  constexpr int PF = 6;  // L2 prefetch distance (row chunks)
  const int n = b.n;
  const int nch = (n + CH - 1) / CH;        // row chunks
  const int nblk = (n + 31 + CH - 1) / CH;  // the compute warp's blocks: one ready phase each
  const bool full = b.ws == C::W;
  const uint64_t ldr4 = 4ull * static_cast<uint64_t>(P.ldr), lds4 = 4ull * static_cast<uint64_t>(P.lds);
  const char* const R0 = reinterpret_cast<const char*>(b.R + b.c0);  // (row 0, band column 0) of ref
  char* const S0 = reinterpret_cast<char*>(b.S + b.c0);
  const uint32_t refR = sm.refR(w), scR = sm.scR(w);
  constexpr int NL = (4 * C::W + 127) / 128 + 1;  // 128-byte lines of one row segment
  auto prefetch = [&](int k) {
    for (int f = t; f < CH * NL; f += 32) {
      const int i = f / NL, ln = f - i * NL;
      const int r = CH * k + 1 + i;
      if (r <= n) {
        const uint64_t ga = (reinterpret_cast<uint64_t>(R0) + static_cast<uint64_t>(r) * ldr4) & ~127ull;
        asm volatile("prefetch.global.L2 [%0];" ::"l"(ga + 128u * ln));
      }
    }
  };
  if (DO_REF)
    for (int k = 0; k < PF && k < nch; ++k) prefetch(k);

  // one unsigned min wraps an offset in [0, 2 ring) into [0, ring) (VIADDMNMX.U32)
  auto wrap = [](uint32_t o, uint32_t ring_bytes) -> uint32_t { return __viaddmin_u32(o, 0u - ring_bytes, o); };
  constexpr uint32_t RBYTES = static_cast<uint32_t>(RR * RS4), SBYTES = static_cast<uint32_t>(SR * RS4);
  // row chunk k of ref: rows r0 = 16k+1 .. 16k+16, row-major (each warp instruction reads 128
  // contiguous bytes of one row); word 32i+t of row R goes to slot R - 2 + L_i, L_i = (32i+t)/K
  // AL (every row 16-byte aligned at the band's first column, full band): staging lane t moves
  // compute lane t's K words of a row with one 16-byte (K = 4) / 8-byte (K = 2) copy, load and
  // store: a warp instruction still covers one contiguous row segment
  constexpr int VW = K == 2 ? 2 : 4;  // words per staging lane in the AL path
  // staging lane t, vector v: 16 bytes (K = 2: 8) of the row segment = band words
  // wd = 32 VW v + VW t .. + VW - 1, owned by compute lane wd / K (NV vectors per lane and row)
  constexpr int NV = C::W / (32 * VW);
  auto copy_row_chunk_al = [&](int k) {
    const int r0 = CH * k + 1;
#pragma unroll
    for (int v = 0; v < NV; ++v) {
      const int wd = 32 * VW * v + VW * t;
      const char* g = R0 + static_cast<int64_t>(r0) * static_cast<int64_t>(ldr4) + 4 * wd;
      const uint32_t o = static_cast<uint32_t>(((r0 - 2 + wd / K + RR) % RR) * RS4 + 4 * C::word_pos(wd));
#pragma unroll
      for (int j = 0; j < CH; ++j) {
        const int r = r0 + j;
        const int ok = r <= n && !(r == 1 && wd / K == 0);
        const uint32_t d = refR + wrap(o + j * RS4, RBYTES);
        if constexpr (VW == 4)
          asm volatile("{ .reg .pred q; setp.ne.b32 q, %0, 0; @q cp.async.cg.shared.global [%1], [%2], 16; }" ::"r"(ok), "r"(d), "l"(g)
                       : "memory");
        else
          asm volatile("{ .reg .pred q; setp.ne.b32 q, %0, 0; @q cp.async.ca.shared.global [%1], [%2], 8; }" ::"r"(ok), "r"(d), "l"(g)
                       : "memory");
        g += ldr4;
      }
    }
  };
  // Score row chunk k out: every shared-memory read of the chunk first, then the arrive that frees
  // its slots (release: it orders the reads; issued before this chunk's global stores, so it does
  // not wait for their L2 acknowledgements), then the coalesced global stores.
  auto release = [&](int k) {
    __syncwarp();  // every lane's ring reads are done before the slots are released
    if (NW_EXP & 128) {  // (timing experiment: relaxed arrive)
      if (t == 0) asm volatile("{ .reg .b64 st; mbarrier.arrive.relaxed.cta.shared::cta.b64 st, [%0]; }" ::"r"(sm.ready(w, k + C::NSB)) : "memory");
    } else if (t == 0) {
      bar_arrive(sm.ready(w, k + C::NSB));
    }
  };
  auto store_row_chunk_al = [&](int k) {
    const int r0 = CH * k + 1;
    int v[NV][CH][VW];
#pragma unroll
    for (int q = 0; q < NV; ++q) {
      const int wd = 32 * VW * q + VW * t;
      const uint32_t o = static_cast<uint32_t>(((r0 - 1 + wd / K) % SR) * RS4 + 4 * C::word_pos(wd));
#pragma unroll
      for (int j = 0; j < CH; ++j) {
        const uint32_t a = scR + wrap(o + j * RS4, SBYTES);
        if constexpr (VW == 4)
          asm volatile("ld.shared.v4.b32 {%0, %1, %2, %3}, [%4];" : "=r"(v[q][j][0]), "=r"(v[q][j][1]), "=r"(v[q][j][2]), "=r"(v[q][j][3]) : "r"(a)
                       : "memory");
        else
          asm volatile("ld.shared.v2.b32 {%0, %1}, [%2];" : "=r"(v[q][j][0]), "=r"(v[q][j][1]) : "r"(a) : "memory");
      }
    }
    release(k);
#pragma unroll
    for (int q = 0; q < NV; ++q) {
      char* g = S0 + static_cast<int64_t>(r0) * static_cast<int64_t>(lds4) + 4 * (32 * VW * q + VW * t);
#pragma unroll
      for (int j = 0; j < CH; ++j) {
        if (r0 + j <= n) {
          if constexpr (VW == 4)
            *reinterpret_cast<int4*>(g) = make_int4(v[q][j][0], v[q][j][1], v[q][j][2], v[q][j][3]);
          else
            *reinterpret_cast<int2*>(g) = make_int2(v[q][j][0], v[q][j][1]);
        }
        g += lds4;
      }
    }
  };
  auto copy_row_chunk = [&](int k) {
    if (AL && full) {
      copy_row_chunk_al(k);
      return;
    }
    const int r0 = CH * k + 1;
    const bool steady = r0 + CH - 1 <= n && full && k > 0;
    const char* g = R0 + static_cast<int64_t>(r0) * static_cast<int64_t>(ldr4) + 4 * t;
    uint32_t o[K];  // byte offset in the ring of (row r0, word 32i+t)
#pragma unroll
    for (int i = 0; i < K; ++i)
      o[i] = static_cast<uint32_t>(((r0 - 2 + (32 * i + t) / K + RR) % RR) * RS4 + 4 * C::word_pos(32 * i + t));
    if (steady) {
#pragma unroll
      for (int j = 0; j < CH; ++j) {
#pragma unroll
        for (int i = 0; i < K; ++i) cpa4(refR + wrap(o[i] + j * RS4, RBYTES), g + 128 * i);  // (o[i]: word 32i+t's slot and position)
        g += ldr4;
      }
    } else {
#pragma unroll 1
      for (int j = 0; j < CH; ++j) {
        const int r = r0 + j;
#pragma unroll
        for (int i = 0; i < K; ++i)
          cpa4_p(r <= n && 32 * i + t < b.ws && !(r == 1 && 32 * i + t < K), refR + wrap(o[i] + j * RS4, RBYTES), g + 128 * i);
        g += ldr4;
      }
    }
  };

  auto store_row_chunk = [&](int k) {
    if (AL && full) {
      store_row_chunk_al(k);
      return;
    }
    const int r0 = CH * k + 1;
    char* g = S0 + static_cast<int64_t>(r0) * static_cast<int64_t>(lds4) + 4 * t;
    // word 32i + t of row r: slot r - 1 + (32i + t)/K, column 32i + t
    uint32_t o[K];
#pragma unroll
    for (int i = 0; i < K; ++i) o[i] = static_cast<uint32_t>(((r0 - 1 + (32 * i + t) / K) % SR) * RS4 + 4 * C::word_pos(32 * i + t));
    int v[CH][K];
#pragma unroll
    for (int j = 0; j < CH; ++j)
#pragma unroll
      for (int i = 0; i < K; ++i) v[j][i] = (NW_EXP & 64) ? j * i : lds32(scR + wrap(o[i] + j * RS4, SBYTES));
    release(k);
    if (r0 + CH - 1 <= n && full) {
#pragma unroll
      for (int j = 0; j < CH; ++j) {
#pragma unroll
        for (int i = 0; i < K; ++i) {
          if (NW_EXP & 32)
            asm volatile("" ::"r"(v[j][i]));
          else
            reinterpret_cast<int*>(g)[32 * i] = v[j][i];
        }
        g += lds4;
      }
    } else {
#pragma unroll
      for (int j = 0; j < CH; ++j) {
        if (r0 + j <= n) {
#pragma unroll
          for (int i = 0; i < K; ++i)
            if (32 * i + t < b.ws) reinterpret_cast<int*>(g)[32 * i] = v[j][i];
        }
        g += lds4;
      }
    }
  };

  // the first NSB blocks rewrite no stored slot: their ready phases get the store arrival now
  if (DO_ST && t == 0)
    for (int c = 0; c < C::NSB; ++c) bar_arrive(sm.ready(w, c));
  int kr = DO_REF ? 0 : nch, ks = DO_ST ? 0 : nch;  // next ref row chunk to copy, next score row chunk to store
  uint64_t tw = 0;
  unsigned idle = 0;
  for (;;) {
    bool did = false;
    // the store first: its slack is NSB - 3 blocks, the ref copies run NRB - 4 blocks ahead
    if (ks < nch && bar_test(sm.cdone(w, ks + 2), phase_of(ks + 2, C::NRDY))) {
      if (kTrace && t == 0 && P.trace3 != nullptr && b.pair * P.nbands + b.band < 2)
        P.trace3[(b.band * 4 + 0) * 8192 + (ks & 8191)] = globaltimer_ns();  // store start
      if (!(NW_EXP & 2))
        store_row_chunk(ks);  // (it releases the chunk's slots between its reads and its stores)
      else
        release(ks);
      if (kTrace && t == 0 && P.trace3 != nullptr && b.pair * P.nbands + b.band < 2)
        P.trace3[(b.band * 4 + 1) * 8192 + (ks & 8191)] = globaltimer_ns();  // store done
      ++ks;
      did = true;
    }
    // row chunk kr writes slots up to 16 kr + 45: slot chunk kr + 2 - NRB must have been read
    if (kr < nch && (kr + 2 - C::NRB < 0 || bar_test(sm.cdone(w, kr + 2 - C::NRB), phase_of(kr + 2 - C::NRB, C::NRDY)))) {
      if (kTrace && t == 0 && P.trace3 != nullptr && b.pair * P.nbands + b.band < 2)
        P.trace3[(b.band * 4 + 2) * 8192 + (kr & 8191)] = globaltimer_ns();  // copy issue
      if (!(NW_EXP & 1)) copy_row_chunk(kr);
      // slot chunk kr - 1 (rows up to 16 kr + 16) is complete once these copies land; after the
      // last row chunk every remaining slot chunk is
      if (kr >= 1) cpa_arrive_noinc(sm.ready(w, kr - 1));
      if (kr == nch - 1)
        for (int c = kr; c < nblk; ++c) cpa_arrive_noinc(sm.ready(w, c));
      if (kr + PF < nch) prefetch(kr + PF);
      ++kr;
      did = true;
    }
    if (kr >= nch && ks >= nch) break;
    if (did) {
      idle = 0;
    } else if (NW_STAGE_SLEEP > 0 && (++idle & 15u) == 0) {
      __nanosleep(NW_STAGE_SLEEP);
    } else if ((++idle & 255u) == 0) {
      const uint64_t now = globaltimer_ns();
      if (idle == 256) tw = now;
      else if (now - tw > P.spin_limit_ns) watchdog_trap(P.err);
    }
  }
  if (DO_REF) asm volatile("cp.async.wait_all;" ::: "memory");
}

// ---- the border-in warp: the group's left border column into band 0's shared in-ring ----------
// lin != null: 64-bit entries {value, tag} of the previous group's last band (or a strip halo),
// polled with relaxed sys-scope loads until the tags match; else the plain score column c0 - 1
// (input data).  Block q (rows 16q+1 .. 16q+16, lanes 0..15) is forwarded once band 0 has read
// block q - NBB of the ring (entfree).
template <class C>
__device__ __forceinline__ void border_in_warp(const StripParams& P, const BandTask& b, const BandSmem<C>& sm, const int t,
                                               const uint32_t gen, const uint64_t* lin, const uint32_t lin_tag, const bool lin_sys) {
  constexpr int CH = C::CH;
  constexpr unsigned FULL = 0xffffffffu;
  const int n = b.n;
  const int nch = (n + CH - 1) / CH;
  const int32_t* const colp = b.S + (b.c0 - 1);
  const long long lds = P.lds;
  const uint32_t ring = sm.link(0);
  for (int q = 0; q < nch; ++q) {
    if (q >= C::NBB) bar_wait(sm.entfree(0, q - C::NBB), phase_of(q - C::NBB, C::NBB), P, 64);
    const int row = CH * q + 1 + t;
    const bool act = t < CH && row <= n;
    int v;
    if (lin != nullptr) {
      auto poll = [&]() { return lin_sys ? ld_rlx_sys_p(act, lin + row) : ld_rlx_gpu_p(act, lin + row); };
      uint64_t e = poll();
      if (!__all_sync(FULL, !act || static_cast<uint32_t>(e >> 32) == lin_tag)) {
        const uint64_t tw = globaltimer_ns();
        unsigned spins = 0;
        do {
          e = poll();
          if ((++spins & 63u) == 0 && globaltimer_ns() - tw > P.spin_limit_ns) watchdog_trap(P.err);
        } while (!__all_sync(FULL, !act || static_cast<uint32_t>(e >> 32) == lin_tag));
      }
      v = static_cast<int>(static_cast<uint32_t>(e));
    } else {
      v = act ? __ldg(colp + static_cast<long long>(row) * lds) : 0;
    }
    st_ent_smem_p(act, ring + 8u * ring_slot<C>(row), pack_entry(v, gen | static_cast<uint32_t>(row)));
  }
}

// ---- the compute warp of band slot w ----------------------------------------------------------
// One code path for every band: the left border from the band's shared in-ring; the right border
// column (the band's last column, row by row) into the next band's in-ring (lk >= 0) or, for the
// group's last band, straight into the global entries the next group reads / a strip halo (lout:
// entry of row r at lout[r], tag lout_tag, sys scope when the halo lives on a peer GPU).
template <class C>
__device__ __forceinline__ void band_compute(const StripParams& P, const BandTask& T, const BandSmem<C>& sm, const int w, const int t,
                                             const uint32_t gen, const int lk, uint64_t* const lout, const uint32_t lout_tag,
                                             const bool lout_sys) {
  constexpr int K = C::K, CH = C::CH;
  constexpr unsigned FULL = 0xffffffffu;
  const int n = T.n, p = T.p, c0 = T.c0, ws = T.ws;
  const int negp = -p, one = 1;
  int cm[K];
#pragma unroll
  for (int m = 0; m < K; ++m) cm[m] = static_cast<int>(opaque(static_cast<uint32_t>(-(m + 1) * p)));  // one VIADDMNMX each
  const uint32_t laneR = sm.refR(w) + C::lane_off(t), laneS = sm.scR(w) + C::lane_off(t);
  const uint32_t lin_ring = sm.link(w), lout_ring = lk >= 0 ? sm.link(lk) : 0u;
  const bool to_smem = lk >= 0, to_global = lout != nullptr;
  // the band's last column: lane out_lane, element out_m (full band: lane 31, K-1)
  const int out_lane = (ws - 1) / K, out_m = (ws - 1) - out_lane * K;
  const bool is_out = t == out_lane;

  // ---- prologue: the top border row (row 0), the corner for lane 0, step 0's ref for lane 0
  int up[K];
#pragma unroll
  for (int m = 0; m < K; ++m) up[m] = (t * K + m < ws) ? __ldg(T.S + c0 + t * K + m) : 0;
  int dg = (t * K < ws) ? __ldg(T.S + c0 + t * K - 1) : 0;
  int vlast = up[K - 1];
  int rvn[K];
#pragma unroll
  for (int m = 0; m < K; ++m) rvn[m] = (t == 0 && m < ws) ? __ldg(T.R + P.ldr + c0 + m) : 0;

  const int nsteps = n + 31;
  const int nblk = (nsteps + CH - 1) / CH;
  const int nch = (n + CH - 1) / CH;
  int curv = 0;  // lane j < 16: border value of row 16Q + 1 + j
  int gov[CH];    // global sink: the last steady block's out-lane values, published after the next arrive
  int gpend = INT32_MIN;  // (their first row; INT32_MIN: none pending)

  // The cell update of one step (lane t, row s + 1 - t) from the ref of this row (rv) and the
  // left value L; writes S[].
  auto cells = [&](const int* rv, const int L, int* S) {
    int Y[K];
#pragma unroll
    for (int m = 0; m < K; ++m) {
      const int d = imad1(m == 0 ? dg : up[m - 1], one, rv[m]);
      const int x = __viaddmax_s32(up[m], negp, d);
      Y[m] = m == 0 ? x : __viaddmax_s32(Y[m - 1], negp, x);
    }
#pragma unroll
    for (int m = 0; m < K; ++m) S[m] = __viaddmax_s32(L, cm[m], Y[m]);
  };
  // One block of 16 steps (ring slots 16Q .. 16Q+15 never wrap inside a block: one base per block
  // plus immediates).  EDGE (the first two blocks, the last blocks, a ragged band): lanes whose row
  // is not in 1..n yet keep their state (top border row); rows past n are computed but never
  // stored.  Lane 31's 16 right-border values are kept in registers and published after the block
  // (a full band's out lane is lane 31; a ragged band is always the last of its pair and publishes
  // nothing).
  auto block = [&](const int s0, const uint32_t aR, const uint32_t aS, auto edge_tag) {
    constexpr bool EDGE = decltype(edge_tag)::value;
    int ov[CH];
    [&]<int... J>(std::integer_sequence<int, J...>) {
      (
          [&] {
            constexpr int j = J;
            int rv[K];
#pragma unroll
            for (int m = 0; m < K; ++m) rv[m] = rvn[m];
            lds_ref<K, 4 * C::HALF>(aR + j * C::RS4, rvn);  // this lane's next row (s + 2 - t)
            const int bval = __shfl_sync(FULL, curv, j);
            const int fl = __shfl_up_sync(FULL, vlast, 1);
            const int L = t == 0 ? bval : fl;
            int S[K];
            cells(rv, L, S);
            sts_score<K, 4 * C::HALF>(aS + j * C::RS4, S);  // row s + 1 - t (rows outside 1..n are never stored)
            if constexpr (EDGE) {
              const bool act = s0 + j + 1 - t >= 1;
#pragma unroll
              for (int m = 0; m < K; ++m) up[m] = act ? S[m] : up[m];
              dg = act ? L : dg;
            } else {
#pragma unroll
              for (int m = 0; m < K; ++m) up[m] = S[m];
              dg = L;
            }
            vlast = up[K - 1];
            ov[j] = S[K - 1];
          }(),
          ...);
    }(std::make_integer_sequence<int, CH>{});
    // lane 31 computed rows s0 - 30 .. s0 - 15 (s0 - 30 even: 16-byte aligned entry pairs)
    const int r0 = s0 - 30;
    auto pair_ok = [&](int k) { return t == 31 && (!EDGE || (r0 + 2 * k >= 1 && r0 + 2 * k + 1 <= n)); };
    if (to_smem) {
      // ring slots (s0 - 32) mod BR + 0..15, contiguous
      const uint32_t a0 = lout_ring + 8u * ring_slot<C>(r0);
      const uint32_t tg0 = gen | static_cast<uint32_t>(r0);  // (gen | r) == gen + r: 0 <= r < 2^30
      [&]<int... Kp>(std::integer_sequence<int, Kp...>) {
        (st_pair_smem_p<16 * Kp>(pair_ok(Kp), a0, pack_entry(ov[2 * Kp], tg0 + 2 * Kp), pack_entry(ov[2 * Kp + 1], tg0 + 2 * Kp + 1)), ...);
      }(std::make_integer_sequence<int, CH / 2>{});
      if constexpr (EDGE) {
        // (a pair straddling row 0 or row n: its one valid entry alone)
#pragma unroll
        for (int k = 0; k < CH / 2; ++k) {
          const int ra = r0 + 2 * k;
          if (ra == 0 && 1 <= n) st_ent_smem_p(t == 31, lout_ring + 8u * ring_slot<C>(1), pack_entry(ov[2 * k + 1], gen | 1u));
          if (ra == n && n >= 1) st_ent_smem_p(t == 31, lout_ring + 8u * ring_slot<C>(n), pack_entry(ov[2 * k], gen | static_cast<uint32_t>(n)));
        }
      }
    } else if (to_global) {
      // published after the next event's cdone arrive: a release arrive behind fresh global
      // stores would wait for their L2 acknowledgements
#pragma unroll
      for (int j = 0; j < CH; ++j) gov[j] = ov[j];
      gpend = r0;
    }
  };
  auto publish_global = [&]() {
    if (gpend == INT32_MIN) return;
    uint64_t* const g0 = lout + gpend;
    const int r0 = gpend;
    auto pair_ok = [&](int k) { return t == 31 && r0 + 2 * k >= 1 && r0 + 2 * k + 1 <= n; };
    if (lout_sys) {
      [&]<int... Kp>(std::integer_sequence<int, Kp...>) {
        (st_pair_global_p<16 * Kp, true>(pair_ok(Kp), g0, pack_entry(gov[2 * Kp], lout_tag), pack_entry(gov[2 * Kp + 1], lout_tag)), ...);
      }(std::make_integer_sequence<int, CH / 2>{});
    } else {
      [&]<int... Kp>(std::integer_sequence<int, Kp...>) {
        (st_pair_global_p<16 * Kp, false>(pair_ok(Kp), g0, pack_entry(gov[2 * Kp], lout_tag), pack_entry(gov[2 * Kp + 1], lout_tag)), ...);
      }(std::make_integer_sequence<int, CH / 2>{});
    }
#pragma unroll
    for (int k = 0; k < CH / 2; ++k) {  // (a pair straddling row 0 or row n: its one valid entry)
      const int ra = r0 + 2 * k;
      if (ra == 0 && 1 <= n) {
        if (lout_sys)
          st_ent_sys_p(t == 31, lout + 1, pack_entry(gov[2 * k + 1], lout_tag));
        else
          st_ent_gpu_p(t == 31, lout + 1, pack_entry(gov[2 * k + 1], lout_tag));
      }
      if (ra == n && n >= 1) {
        if (lout_sys)
          st_ent_sys_p(t == 31, lout + n, pack_entry(gov[2 * k], lout_tag));
        else
          st_ent_gpu_p(t == 31, lout + n, pack_entry(gov[2 * k], lout_tag));
      }
    }
    gpend = INT32_MIN;
  };

  // (-DNW_TRACE=1 builds only) cycles per phase: [0] ready waits, [1] out-ring waits, [2] border
  // block, [3] whole events, [4] steady 16-step blocks
  long long tr[5] = {0, 0, 0, 0, 0};
  const unsigned long long tr_start = kTrace ? globaltimer_ns() : 0ull;
  unsigned long long tr_first = tr_start;
  auto clk = [&]() -> long long { return kTrace ? clock64() : 0ll; };
  for (int Q = 0; Q < nblk; ++Q) {
    const int s0 = CH * Q;
    const long long te0 = clk();
    // ---- event Q: slot chunk Q-1 read, row chunk Q-3 complete (lane 31 finished row 16Q-31)
    __syncwarp();
    bar_arrive_p(t == 0 && Q >= 1, sm.cdone(w, Q - 1));
    publish_global();
    long long tc = te0;
    // the block's ref slots landed and its score slots free (ready), and border block Q (rows
    // 16Q+1 .. 16Q+16, lane j): both requests issued back to back, then checked
    const bool has_border = s0 + 1 <= n;
    const int row = s0 + 1 + t;
    const uint32_t ba = lin_ring + 8u * ring_slot<C>(row);
    const uint32_t want = gen | static_cast<uint32_t>(row);
    uint64_t e = 0ull;
    const bool rdy = (NW_EXP & 4) || bar_test(sm.ready(w, Q), phase_of(Q, C::NRDY));
    if (has_border && t < CH) e = ld_rlx_cta_smem(ba);
    if (!rdy) bar_spin(sm.ready(w, Q), phase_of(Q, C::NRDY), P, 0);
    if (kTrace && t == 0 && P.trace3 != nullptr && T.pair * P.nbands + T.band < 2)
      P.trace3[(T.band * 4 + 3) * 8192 + (Q & 8191)] = globaltimer_ns();  // ready observed
    if (kTrace) { const long long c = clk(); tr[0] += c - tc; tc = c; }
    // every BP events: the next BP blocks' out-ring writes (rows <= 16(Q+BP)-15, border block
    // Q+BP-2 at most) find their slots read
    if (to_smem) {
      const int bb = Q + C::BP - 2 - C::NBB;
      if (!(NW_EXP & 8) && Q % C::BP == 0 && bb >= 0) bar_wait(sm.entfree(lk, bb), phase_of(bb, C::NBB), P);
    }
    if (kTrace) { const long long c = clk(); tr[1] += c - tc; tc = c; }
    if (has_border) {
      auto ok = [&](uint64_t v) { return t >= CH || row > n || static_cast<uint32_t>(v >> 32) == want; };
      if (!(NW_EXP & 8) && !__all_sync(FULL, ok(e))) {
        const uint64_t tw = globaltimer_ns();
        unsigned spins = 0;
        do {
          e = (t < CH) ? ld_rlx_cta_smem(ba) : 0ull;
          if ((++spins & 255u) == 0 && globaltimer_ns() - tw > P.spin_limit_ns) watchdog_trap(P.err);
        } while (!__all_sync(FULL, ok(e)));
      }
      curv = static_cast<int>(static_cast<uint32_t>(e));
      __syncwarp();
      bar_arrive_p(t == 0, sm.entfree(w, Q));  // block Q read (its values are in registers)
      if (kTrace && Q == 0) tr_first = globaltimer_ns();
    }
    if (kTrace) { const long long c = clk(); tr[2] += c - tc; tr[3] += c - te0; tc = c; }
    // ---- 16 steps (ring slots 16Q .. 16Q+15: no wrap inside a block)
    const uint32_t aR = laneR + static_cast<uint32_t>(s0 % C::RR) * C::RS4;
    const uint32_t aS = laneS + static_cast<uint32_t>(s0 % C::SR) * C::RS4;
    if (Q >= 2 && s0 + CH <= n && ws == C::W) {
      block(s0, aR, aS, std::false_type{});
      if (kTrace) tr[4] += clk() - tc;
    } else {
      block(s0, aR, aS, std::true_type{});
    }
  }
  // every slot chunk read and every row chunk complete: release what the events did not
  __syncwarp();
  if (t == 0)
    for (int c = nblk - 1; c <= max(nblk - 1, nch + 1); ++c) bar_arrive(sm.cdone(w, c));
  publish_global();
  if (kTrace && t == 0 && P.trace != nullptr) {
    const long long task = T.pair * P.nbands + T.band;
    if (task < P.trace_cap) {
      unsigned smid;
      asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
      unsigned long long* e = P.trace + 8 * task;
      e[0] = static_cast<unsigned long long>(task);
      e[1] = tr_start;
      e[2] = globaltimer_ns();
      e[3] = smid;
      for (int k = 0; k < 4; ++k) e[4 + k] = static_cast<unsigned long long>(tr[k]);
      P.trace2[8 * task] = static_cast<unsigned long long>(tr[4]);
      P.trace2[8 * task + 1] = tr_first;
    }
  }
}

// ---- the kernel -------------------------------------------------------------------------------
template <class C, bool AL>
__global__ void __launch_bounds__(32 * C::NWARPS, 1) nw_band_kernel(const __grid_constant__ StripParams P) {
  extern __shared__ __align__(128) unsigned char smem[];
  const int t = threadIdx.x & 31, wa = threadIdx.x >> 5;
  BandSmem<C> sm;
  sm.base = opaque(smem_u32(smem));  // kept in a register (else ptxas re-derives the shared window per use)
  unsigned long long* const s_group = reinterpret_cast<unsigned long long*>(smem);
  // border in-rings start invalid: shared memory keeps an earlier launch's entries, whose tags
  // (gen | row) this launch reuses (tag 0xFFFFFFFF never equals gen | row, row < 2^30)
  for (int w = 0; w < C::NC; ++w)
    for (int i = threadIdx.x; i < C::BR; i += blockDim.x)
      reinterpret_cast<unsigned long long*>(smem + (sm.link(w) - sm.base))[i] = ~0ull;
  uint32_t gcount = 0;
  for (;;) {
    if (threadIdx.x == 0) *s_group = atomicAdd(P.ticket, 1ull);
    __syncthreads();
    const long long tk = static_cast<long long>(*s_group - P.ticket_base);
    if (tk < 0 || tk >= P.ngroups) break;
    // pair mode: a ticket is a whole pair, its groups swept one after the other
    const int nsub = P.pair_mode ? P.gpp : 1;
    for (int sub = 0; sub < nsub; ++sub) {
      const long long grp = P.pair_mode ? tk * P.gpp + sub : tk;
      const long long pair = grp / P.gpp;
      const int g = static_cast<int>(grp - pair * P.gpp);
      // mbarriers: fresh for every group (the previous group's arrivals have all been consumed)
      if (threadIdx.x == 0) {
        if (gcount > 0)
          for (int i = 0; i < C::NBAR; ++i) bar_inval(sm.bar(i));
        for (int w = 0; w < C::NC; ++w) {
          for (int k = 0; k < C::NRDY; ++k) {
            bar_init(sm.cdone(w, k), 1);
            bar_init(sm.ready(w, k), 33);  // 32 noinc ref arrivals + the store arrival
          }
          for (int k = 0; k < C::NBB; ++k) bar_init(sm.entfree(w, k), 1);
        }
      }
      __syncthreads();
      const int band0 = g * C::NC;
      const int nb = min(C::NC, P.nbands - band0);  // bands of this group
      const uint32_t gen = (gcount & 3u) << 30;
      const bool is_stage = C::SPLIT ? (wa == 1 || wa == 2) : (wa >= C::NC && wa < 2 * C::NC);
      const int w = wa < C::NC ? wa : (is_stage && !C::SPLIT ? wa - C::NC : 0);
      BandTask T;
      T.n = static_cast<int>(P.n);
      T.p = P.p;
      T.band = band0 + w;
      T.g = g;
      T.pair = pair;
      T.c0 = band_c0(T.band, C::W);
      T.ws = T.band < P.nbands ? band_ws(P.width, T.band, C::W) : 0;
      T.last_band = T.band == P.nbands - 1;
      T.S = P.score + pair * P.pss;
      T.R = P.ref + pair * P.psr;
      if ((NW_EXP & 16) && wa >= C::NC) {
        // (timing experiment: no helper warps)
      } else if (wa == C::W_BORDER) {
        // border-in warp: band 0 of the group's left border (plain column, strip halo or the
        // previous group's entries)
        const uint64_t* lin = nullptr;
        uint32_t lin_tag = 0;
        if (band0 == 0) {
          lin = P.halo_in;
          lin_tag = P.halo_epoch;
        } else {
          lin = P.xbuf + (pair * (P.gpp - 1) + (g - 1)) * band_xstride(P.n);  // entry of row r at lin[r]
          lin_tag = P.epoch;
        }
        border_in_warp<C>(P, T, sm, t, gen, lin, lin_tag, band0 == 0);  // (a strip halo may live on a peer GPU)
      } else if (w < nb && (wa < C::NC || is_stage)) {
        if (is_stage) {
          if (!C::SPLIT)
            band_stage_warp<C, AL, kStageRef | kStageStore>(P, T, sm, w, t);
          else if (wa == 1)
            band_stage_warp<C, AL, kStageRef>(P, T, sm, w, t);
          else
            band_stage_warp<C, AL, kStageStore>(P, T, sm, w, t);
        } else if (w + 1 < nb) {
          band_compute<C>(P, T, sm, w, t, gen, w + 1, nullptr, 0, false);
        } else if (T.last_band) {  // the pair's last band: a strip halo or nothing
          band_compute<C>(P, T, sm, w, t, gen, -1, P.halo_out, P.halo_epoch, P.halo_out != nullptr && P.halo_out_sys != 0);
        } else {  // the group's last band: the next group's global entries
          band_compute<C>(P, T, sm, w, t, gen, -1, P.xbuf + (pair * (P.gpp - 1) + g) * band_xstride(P.n), P.epoch, false);
        }
      }
      __syncthreads();  // group end: rings, links and mbarriers reusable
      ++gcount;
    }
  }
}

}  // namespace nwb200
