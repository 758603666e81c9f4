// nw_wave.cuh — the persistent NW wavefront kernel, v5: self-staging warps.
//
// What it computes (Fig. 2, with Rodinia's cell function, R1):
//     score[i][j] = max(score[i-1][j-1] + ref[i][j], score[i-1][j] - p, score[i][j-1] - p)
// for every interior cell, each value written ONCE, in place, into score (the short-circuited
// update of P:512-516 / P:616-656: no temporary, no copy).
//
// Structure (same schedule as nw_strip.cuh, pinned by P7 through band_c0 / band_ws / lane_row):
//   * A band = W = 32*K adjacent columns, all rows, swept by ONE warp; lane t owns K adjacent
//     columns and at step s computes row s+1-t (the intra-tile anti-diagonals of P:498-501,
//     skewed one row per lane).  The left value arrives from lane t-1 by SHFL.UP; each cell is
//     two DPX VIADDMNMX (max-plus prefix form).
//   * A CTA of NW warps claims NW consecutive bands through one atomic ticket (wavefront order;
//     band k waits only on band k-1, so no deadlock without co-residency).
//   * The warp stages its own memory traffic, one row per step, interleaved with the sweep so it
//     fills the issue slots the latency-bound recurrence leaves idle (measured: SHFL 24 cycles,
//     DPX 4.75, LDS 29; scripts/ubench*.cu):
//       - ref row s+LOOK: 16-byte cp.async (LDGSTS) of the row's 16-byte aligned superset into a
//         64-row shared ring; row s+LOOK+PFD is prefetched into L2;
//       - score row s-SD: LDS.128 + STG.128 of the 16-byte aligned interior (+ scalar head/tail
//         words: the Rodinia pitch n+1 puts every row at a different 16-byte phase) from a
//         64-row shared ring the lanes fill with STS.
//     Element x of row r sits at ring((r-1) & 63) + (G(r) & 31) + x, G(r) = the global word
//     address of (r, c0): shared and global 16-byte phases agree, and for an odd pitch the 32
//     skewed rows a warp touches fall in 32 different banks.
//   * Events every CH = 8 steps: cp.async commit / wait (ref rows of the next blocks landed),
//     border-block check, back-pressure, __syncwarp (makes the ring writes of other lanes
//     visible).  There is no other synchronisation inside a band: no staging warp, no mbarrier.
//   * Band handoff (the paper's Fig. 9 ordering W ∩ R = ∅): the lane holding the band's last
//     column publishes every row as a 64-bit entry {value, tag} (flag fused with the value):
//       - to warp w+1 of the CTA: a 256-entry shared ring (tag = gen << 30 | row), back-pressure
//         on the consumer's published progress;
//       - to another CTA / GPU: a full-length global buffer (tag = launch epoch), relaxed
//         gpu / sys scope stores.
//     The consumer holds one 8-row block of entries per event (lanes 0..7) and loads the next
//     blocks ahead (1 block for a shared source, 2 for a global one); a stale block is re-polled
//     synchronously under a %globaltimer watchdog (kErrWatchdog + trap on expiry).
#pragma once
#include <cstdint>

#include "nw_ptx.cuh"
#include "nw_strip.cuh"

namespace nwb200 {

template <int K_, bool SEQ_, int NW_>
struct WaveCfg {
  static constexpr int K = K_, NW = NW_;
  static constexpr bool SEQ = SEQ_;
  static constexpr int W = 32 * K;
  static constexpr int CH = 8;        // event period (steps) = staging chunk = border block (rows)
  static constexpr int RS = W + 36;   // ring row slot (words): W + 3 head + 3 tail + 28 swizzle
  static constexpr int LA = 4;        // ref chunk c is issued during block c - LA
  static constexpr int SDB = 5;       // score chunk c (complete after step CH*c+CH+30) stored in block c + SDB
  static constexpr int RR = CH * (LA + 5);  // ref ring rows: chunk c lives from block c-LA to c+4
  static constexpr int SR = CH * (SDB + 1); // score ring rows: chunk c lives from block c to c+SDB
  static constexpr int PFB = 8;       // L2 prefetch distance (chunks) beyond the cp.async lookahead
  static constexpr int BR = 256;      // shared border ring entries
  static constexpr int PR = W / 4 + 1;            // 16-byte pieces of a ref row superset (max)
  static constexpr int PS = W / 4;                // 16-byte pieces of a score row interior (max)
  static constexpr int ITR = SEQ ? 0 : (CH * PR + 31) / 32;
  static constexpr int ITS = (CH * PS + 31) / 32;
  static constexpr int REF_WORDS = SEQ ? 0 : RR * RS;
  static constexpr int PROF_WORDS = SEQ ? 32 * 32 : 0;
  static constexpr int BPRE_BYTES = 4 * 8 * (CH + 2);  // border prefetch ring: 4 blocks x (CH+2) entries
  static constexpr size_t kWarpSmem = 4ull * (REF_WORDS + SR * RS + PROF_WORDS) + BPRE_BYTES;
  static constexpr size_t kCtaHdr = 128 + static_cast<size_t>(NW - 1) * BR * 8;
  static constexpr size_t kSmem = kCtaHdr + NW * kWarpSmem;
  static constexpr int NLINES = (4 * W + 12 + 127) / 128 + 1;  // 128-byte lines of one ref row segment
  static_assert(RS % 4 == 0 && kWarpSmem % 16 == 0 && kCtaHdr % 16 == 0, "16-byte aligned rings");
  static_assert((RS * CH) % 32 == 0, "chunk moves keep banks");
  static_assert(ITS <= CH, "score pieces spread over the block's steps");
  static_assert(NW <= 8, "header space");
};

// cp.async 16 bytes with a source size (bytes beyond src_bytes are zero-filled, never read)
__device__ __forceinline__ void cp_async16_n(bool p, uint32_t dst, const void* src, int src_bytes) {
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %0, 0; @q cp.async.cg.shared.global [%1], [%2], 16, %3; }" ::"r"(
                   static_cast<int>(p)),
               "r"(dst), "l"(src), "r"(src_bytes)
               : "memory");
}
// predicated shared -> global copies through registers (one predicate, no register moves)
__device__ __forceinline__ void copy_s2g16_p(bool p, void* g, uint32_t a) {
  asm volatile("{ .reg .pred q; .reg .b32 x, y, z, w; setp.ne.b32 q, %0, 0;\n\t"
               "@q ld.shared.v4.b32 {x, y, z, w}, [%2];\n\t"
               "@q st.global.v4.b32 [%1], {x, y, z, w}; }" ::"r"(static_cast<int>(p)),
               "l"(g), "r"(a)
               : "memory");
}
__device__ __forceinline__ void copy_s2g4_p(bool p, void* g, uint32_t a) {
  asm volatile("{ .reg .pred q; .reg .b32 x; setp.ne.b32 q, %0, 0;\n\t"
               "@q ld.shared.b32 x, [%2];\n\t"
               "@q st.global.b32 [%1], x; }" ::"r"(static_cast<int>(p)),
               "l"(g), "r"(a)
               : "memory");
}
__device__ __forceinline__ void cp_async16_pp(bool p, uint32_t dst, const void* src) {
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %0, 0; @q cp.async.cg.shared.global [%1], [%2], 16; }" ::"r"(static_cast<int>(p)),
               "r"(dst), "l"(src)
               : "memory");
}
__device__ __forceinline__ int4 lds128_np(bool p, uint32_t a) {
  int4 v;
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %4, 0; @q ld.shared.v4.b32 {%0, %1, %2, %3}, [%5]; }"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
               : "r"(static_cast<int>(p)), "r"(a)
               : "memory");
  return v;
}
__device__ __forceinline__ void stg128_np(bool p, void* ptr, int4 v) {
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %0, 0; @q st.global.v4.b32 [%1], {%2, %3, %4, %5}; }" ::"r"(static_cast<int>(p)),
               "l"(ptr), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
               : "memory");
}
__device__ __forceinline__ int lds32_np(bool p, uint32_t a) {
  int v;
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %1, 0; @q ld.shared.b32 %0, [%2]; }" : "=r"(v) : "r"(static_cast<int>(p)), "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ void stg32_np(bool p, void* ptr, int v) {
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %0, 0; @q st.global.b32 [%1], %2; }" ::"r"(static_cast<int>(p)), "l"(ptr), "r"(v)
               : "memory");
}
// shared-ring store of a computed score (ordered by the events' __syncwarp, not by the compiler)
__device__ __forceinline__ void sts32_ring(uint32_t a, int v) {
  asm volatile("st.shared.b32 [%0], %1;" ::"r"(a), "r"(v));
}
__device__ __forceinline__ void st_entry_gpu_p(bool pred, uint64_t* p, uint32_t lo, uint32_t hi) {
  asm volatile("{ .reg .pred q; .reg .b64 e; setp.ne.b32 q, %0, 0; mov.b64 e, {%2, %3}; @q st.relaxed.gpu.global.b64 [%1], e; }" ::"r"(
                   static_cast<int>(pred)),
               "l"(p), "r"(lo), "r"(hi)
               : "memory");
}
__device__ __forceinline__ void st_entry_sys_p(bool pred, uint64_t* p, uint32_t lo, uint32_t hi) {
  asm volatile("{ .reg .pred q; .reg .b64 e; setp.ne.b32 q, %0, 0; mov.b64 e, {%2, %3}; @q st.relaxed.sys.global.b64 [%1], e; }" ::"r"(
                   static_cast<int>(pred)),
               "l"(p), "r"(lo), "r"(hi)
               : "memory");
}
__device__ __forceinline__ void st_entry_smem_p(bool pred, uint32_t a, uint32_t lo, uint32_t hi) {
  asm volatile("{ .reg .pred q; .reg .b64 e; setp.ne.b32 q, %0, 0; mov.b64 e, {%2, %3}; @q st.volatile.shared.b64 [%1], e; }" ::"r"(
                   static_cast<int>(pred)),
               "r"(a), "r"(lo), "r"(hi)
               : "memory");
}

// One band (task) swept by one warp.
template <class C>
__device__ __forceinline__ void wave_band(const StripParams& P, const long long task, const int w, const int t,
                                          unsigned char* const smem, unsigned char* const wsm, const uint32_t gen,
                                          const int sink) {
  constexpr int K = C::K, RS = C::RS, CH = C::CH, RR = C::RR, SR = C::SR;
  constexpr bool SEQ = C::SEQ;
  constexpr unsigned FULL = 0xffffffffu;
  const bool tracing = P.trace != nullptr;
  const unsigned long long t_task0 = tracing ? globaltimer_ns() : 0ull;
  long long spin_cyc = 0, ev_cyc = 0, bp_cyc = 0, wait_cyc = 0;

  const int n = static_cast<int>(P.n);
  const int p = P.p;
  const long long pair = task / P.nbands;
  const int band = static_cast<int>(task - pair * P.nbands);
  const bool last_band = band == P.nbands - 1;
  const int c0 = band_c0(band, C::W);
  const int ws = band_ws(P.width, band, C::W);
  int32_t* const S = P.score + pair * P.pss;
  const int32_t* const R = SEQ ? nullptr : P.ref + pair * P.psr;
  const int nchunks = (n + CH - 1) / CH;
  constexpr int kNever = 1 << 30;  // row index of a staging piece that does not exist (never < rlim)

  // ---- shared layout of this warp
  const uint32_t refR = opaque(smem_u32(wsm));
  const uint32_t scR = opaque(smem_u32(wsm) + 4u * C::REF_WORDS);
  uint32_t* const prof = reinterpret_cast<uint32_t*>(wsm + 4 * (C::REF_WORDS + SR * RS));
  const uint32_t bpre = smem_u32(wsm) + 4u * (C::REF_WORDS + SR * RS + C::PROF_WORDS);  // 4 x (CH+2) entries
  const uint32_t s_prog = smem_u32(smem + 8);     // [4w]: rows consumed by warp w (smem source)
  const uint32_t s_bring = smem_u32(smem + 128);  // [(w) * BR * 8]: ring warp w -> w+1

  // ---- border source (left), uniform per task
  int src;
  const uint64_t* lin = nullptr;
  uint32_t lin_epoch = 0;
  bool lin_sys = false;
  if (band == 0) {
    src = P.halo_in ? kSrcGlobal : kSrcPlain;
    lin = P.halo_in;
    lin_sys = true;
    lin_epoch = P.halo_epoch;
  } else if (w > 0) {
    src = kSrcSmem;
  } else {
    src = kSrcGlobal;
    lin = P.xbuf + (pair * (P.nbands - 1) + band - 1) * xstride(n);
    lin_epoch = P.epoch;
  }
  const uint32_t bring_in = s_bring + (w - 1) * C::BR * 8;
  const uint32_t bring_out = s_bring + w * C::BR * 8;
  const uint32_t prog_in = s_prog + 4 * w;        // written by this warp (consumer of w-1)
  const uint32_t prog_out = s_prog + 4 * (w + 1); // read by this warp (producer for w+1)
  const int32_t* const colp = S + (c0 - 1);       // plain left border column
  // ---- sink (right)
  uint64_t* lout = nullptr;
  uint32_t lout_tag = 0;
  const bool sink_smem = sink == kSinkSmem;
  bool sink_gpu = false, sink_sys = false;
  if (sink == kSinkGlobal) {
    if (last_band) {
      lout = P.halo_out;
      lout_tag = P.halo_epoch;
      sink_sys = P.halo_out_sys != 0;
      sink_gpu = !sink_sys;
    } else {
      lout = P.xbuf + (pair * (P.nbands - 1) + band) * xstride(n);
      lout_tag = P.epoch;
      sink_gpu = true;
    }
  }
  const int out_lane = (ws - 1) / K;
  const bool do_out = t == out_lane && sink != kSinkNone;

  // ---- global word addresses of (0, c0) and the end of ref
  const uintptr_t GR0 = SEQ ? 0 : (reinterpret_cast<uintptr_t>(R) >> 2) + c0;
  const uintptr_t GS0 = (reinterpret_cast<uintptr_t>(S) >> 2) + c0;
  const uintptr_t rend = SEQ ? 0 : reinterpret_cast<uintptr_t>(R + static_cast<long long>(n) * P.ldr + P.width + 1);
  const long long ldr = P.ldr, lds = P.lds;

  // ---- border blocks: lane j < CH of block q holds the entry of row CH*q + 1 + j
  auto load_block = [&](int q) -> uint64_t {
    const int row = CH * q + 1 + t;
    if (t >= CH || row > n) return 0ull;
    if (src == kSrcGlobal) return lin_sys ? ld_relaxed_sys(lin + row) : ld_relaxed_gpu(lin + row);
    if (src == kSrcSmem) return lds64_volatile(bring_in + 8u * (row & (C::BR - 1)));
    return static_cast<uint32_t>(__ldg(colp + static_cast<long long>(row) * lds));
  };
  // Global / plain sources: block q's entries are copied by cp.async three blocks ahead (they join
  // the ref pieces' commit group of that block, so the event's wait covers them) into slot q & 3
  // of a shared ring: no register holds an in-flight load across an event (a register move
  // of one would stall the warp for the whole load latency).  Slot of block q: entries of rows
  // CH*q .. CH*q+CH+1 (global: 16-byte pairs (2k, 2k+1) through L2 only, never via L1 since the
  // entries are polled; plain: the 4-byte values of score column c0-1).
  auto prefetch_block = [&](int q) {
    const uint32_t slot = bpre + 8u * (CH + 2) * static_cast<uint32_t>(q & 3);
    if (src == kSrcGlobal) {
      const int row = CH * q + 2 * t;
      cp_async16_cg_p(t <= CH / 2 && row <= n, slot + 16u * t, lin + row);
    } else if (src == kSrcPlain) {
      const int row = CH * q + 1 + t;
      cp_async4_p(t < CH && row <= n, slot + 8u * (1 + t), colp + static_cast<long long>(row) * lds);
    }
  };
  auto read_block = [&](int q) -> uint64_t {
    const uint32_t slot = bpre + 8u * (CH + 2) * static_cast<uint32_t>(q & 3);
    return t < CH ? lds64_volatile(slot + 8u * (1 + t)) : 0ull;
  };
  auto block_ok = [&](uint64_t e, int q) -> bool {
    const int row = CH * q + 1 + t;
    bool ok = true;
    if (t < CH && row <= n) {
      const uint32_t hi = static_cast<uint32_t>(e >> 32);
      if (src == kSrcGlobal) ok = hi == lin_epoch;
      else if (src == kSrcSmem) ok = hi == (gen | static_cast<uint32_t>(row));
    }
    return __all_sync(FULL, ok) != 0;
  };

  // ---- staging geometry.  Chunk c = rows CH*c+1 .. CH*c+CH.  In iteration it lane t moves the
  // 16-byte piece k of row i of a chunk (f = t + 32*it, i = f / pieces, k = f % pieces).  Chunk c
  // is chunk 0 moved by c*CH rows: global addresses by c*CH*ld words, ring rows by c*CH, the
  // swizzle G & 31 by c*CH*ld mod 32; CH is a multiple of 4, so the 16-byte phase of row i is the
  // same in every chunk and every per-lane offset below is computed once per task.
  uintptr_t rsrc[C::ITR > 0 ? C::ITR : 1];  // chunk-0 source byte address (16-byte aligned)
  uint32_t rdst[C::ITR > 0 ? C::ITR : 1];   // ring byte offset within a chunk: i*RS*4 + 16k
  int rg[C::ITR > 0 ? C::ITR : 1];          // G(row i of chunk 0) & 31
  int rrow[C::ITR > 0 ? C::ITR : 1];        // i, or kNever when piece k does not exist
  uint32_t rclip = 0;      // bit it: the piece crosses the end of ref in the last chunk (last band)
  const uintptr_t rstride = 4u * static_cast<uintptr_t>(CH * ldr), sstride = 4u * static_cast<uintptr_t>(CH * lds);
  if constexpr (!SEQ) {
#pragma unroll
    for (int it = 0; it < C::ITR; ++it) {
      const int f = t + 32 * it;
      const int i = f / C::PR, k = f - (f / C::PR) * C::PR;
      const uintptr_t G = GR0 + static_cast<uintptr_t>((1 + i) * ldr);
      const int a = static_cast<int>(G & 3);
      rsrc[it] = 4u * (G - a) + 16u * k;
      rdst[it] = 4u * (i * RS) + 16u * k;
      rg[it] = static_cast<int>(G & 31);
      rrow[it] = (i < CH && 4 * k < a + ws) ? i : kNever;
      const uintptr_t last_ga = rsrc[it] + static_cast<uintptr_t>(nchunks - 1) * rstride;
      if (last_band && rrow[it] < n - (nchunks - 1) * CH && last_ga + 16u > rend) rclip |= 1u << it;
    }
  }
  uintptr_t sdst[C::ITS];  // chunk-0 destination byte address of interior piece k of row i
  uint32_t ssrc[C::ITS];   // ring byte offset within a chunk (without the swizzle)
  int sg[C::ITS];          // G_S(row i of chunk 0) & 31
  int srow[C::ITS];        // i, or kNever when the piece does not exist
#pragma unroll
  for (int it = 0; it < C::ITS; ++it) {
    const int f = t + 32 * it;
    const int i = f / C::PS, k = f - (f / C::PS) * C::PS;
    const uintptr_t G = GS0 + static_cast<uintptr_t>((1 + i) * lds);
    const int a = static_cast<int>(G & 3);
    int h = (4 - a) & 3;
    h = h < ws ? h : ws;
    const int nint = (ws - h) >> 2;
    sdst[it] = 4u * (G + h) + 16u * k;
    ssrc[it] = 4u * (i * RS + h) + 16u * k;
    sg[it] = static_cast<int>(G & 31);
    srow[it] = (i < CH && k < nint) ? i : kNever;
  }
  // head / tail words of row t % CH (lanes < 2 CH): words [ht_x0, ht_x1) of the row
  int ht_x0, ht_x1, ht_gsw;
  uintptr_t ht_g;
  {
    const int i = t % CH;
    const uintptr_t G = GS0 + static_cast<uintptr_t>((1 + i) * lds);
    const int a = static_cast<int>(G & 3);
    int h = (4 - a) & 3;
    h = h < ws ? h : ws;
    const int nint = (ws - h) >> 2;
    if (t < CH) {
      ht_x0 = 0;
      ht_x1 = h;
    } else {
      ht_x0 = h + 4 * nint;
      ht_x1 = t < 2 * CH ? ws : ht_x0;
    }
    ht_g = 4u * G;
    ht_gsw = static_cast<int>(G & 31);
  }
  const int rDc = static_cast<int>((CH * ldr) & 31), sDc = static_cast<int>((CH * lds) & 31);

  // per-block chunk geometry (set at each event)
  uintptr_t s_cb = 0, r_cb = 0;
  uint32_t s_sb = 0, r_db = 0;
  int s_Dc = 0, r_Dc = 0, s_rlim = 0, r_rlim = 0;
  bool r_last = false;
  auto set_chunks = [&](int Q) {
    const int cs = Q - C::SDB, cr = Q + C::LA;
    s_cb = static_cast<uintptr_t>(cs) * sstride;
    s_sb = scR + 4u * static_cast<uint32_t>((((cs % (SR / CH)) + SR / CH) % (SR / CH)) * CH * RS);
    s_Dc = (cs * sDc) & 31;
    s_rlim = (cs >= 0 && cs < nchunks) ? n - cs * CH : 0;
    r_cb = static_cast<uintptr_t>(cr) * rstride;
    r_db = refR + 4u * static_cast<uint32_t>(((cr * CH) % RR) * RS);
    r_Dc = (cr * rDc) & 31;
    r_rlim = n - cr * CH;
    r_last = cr == nchunks - 1;
  };
  // ref chunk c: predicated cp.async of the iterations it == j (mod CH) (step j of a block)
  auto issue_ref_part = [&](int j) {
    if constexpr (!SEQ) {
#pragma unroll
      for (int it = j; it < C::ITR; it += CH)
        cp_async16_pp(rrow[it] < r_rlim && !(r_last && ((rclip >> it) & 1u)),
                      r_db + rdst[it] + 4u * static_cast<uint32_t>((rg[it] + r_Dc) & 28), reinterpret_cast<const void*>(rsrc[it] + r_cb));
    }
  };
  // the pieces of the matrix's last row that cross the end of ref: 4-byte copies of the words
  // that exist (never read past the final element); once per task, with chunk nchunks-1
  auto issue_ref_clip = [&]() {
    if constexpr (!SEQ) {
      const int c = nchunks - 1;
      const uintptr_t cb = static_cast<uintptr_t>(c) * rstride;
      const uint32_t db = refR + 4u * static_cast<uint32_t>(((c * CH) % RR) * RS);
      const int Dc = (c * rDc) & 31;
#pragma unroll
      for (int it = 0; it < C::ITR; ++it) {
        if ((rclip >> it) & 1u) {
          const uintptr_t ga = rsrc[it] + cb;
          const uint32_t dst = db + rdst[it] + 4u * static_cast<uint32_t>((rg[it] + Dc) & 28);
          for (int x = 0; x < 4; ++x)
            if (ga + 4u * x < rend) cp_async4(dst + 4u * x, reinterpret_cast<const void*>(ga + 4u * x));
        }
      }
    }
  };
  // L2 prefetch of ref chunk c: every 128-byte line of each row segment (step 0 of a block)
  auto prefetch_ref = [&](int c) {
    if constexpr (!SEQ) {
#pragma unroll
      for (int it = 0; it < (CH * C::NLINES + 31) / 32; ++it) {
        const int f = t + 32 * it;
        const int i = f / C::NLINES, ln = f - (f / C::NLINES) * C::NLINES;
        const int row = c * CH + 1 + i;
        const uintptr_t g0 = reinterpret_cast<uintptr_t>(R + static_cast<long long>(row) * ldr + c0) & ~static_cast<uintptr_t>(127);
        prefetch_l2_p(i < CH && row <= n, reinterpret_cast<const void*>(g0 + 128u * ln));
      }
    }
  };
  // score chunk c: LDS.128 + STG.128 of the interior pieces it == j (mod CH); step CH-1 also
  // moves the unaligned head / tail words
  // Score chunk c = Q - SDB leaves during block Q, software-pipelined so no LDS -> STG pair
  // stalls the warp: interior piece it is loaded (LDS.128) at step it and stored (STG.128) at
  // step it+1 (piece CH-1 at step 0 of the next block); the <= 3 unaligned head (lanes 0..CH-1)
  // / tail (lanes CH..2CH-1) words of row t % CH are loaded at step 1 and stored at step 2.
  int4 sv = make_int4(0, 0, 0, 0);
  uintptr_t sga = 0;
  bool sgo = false;
  int hv[3] = {0, 0, 0};
  uintptr_t hga = 0;
  uint32_t hgo = 0;
  auto store_part = [&](int j) {
    if (j >= 1 ? j - 1 < C::ITS : C::ITS == CH) stg128_np(sgo, reinterpret_cast<void*>(sga), sv);
    if (j < C::ITS) {
      sgo = srow[j] < s_rlim;
      sga = sdst[j] + s_cb;
      sv = lds128_np(sgo, s_sb + ssrc[j] + 4u * static_cast<uint32_t>((sg[j] + s_Dc) & 31));
    }
    if (j == 1) {
      const bool row_ok = (t % CH) < s_rlim;
      const uint32_t hb = s_sb + 4u * static_cast<uint32_t>((t % CH) * RS + ((ht_gsw + s_Dc) & 31) + ht_x0);
      hgo = 0;
#pragma unroll
      for (int x = 0; x < 3; ++x) {
        const bool g = row_ok && ht_x0 + x < ht_x1;
        hgo |= static_cast<uint32_t>(g) << x;
        hv[x] = lds32_np(g, hb + 4u * x);
      }
      hga = ht_g + s_cb + 4u * ht_x0;
    }
    if (j == 2) {
#pragma unroll
      for (int x = 0; x < 3; ++x) stg32_np((hgo >> x) & 1u, reinterpret_cast<void*>(hga + 4u * x), hv[x]);
    }
  };

  // ---- prologue: top border row, first border blocks, ref chunks 0 .. LA-1
  int Pv[K];
#pragma unroll
  for (int m = 0; m < K; ++m) Pv[m] = (t * K + m < ws) ? __ldg(S + c0 + t * K + m) : 0;
  int Lprev = (t * K < ws) ? __ldg(S + c0 + t * K - 1) : 0;  // diag input of the first row
  int vlast = Pv[K - 1];
  uint64_t e1 = src == kSrcSmem ? load_block(0) : 0ull;  // shared source: the next block's entries
  if (src != kSrcSmem)
    for (int q = 0; q < 3; ++q) prefetch_block(q);  // joins the first ref group (complete at event 0)
  // LA commit groups before event 0 (SEQ: border copies only); event Q's wait completes the
  // group of block Q-3 (the prologue's groups stand for blocks -LA .. -1)
  for (int c = 0; c < C::LA; ++c) {
    if constexpr (!SEQ) {
      set_chunks(c - C::LA);
#pragma unroll
      for (int j = 0; j < CH; ++j) issue_ref_part(j);
      if (c == nchunks - 1) issue_ref_clip();
    }
    cp_async_commit();
  }
  if constexpr (!SEQ)
    for (int c = C::LA; c < C::LA + C::PFB; ++c) prefetch_ref(c);
  // SEQ: per-band substitution profile prof[x][t] = pack_m subst[x][b[c0-1+tK+m]] (int8 x K)
  const uint8_t* const A = SEQ ? P.seq_a + pair * P.psa : nullptr;
  int a_cur = 0, a_nxt = 0;  // residues of this lane's current / next row (software pipeline)
  if constexpr (SEQ) {
    const uint8_t* const Bq = P.seq_b + pair * P.psb;
    int bj[K];
#pragma unroll
    for (int m = 0; m < K; ++m) bj[m] = (t * K + m < ws) ? (Bq[c0 - 1 + t * K + m] & 31) : 0;
    for (int x = 0; x < 32; ++x) {
      uint32_t wv = 0;
#pragma unroll
      for (int m = 0; m < K; ++m) wv |= static_cast<uint32_t>(static_cast<uint8_t>(P.subst[x * 32 + bj[m]])) << (8 * m);
      prof[x * 32 + t] = wv;
    }
    a_cur = A[min(max(-t, 0), n - 1)] & 31;     // row 1-t
    a_nxt = A[min(max(1 - t, 0), n - 1)] & 31;  // row 2-t
    __syncwarp();
  }
  const uint32_t* const profp = prof + t;

  // per-lane ring addressing: the lane's current row r = s + 1 - t sits at score ring row
  // rowS = (r-1) mod SR; its next row at ref ring row rowR = r mod RR
  const uint32_t laneR = refR + 4u * t * K, laneS = scR + 4u * t * K;
  int r = 1 - t;
  uint32_t offS = 4u * RS * static_cast<uint32_t>(((r - 1) % SR + SR) % SR);  // byte offset of ring row (r-1) mod SR
  uint32_t offR = 4u * RS * static_cast<uint32_t>((r % RR + RR) % RR);        // byte offset of ring row r mod RR
  int gS = static_cast<int>((GS0 + static_cast<uintptr_t>(static_cast<intptr_t>(r) * lds)) & 31);
  int gR = static_cast<int>((GR0 + static_cast<uintptr_t>(static_cast<intptr_t>(r + 1) * ldr)) & 31);
  const int ldr32 = static_cast<int>(ldr & 31), lds32 = static_cast<int>(lds & 31);
  int negp[K];  // -(m+1) p
#pragma unroll
  for (int m = 0; m < K; ++m) negp[m] = static_cast<int>(opaque(static_cast<uint32_t>(-(m + 1) * p)));
  uint32_t tok = 0;  // produced after each event's cp.async wait, consumed by the ref loads
  int rvn[K];        // ref of the lane's NEXT row (loaded one step ahead)
#pragma unroll
  for (int m = 0; m < K; ++m) rvn[m] = 0;
  int bp_cache = 0;  // last consumer progress read (back-pressure, smem sink)
  uint64_t cur = 0ull;

  // one wavefront step (j = step within the block, static); ALL = every lane's row in 1..n
  auto step = [&](const int Q, const int j, auto all_tag) {
    constexpr bool ALL = decltype(all_tag)::value;
    const int s = Q * CH + j;
    // ---- staging pieces (independent of the recurrence: they fill idle issue slots)
    issue_ref_part(j);
    if (j == 0) prefetch_ref(Q + C::LA + C::PFB);
    store_part(j);
    // ---- ref of this step's row (loaded last step) and the next row's loads
    int rv[K];
    if constexpr (SEQ) {
      const uint32_t pw = profp[32 * a_cur];
#pragma unroll
      for (int m = 0; m < K; ++m) rv[m] = prmt_sext(pw, 0x8880u + 0x1111u * m);
      a_cur = a_nxt;
      a_nxt = __ldg(A + min(max(r + 1, 0), n - 1)) & 31;  // residue of row r+2
    } else {
#pragma unroll
      for (int m = 0; m < K; ++m) rv[m] = rvn[m];
      const uint32_t an = laneR + offR + 4u * static_cast<uint32_t>(gR & 31);
#pragma unroll
      for (int m = 0; m < K; ++m) rvn[m] = lds_tok(an + 4 * m, tok);
    }
    // ---- left value: lane t-1's last column of this row, lane 0: the border entry
    const int bval = __shfl_sync(FULL, static_cast<int>(static_cast<uint32_t>(cur)), j);
    const int from_left = __shfl_up_sync(FULL, vlast, 1);
    const int L = (t == 0) ? bval : from_left;
    bool active = true;
    if (!ALL) active = r >= 1 && r <= n;
    if (active) {
      int Y[K];
      {
        int d = Lprev;
#pragma unroll
        for (int m = 0; m < K; ++m) {
          const int x = __viaddmax_s32(Pv[m], -p, d + rv[m]);  // max(up - p, diag + ref)
          Y[m] = m == 0 ? x : __viaddmax_s32(Y[m - 1], -p, x);
          d = Pv[m];
        }
      }
#pragma unroll
      for (int m = 0; m < K; ++m) Pv[m] = __viaddmax_s32(L, negp[m], Y[m]);  // max(L - (m+1)p, Y_m)
      Lprev = L;
      const uint32_t aS = laneS + offS + 4u * static_cast<uint32_t>(gS & 31);
#pragma unroll
      for (int m = 0; m < K; ++m) sts32_ring(aS + 4 * m, Pv[m]);
      const uint32_t vo = static_cast<uint32_t>(Pv[K - 1]);
      st_entry_smem_p(do_out && sink_smem, bring_out + 8u * (r & (C::BR - 1)), vo, gen | static_cast<uint32_t>(r));
      st_entry_gpu_p(do_out && sink_gpu, lout + r, vo, lout_tag);
      st_entry_sys_p(do_out && sink_sys, lout + r, vo, lout_tag);
    }
    (void)s;
    vlast = Pv[K - 1];
    ++r;
    offS = offS + 4u * RS == 4u * RS * SR ? 0u : offS + 4u * RS;
    offR = offR + 4u * RS == 4u * RS * RR ? 0u : offR + 4u * RS;
    gR += ldr32;
    gS += lds32;
  };

  const int nsteps = n + 31;                       // compute steps 0 .. n+30
  const int nblk = nchunks + C::SDB;               // score chunk nchunks-1 stored in block nchunks-1+SDB
  for (int Q = 0; Q < nblk; ++Q) {
    const int sig0 = Q * CH;
    const long long c_ev0 = tracing ? clock64() : 0;
    // ---- event Q
    cp_async_commit();   // copies issued during block Q-1 (ref chunk Q-1+LA, border block Q+2)
    cp_async_wait<2>();  // blocks <= Q-3 landed: ref chunks <= Q+1 (block Q reads rows <= CH*Q+CH+1),
                         // border blocks <= Q
    if (tracing) wait_cyc += clock64() - c_ev0;
    __syncwarp();        // ring writes of every lane (cp.async landed, score STS) visible warp-wide
    set_chunks(Q);
    if (!SEQ && Q + C::LA == nchunks - 1) issue_ref_clip();  // joins block Q's group
    if (sig0 < nsteps) {
      if (src == kSrcSmem) {
        cur = e1;
        e1 = load_block(Q + 1);
      } else {
        cur = read_block(Q);     // issued at event Q-3
        prefetch_block(Q + 3);   // into the slot of block Q-1 (read at the previous event)
      }
      if (src != kSrcPlain && !block_ok(cur, Q)) {
        const long long c0c = clock64();
        const uint64_t tw = globaltimer_ns();
        unsigned spins = 0;
        do {
          cur = load_block(Q);
          if ((++spins & 255u) == 0 && globaltimer_ns() - tw > P.spin_limit_ns) watchdog_trap(P.err);
        } while (!block_ok(cur, Q));
        spin_cyc += clock64() - c0c;
      }
      if (src == kSrcSmem && t == 0) sts32_volatile(prog_in, sig0 + CH);  // rows <= sig0+CH consumed
      if (sink_smem) {
        // rows written in this block are <= sig0+CH; the slot of row x held row x-BR
        const int need = sig0 + CH - C::BR;
        if (need > bp_cache && need > (bp_cache = lds32_volatile(prog_out))) {
          const long long c0c = clock64();
          const uint64_t tw = globaltimer_ns();
          while (need > (bp_cache = lds32_volatile(prog_out)))
            if (globaltimer_ns() - tw > P.spin_limit_ns) watchdog_trap(P.err);
          bp_cyc += clock64() - c0c;
        }
      }
    }
    asm volatile("mov.u32 %0, 0;" : "=r"(tok)::"memory");  // the block's ref loads stay below
    if constexpr (!SEQ) {
      if (Q == 0) {  // the first row's ref values
        const uint32_t a0 = laneR + 4u * static_cast<uint32_t>((((r - 1) % RR + RR) % RR) * RS +
                                                               static_cast<int>((GR0 + static_cast<uintptr_t>(static_cast<intptr_t>(r) * ldr)) & 31));
#pragma unroll
        for (int m = 0; m < K; ++m) rvn[m] = lds_tok(a0 + 4 * m, tok);
      }
    }
    if (tracing) ev_cyc += clock64() - c_ev0;
    // ---- CH steps
    if (sig0 >= 31 && sig0 + CH <= n) {
#pragma unroll
      for (int j = 0; j < CH; ++j) step(Q, j, std::true_type{});
    } else {
#pragma unroll
      for (int j = 0; j < CH; ++j) step(Q, j, std::false_type{});
    }
  }
  if (C::ITS == CH) stg128_np(sgo, reinterpret_cast<void*>(sga), sv);  // the last piece of the last chunk
  if (tracing && t == 0 && task < P.trace_cap) {
    unsigned smid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    unsigned long long* e = P.trace + 8 * task;
    e[0] = static_cast<unsigned long long>(task);
    e[1] = t_task0;
    e[2] = globaltimer_ns();
    e[3] = smid;
    e[4] = static_cast<unsigned long long>(ev_cyc);
    e[5] = static_cast<unsigned long long>(bp_cyc);
    e[6] = static_cast<unsigned long long>(spin_cyc);
    e[7] = static_cast<unsigned long long>(wait_cyc);
  }
}

template <class C>
__global__ void __launch_bounds__(32 * C::NW, 1) nw_wave_kernel(const __grid_constant__ StripParams P) {
  constexpr int NW = C::NW;
  extern __shared__ __align__(128) unsigned char smem[];
  const int t = threadIdx.x & 31;
  const int w = threadIdx.x >> 5;
  // CTA header: [0] group ticket, [8 + 4w] consumer progress of warp w, [128..] border rings
  unsigned long long* const s_group = reinterpret_cast<unsigned long long*>(smem);
  const uint32_t s_prog = smem_u32(smem + 8);
  unsigned char* const wsm = smem + C::kCtaHdr + w * C::kWarpSmem;
  // shared border rings start invalid (tag 0xFFFFFFFF never equals gen | row, row < 2^30)
  for (int i = threadIdx.x; i < (NW - 1) * C::BR; i += 32 * NW) reinterpret_cast<unsigned long long*>(smem + 128)[i] = ~0ull;
  if (threadIdx.x < NW) sts32_volatile(s_prog + 4 * threadIdx.x, 0);
  __syncthreads();

  int gcount = 0;  // groups processed by this CTA (generation of the shared border tags)
  for (;;) {
    if (threadIdx.x == 0) *s_group = atomicAdd(P.ticket, 1ull);
    __syncthreads();
    const long long group = static_cast<long long>(*s_group - P.ticket_base);
    if (group >= P.ngroups) break;
    const long long task = group * NW + w;
    const uint32_t gen = static_cast<uint32_t>(gcount & 3) << 30;
    if (task < P.ntasks) {
      const int band = static_cast<int>(task % P.nbands);
      const bool last_band = band == P.nbands - 1;
      int sink;
      if (last_band)
        sink = P.halo_out ? kSinkGlobal : kSinkNone;
      else
        sink = (w < NW - 1) ? kSinkSmem : kSinkGlobal;
      wave_band<C>(P, task, w, t, smem, wsm, gen, sink);
    }
    __syncthreads();  // group end: every warp done (shared border rings / progress reusable)
    if (threadIdx.x < NW) sts32_volatile(s_prog + 4 * threadIdx.x, 0);
    ++gcount;
  }
}

}  // namespace nwb200
