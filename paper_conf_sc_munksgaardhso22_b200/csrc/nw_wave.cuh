// nw_wave.cuh — the persistent NW wavefront kernel (v6): self-staging warps over row-aligned
// shared rings.
//
// What it computes (Fig. 2, with Rodinia's cell function, R1):
//     score[i][j] = max(score[i-1][j-1] + ref[i][j], score[i-1][j] - p, score[i][j-1] - p)
// for every interior cell, each value written ONCE, in place, into score (the short-circuited
// update of P:512-516 / P:616-656: no temporary, no copy).
//
// Structure (the band schedule of nw_common.cuh, pinned by P7 through band_c0 / band_ws / lane_row):
//   * A band = W = 32*K adjacent columns, all rows, swept by ONE warp; lane t owns the K adjacent
//     columns c0+tK .. c0+tK+K-1 and at step s computes row s+1-t (the intra-tile anti-diagonals
//     of P:498-501, skewed one row per lane).  The left value arrives from lane t-1 by SHFL.UP;
//     each cell is two DPX VIADDMNMX (max-plus prefix form).
//   * A CTA of NW warps claims NW consecutive bands through one atomic ticket (wavefront order;
//     band k waits only on band k-1, so no deadlock without co-residency).
//   * The sweep is latency/issue bound with one warp per SM sub-partition (measured: SHFL 24
//     cycles, DPX 4.75, LDS 29; scripts/ubench*.cu; ncu: "wait" + "selected" dominate), so the
//     compute warp does nothing but the recurrence: wide bands (K = 8: 256 cells per step),
//     row-ALIGNED shared rings (a lane's K ref values are K/4 LDS.128, its K results K/4
//     STS.128), and a paired STAGING warp (another sub-partition) moves the memory traffic:
//       - ref rows: K 4-byte cp.async per lane and row (word 32i+t of the row segment -> ring
//         word 32i+t: the copy realigns the row whatever its 16-byte phase, which the Rodinia
//         pitch n+1 changes from row to row), 8-row chunks, plus an L2 prefetch further ahead;
//       - score rows: K LDS.32 + K coalesced STG.32 per lane and row.
//     Ring row x of row r is (r-1) & (RR-1) (ref) / (r-1) & 63 (score); the row stride RS = W + 4*delta words shifts the
//     16-byte bank group by delta per row, which makes the skewed LDS/STS.128 of the 32 lanes
//     (32 different rows) conflict free (K=8: delta=1, K=4: delta=2).
//     The two warps synchronise through two 64-bit progress words in shared memory (release /
//     acquire, polled only when the cached value is insufficient): compute -> staging {ref rows
//     consumed, score rows complete}, staging -> compute {ref rows landed, score rows stored}.
//   * Compute-warp events every CE = 16 steps (blocks fully unrolled, border-lane indices
//     immediates): publish the progress word, compare the staging progress read 14 steps into the
//     previous block (in a shuffle's shadow; re-read and spin only if short), take the border
//     block, back-pressure on a shared sink.  No other synchronisation inside a band.
//   * Band handoff (the paper's Fig. 9 ordering W ∩ R = ∅): the lane holding the band's last
//     column publishes every row as a 64-bit entry {value, tag} (flag fused with the value;
//     steady blocks publish 8 rows at a time as four 16-byte pairs):
//       - to warp w+1 of the CTA: a 256-entry shared ring (tag = gen << 30 | row), back-pressure
//         on the consumer's published progress;
//       - to another CTA / GPU: a full-length global buffer (tag = launch epoch), relaxed
//         gpu / sys scope stores.
//     The consumer holds one 16-row block of entries per event (lanes 0..15): a polled producer
//     column is loaded into registers 4 steps into the previous block (relaxed 8-byte loads); a
//     complete one (the input column, or in pair mode a finished band) is copied three blocks
//     ahead by cp.async into a small shared ring; a shared source is read one block ahead.  A
//     stale block is re-polled synchronously under a %globaltimer watchdog (trap on expiry).
//   * Layouts whose interior rows are 16-byte aligned stage with 16-byte copies / stores
//     (StripParams::vec16).  The host pipeline (nw_fill[_batch]_host) gates the ref warp on
//     arrived row blocks and counts stored row blocks for the copy-out stream.
#pragma once
#include <cstdint>
#include <utility>

#include "nw_ptx.cuh"
#include "nw_common.cuh"

namespace nwb200 {

// K columns per lane (band width W = 32 K), SEQ (ref generated from the sequences), NW bands
// (compute warps) per CTA, SPB staging warps per band (1: one warp moves ref in and score out;
// 2: separate ref and store warps; 3: a ref warp and two store warps taking alternate chunks).  Warp w runs on SM sub-partition w % 4: the compute warps
// take sub-partitions 0..NW-1 and the staging warps the others (NW * (1 + SPB) <= 4).
#ifndef NW_RR
#define NW_RR 128
#endif
#ifndef NW_PFC
#define NW_PFC 4  // L2 prefetch distance of the ref stream, in 8-row chunks (A/B: 3-6 best on config 4, 33.0 vs 34.5 ms at 12; config 3 flat)
#endif
#ifndef NW_BD_GLOBAL
#define NW_BD_GLOBAL 1  // border prefetch distance (blocks) of a polled global source
#endif
#ifndef NW_PFC4
#define NW_PFC4 12  // the same for the K = 4 kernels (tiles 16..128)
#endif
#ifndef NW_BORDER_REG
#define NW_BORDER_REG 1  // polled global border blocks loaded into registers at mid-block (0: cp.async copy)
#endif
#ifndef NW_PRE_AT4
#define NW_PRE_AT4 4
#endif
#ifndef NW_PRE_AT
#define NW_PRE_AT 14  // step at which the next event's staging progress is read (A/B, scripts/gpu_ab.sh)
#endif
#ifndef NW_PF_AT
#define NW_PF_AT 4
#endif
// Experiment builds only (scripts/, _build.build_variant): NW_DEBUG_SKIP skips parts of the
// staging (bits 0-3: results invalid), relaxes the progress words (bit 4) or switches the L2
// prefetch to bulk prefetches (bit 5); NW_STAGE_SLEEP_NS backs idle staging warps off.  Both are
// compile-time: the shipped library has neither (a run-time switch could silently corrupt results).
#ifndef NW_DEBUG_SKIP
#define NW_DEBUG_SKIP 0u
#endif
// NW_STEP_EXP (experiment builds only, results invalid): strip parts of the steady step to time
// them -- 1 border-entry stores, 2 score-ring stores, 4 ref-ring loads, 8 border shuffle, 16 SEL
#ifndef NW_STEP_EXP
#define NW_STEP_EXP 0
#endif
#ifndef NW_STAGE_SLEEP_NS
#define NW_STAGE_SLEEP_NS 0
#endif
// CL > 1: thread-block clusters of CL CTAs (one band each, NW = 1) take CL consecutive bands;
// inside a cluster the border column goes straight into the next CTA's shared memory (DSMEM).
template <int K_, bool SEQ_, int NW_, int SPB_, int CL_ = 1>
struct WaveCfg {
  static constexpr int K = K_, NW = NW_, SPB = SPB_, CL = CL_;
  static_assert(CL == 1 || NW == 1, "clusters of single-band CTAs");
  static constexpr bool SEQ = SEQ_;
  static constexpr int W = 32 * K;
  static constexpr int CH = 8;                  // staging chunk (rows)
  static constexpr int CE = 16;                 // compute-warp event period (steps) = border block (rows)
  static constexpr int DELTA = K == 4 ? 2 : 1;  // 16-byte bank-group shift per ring row
  static constexpr int RS = W + 4 * DELTA;      // ring row stride (words)
  static constexpr int RR = NW_RR;               // ref ring rows (the staging warp's lookahead)
  static constexpr int SR = 64;                 // score ring rows
  static constexpr int PFC = K == 8 ? NW_PFC : NW_PFC4;  // L2 prefetch distance (chunks of CH rows) of the staging warp
  static constexpr int BR = 256;                // shared border ring entries
  static constexpr int NL = (4 * W + 127) / 128 + 1;  // 128-byte lines touched by one row segment
  static constexpr int REF_WORDS = SEQ ? 0 : RR * RS;
  static constexpr int PROF_WORDS = SEQ ? 32 * 32 * K : 0;  // int32 prof[x][lane][K] (+2p, gap-normalised)
  static constexpr int BPRE_BYTES = 4 * 8 * (CE + 2);  // border prefetch ring: 4 blocks x (CE+2) entries
  static constexpr int HDR_BYTES = 128;                // progress words: [0] compute -> staging, [8] ref -> compute, [16] store -> compute
  // NW = 2, SPB = 2: eight warps so that the two compute warps (0, 1) have SM sub-partitions 0
  // and 1 to themselves: ref warps 2, 3 and store warps 6, 7 share sub-partitions 2 and 3, warps
  // 4 and 5 idle (with six warps the store warps 4, 5 took issue slots from the compute warps)
  static constexpr bool SPREAD = NW == 2 && SPB == 2;
  static constexpr int NWARPS = SPREAD ? 8 : NW * (1 + SPB);  // per band: a compute warp and SPB staging warps
  static constexpr size_t kWarpSmem = HDR_BYTES + 4ull * (REF_WORDS + SR * RS + PROF_WORDS) + BPRE_BYTES;
  // CTA header: ticket, progress words, the border rings between consecutive bands (NW - 1
  // between the warps of the CTA; CL > 1: one incoming ring written by the previous CTA)
  static constexpr size_t kCtaHdr = 128 + static_cast<size_t>(CL > 1 ? 1 : NW - 1) * BR * 8;
  static constexpr size_t kSmem = kCtaHdr + NW * kWarpSmem;
  static_assert(K == 4 || K == 8, "K/4 LDS.128 per step");
  static_assert((RS * 4 / 16) % 8 == DELTA, "bank-group shift");
  static_assert(kWarpSmem % 32 == 0 && kCtaHdr % 32 == 0 && (HDR_BYTES + 4 * (REF_WORDS + SR * RS)) % 32 == 0,
                "32-byte aligned rings (the profile's half-swap flips address bit 4)");
  static_assert(NL <= 32 && NW <= 8 && SPB >= 1 && SPB <= 3 && NWARPS <= 8, "geometry");
  static_assert(RR % CH == 0 && (RR & (RR - 1)) == 0 && SR % CH == 0 && (SR & (SR - 1)) == 0 && RR >= 64 && SR >= 64,
                "rings of whole chunks, powers of two, large enough for the staging schedule");
};

// ---- inline PTX helpers (immediate offsets keep the per-step staging at one instruction per copy)
template <int DOFF, int SOFF>
__device__ __forceinline__ void cp_async4_imm2(uint32_t dst, uint64_t src) {
  asm volatile("cp.async.ca.shared.global [%0+%2], [%1+%3], 4;" ::"r"(dst), "l"(src), "n"(DOFF), "n"(SOFF) : "memory");
}
// one row: K 4-byte copies / K 4-byte shared loads at compile-time offsets DBASE + 128 I
template <int DBASE, int K>
__device__ __forceinline__ void cp_row(uint32_t d0, uint64_t src) {
  [&]<int... I>(std::integer_sequence<int, I...>) { (cp_async4_imm2<DBASE + 128 * I, 128 * I>(d0, src), ...); }(std::make_integer_sequence<int, K>{});
}
template <int OFF>
__device__ __forceinline__ void cp_async4_imm_p(bool p, uint32_t dst, uint64_t src) {
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %0, 0; @q cp.async.ca.shared.global [%1+%3], [%2+%3], 4; }" ::"r"(
                   static_cast<int>(p)),
               "r"(dst), "l"(src), "n"(OFF)
               : "memory");
}
// 16-byte forms for layouts whose interior rows start 16-byte aligned (StripParams::vec16)
template <int DOFF, int SOFF>
__device__ __forceinline__ void cp_async16_imm2(uint32_t dst, uint64_t src) {
  asm volatile("cp.async.cg.shared.global [%0+%2], [%1+%3], 16;" ::"r"(dst), "l"(src), "n"(DOFF), "n"(SOFF) : "memory");
}
template <int OFF>
__device__ __forceinline__ int4 lds128_imm(uint32_t a) {
  int4 v;
  asm volatile("ld.shared.v4.b32 {%0, %1, %2, %3}, [%4+%5];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a), "n"(OFF) : "memory");
  return v;
}
template <int OFF>
__device__ __forceinline__ void stg128_imm(uint64_t g, int4 v) {
  asm volatile("st.global.v4.b32 [%0+%5], {%1, %2, %3, %4};" ::"l"(g), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w), "n"(OFF) : "memory");
}
template <int OFF>
__device__ __forceinline__ int lds32_imm(uint32_t a) {
  int v;
  asm volatile("ld.shared.b32 %0, [%1+%2];" : "=r"(v) : "r"(a), "n"(OFF) : "memory");
  return v;
}
template <int DBASE, int K>
__device__ __forceinline__ void lds_row(uint32_t a0, int* v) {
  [&]<int... I>(std::integer_sequence<int, I...>) { ((v[I] = lds32_imm<DBASE + 128 * I>(a0)), ...); }(std::make_integer_sequence<int, K>{});
}
template <int OFF>
__device__ __forceinline__ void stg32_imm(uint64_t g, int v) {
  asm volatile("st.global.b32 [%0+%2], %1;" ::"l"(g), "r"(v), "n"(OFF) : "memory");
}
template <int OFF>
__device__ __forceinline__ void stg32_imm_p(bool p, uint64_t g, int v) {
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %0, 0; @q st.global.b32 [%1+%3], %2; }" ::"r"(static_cast<int>(p)), "l"(g), "r"(v),
               "n"(OFF)
               : "memory");
}
// ref ring loads: not volatile (the compiler may schedule them), but they consume the token
// produced after each event's wait, so they never move above it
template <int OFF>
__device__ __forceinline__ int4 lds128_tok(uint32_t a, uint32_t tok) {
  int4 v;
  asm("ld.shared.v4.b32 {%0, %1, %2, %3}, [%4+%6];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a), "r"(tok), "n"(OFF));
  return v;
}
// score ring stores (ordered by the events' __syncwarp, not by the compiler)
template <int OFF>
__device__ __forceinline__ void sts128_ring(uint32_t a, int x, int y, int z, int w) {
  asm volatile("st.shared.v4.b32 [%0+%5], {%1, %2, %3, %4};" ::"r"(a), "r"(x), "r"(y), "r"(z), "r"(w), "n"(OFF));
}
// Border-entry stores {value, tag}.  Every entry is ONE 8-byte element (a .b64 scalar or an element
// of a .v2.b64 vector), so a relaxed load that sees an entry's tag sees the value stored with it
// (single-copy atomicity of aligned 8-byte elements; PTX treats a vector access as accesses to its
// elements).  The two 32-bit halves are packed into the 64-bit operand inside the asm block.
#define NW_ENT1(SCOPE_SPACE, ADDR_T)                                                                         \
  asm volatile("{ .reg .pred q; .reg .b64 e; setp.ne.b32 q, %0, 0; mov.b64 e, {%2, %3}; @q st." SCOPE_SPACE \
               ".b64 [%1], e; }" ::"r"(static_cast<int>(pred)),                                              \
               ADDR_T(p), "r"(lo), "r"(hi)                                                                   \
               : "memory")
#define NW_ENT2(SCOPE_SPACE, ADDR_T)                                                                          \
  asm volatile("{ .reg .pred q; .reg .b64 e0, e1; setp.ne.b32 q, %0, 0; mov.b64 e0, {%2, %3}; mov.b64 e1, {%4, %5}; " \
               "@q st." SCOPE_SPACE ".v2.b64 [%1], {e0, e1}; }" ::"r"(static_cast<int>(pred)),                \
               ADDR_T(p), "r"(v0), "r"(t0), "r"(v1), "r"(t1)                                                  \
               : "memory")
__device__ __forceinline__ void st_entry_gpu_p(bool pred, uint64_t* p, uint32_t lo, uint32_t hi) { NW_ENT1("relaxed.gpu.global", "l"); }
__device__ __forceinline__ void st_entry_sys_p(bool pred, uint64_t* p, uint32_t lo, uint32_t hi) { NW_ENT1("relaxed.sys.global", "l"); }
__device__ __forceinline__ void st_entry_smem_p(bool pred, uint32_t p, uint32_t lo, uint32_t hi) { NW_ENT1("volatile.shared", "r"); }

// two consecutive border entries (rows 2k, 2k+1: 16-byte aligned) in one store of two 8-byte elements
__device__ __forceinline__ void st_pair_gpu_p(bool pred, uint64_t* p, uint32_t v0, uint32_t t0, uint32_t v1, uint32_t t1) {
  NW_ENT2("relaxed.gpu.global", "l");
}
__device__ __forceinline__ void st_pair_sys_p(bool pred, uint64_t* p, uint32_t v0, uint32_t t0, uint32_t v1, uint32_t t1) {
  NW_ENT2("relaxed.sys.global", "l");
}
__device__ __forceinline__ void st_pair_smem_p(bool pred, uint32_t p, uint32_t v0, uint32_t t0, uint32_t v1, uint32_t t1) {
  NW_ENT2("volatile.shared", "r");
}

// DSMEM (shared::cluster addresses from mapa): the next CTA's incoming ring / progress word
__device__ __forceinline__ uint32_t mapa_u32(uint32_t a, uint32_t rank) {
  uint32_t d;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(rank));
  return d;
}
__device__ __forceinline__ void st_pair_dsmem_p(bool pred, uint32_t p, uint32_t v0, uint32_t t0, uint32_t v1, uint32_t t1) {
  NW_ENT2("relaxed.cluster.shared::cluster", "r");
}
__device__ __forceinline__ void st_entry_dsmem_p(bool pred, uint32_t p, uint32_t lo, uint32_t hi) {
  NW_ENT1("relaxed.cluster.shared::cluster", "r");
}
__device__ __forceinline__ int ld_dsmem_b32(uint32_t a) {
  int v;
  asm volatile("ld.relaxed.cluster.shared::cluster.b32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ uint32_t cluster_ctarank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned; barrier.cluster.wait.acquire.aligned;" ::: "memory");
}

enum : int { kRoleRef = 1, kRoleStore = 2, kRoleIdle = 4 };  // staging-warp roles

// Shared per-band geometry of the compute and staging warps.
template <class C>
struct BandGeo {
  int n, p, band, c0, ws;
  bool last_band;
  long long pair;
  int32_t* S;
  const int32_t* Rf;
  uint32_t hdr, refR, scR, prof, bpre;  // shared addresses of the band's regions
  __device__ __forceinline__ BandGeo(const StripParams& P, long long task, unsigned char* wsm) {
    n = static_cast<int>(P.n);
    p = P.p;
    pair = task / P.nbands;
    band = static_cast<int>(task - pair * P.nbands);
    last_band = band == P.nbands - 1;
    c0 = band_c0(band, C::W);
    ws = band_ws(P.width, band, C::W);
    S = P.score + pair * P.pss;
    Rf = C::SEQ ? nullptr : P.ref + pair * P.psr;
    hdr = opaque(smem_u32(wsm));  // kept in a register (else ptxas re-derives the shared window per use)
    refR = hdr + C::HDR_BYTES;
    scR = refR + 4u * C::REF_WORDS;
    prof = scR + 4u * C::SR * C::RS;
    bpre = prof + 4u * C::PROF_WORDS;
  }
};

// progress-word accessors (all lanes load: the value is uniform; lane 0 stores after __syncwarp)
__device__ __forceinline__ void prog_publish(uint32_t a, int lo, int hi, bool relaxed = false) {
  __syncwarp();  // every lane's prior shared-memory accesses happen before lane 0's release
  if ((threadIdx.x & 31) == 0) {
    if (relaxed)
      asm volatile("{ .reg .b64 e; mov.b64 e, {%1, %2}; st.volatile.shared.b64 [%0], e; }" ::"r"(a), "r"(lo), "r"(hi) : "memory");
    else
      st_release_cta_v2(a, static_cast<uint32_t>(lo), static_cast<uint32_t>(hi));
  }
}
__device__ __forceinline__ void prog_read(uint32_t a, int& lo, int& hi) {
  const uint64_t v = ld_acquire_cta(a);
  lo = static_cast<int>(static_cast<uint32_t>(v));
  hi = static_cast<int>(static_cast<uint32_t>(v >> 32));
}

// The staging warp of a band: ref rows in (8-row chunks of 4-byte cp.async, paced by the ring
// space the compute warp has released), score rows out (LDS.32 + coalesced STG.32 once the compute
// warp has completed them), L2 prefetch ahead of the ref stream.
// half (store roles): -1 = every score chunk, 0 / 1 = the even / odd chunks (SPB = 3).  A store
// warp publishes, in its progress word (hdr + 16 + 8 half), the index of its next chunk: all of
// its chunks below it are stored.
template <class C, bool RAGGED, int ROLE>
__device__ __forceinline__ void wave_stage(const StripParams& P, const long long task, const int t, unsigned char* const wsm,
                                           const int half = -1) {
  constexpr bool DO_REF = (ROLE & kRoleRef) != 0, DO_ST = (ROLE & kRoleStore) != 0;
  constexpr int K = C::K, CH = C::CH, RR = C::RR, SR = C::SR;
  constexpr uint32_t RS4 = 4u * C::RS;
  constexpr bool SEQ = C::SEQ;
  const BandGeo<C> g(P, task, wsm);
  const int n = g.n;
  const int nch = (n + CH - 1) / CH;
  const uint32_t from_c = g.hdr, to_ref = opaque(g.hdr + 8), to_st = opaque(g.hdr + 16 + 8 * (half > 0));
  const int kstep = half >= 0 ? 2 : 1;  // score chunks handled: ks, ks + kstep, ...
  uint32_t wmask = 0;  // RAGGED: bit i = word 32i+t of the row segment exists
#pragma unroll
  for (int i = 0; i < K; ++i) wmask |= static_cast<uint32_t>(32 * i + t < g.ws) << i;
  const uint64_t ldr4 = 4ull * static_cast<uint64_t>(P.ldr), lds4 = 4ull * static_cast<uint64_t>(P.lds);
  const uint64_t gR0 = SEQ ? 0ull : reinterpret_cast<uint64_t>(g.Rf + g.c0 + t);  // (row 0, word t) of the ref segment
  const bool vec16 = P.vec16 != 0;  // interior rows 16-byte aligned: 16-byte copies / stores (host-checked)
  // progress words: release stores / acquire loads (NW_DEBUG_SKIP bit 4, experiment builds: relaxed;
  // measured: no difference, 3.08 vs 3.11 ms at n = 32768, 37.65 vs 37.53 ms on config 4)
  constexpr bool strict = (NW_DEBUG_SKIP & 16u) == 0;
  const uint64_t gS0 = reinterpret_cast<uint64_t>(g.S + g.c0 + t);
  int consumed = 0, complete = 0;  // cached compute-warp progress
  int landed = 0, stored = 0;      // published to the compute warp
  // chunk k of ref: rows CH*k+1 .. CH*k+CH (row i of the chunk: K copies per lane).  Chunks are
  // issued / stored in order, so the global row pointers advance incrementally; ring offsets
  // within a chunk are compile-time immediates (a chunk never wraps: RR, SR multiples of CH).
  uint64_t gR = SEQ ? 0ull : gR0 + ldr4;  // (row CH*kr+1, word t) of the next ref chunk
  auto issue_chunk = [&](int k) {
    if constexpr (!SEQ) {
      const uint32_t d0 = g.refR + static_cast<uint32_t>((CH * k) & (RR - 1)) * RS4 + 4u * t;
      uint64_t gsrc = gR;
      gR += CH * ldr4;
      if (!RAGGED && vec16 && CH * k + CH <= n) {
        // 16-byte copies: lane t moves words 4t..4t+3 (+128: K = 8) of each row, 1 or 2 per row
        const uint32_t dv = g.refR + static_cast<uint32_t>((CH * k) & (RR - 1)) * RS4 + 16u * t;
        uint64_t gv = gsrc - 4ull * t + 16ull * t;
        [&]<int... R>(std::integer_sequence<int, R...>) {
          ((cp_async16_imm2<R * 4 * C::RS, 0>(dv, gv), (K == 8 ? cp_async16_imm2<R * 4 * C::RS + 512, 512>(dv, gv) : void()), gv += ldr4), ...);
        }(std::make_integer_sequence<int, CH>{});
      } else if (!RAGGED && CH * k + CH <= n) {
        [&]<int... R>(std::integer_sequence<int, R...>) {
          ((cp_row<R * 4 * C::RS, K>(d0, gsrc), gsrc += ldr4), ...);
        }(std::make_integer_sequence<int, CH>{});
      } else {
#pragma unroll
        for (int i = 0; i < CH; ++i) {
          const int ri = CH * k + 1 + i;
          const uint32_t d = d0 + static_cast<uint32_t>(i) * RS4;
          if (ri <= n) {
            [&]<int... I>(std::integer_sequence<int, I...>) {
              (cp_async4_imm_p<128 * I>(!RAGGED || ((wmask >> I) & 1u), d, gsrc), ...);
            }(std::make_integer_sequence<int, K>{});
          }
          gsrc += ldr4;
        }
      }
    }
  };
  // L2 prefetch of chunk k's rows: CH rows x NL 128-byte lines, lane t handles lines t, t+32, ...
  // (NW_DEBUG_SKIP bit 5, experiment builds: one cp.async.bulk.prefetch.L2 per row instead)
  const uint32_t pf_bytes = static_cast<uint32_t>((4 * g.ws + 12 + 15) & ~15);
  auto prefetch_chunk = [&](int k) {
    if constexpr (!SEQ) {
      if constexpr ((NW_DEBUG_SKIP & 32u) != 0) {
        const int rp = CH * k + 1 + t;
        if (t < CH && rp <= n) {
          const uint64_t ga = (reinterpret_cast<uint64_t>(g.Rf + g.c0) + static_cast<uint64_t>(static_cast<long long>(rp)) * ldr4) & ~15ull;
          asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(ga), "r"(pf_bytes) : "memory");
        }
        return;
      }
#pragma unroll
      for (int f = t; f < CH * C::NL; f += 32) {
        const int i = f / C::NL, ln = f - (f / C::NL) * C::NL;
        const int rp = CH * k + 1 + i;
        const uint64_t ga = (reinterpret_cast<uint64_t>(g.Rf + g.c0) + static_cast<uint64_t>(static_cast<long long>(rp)) * ldr4) & ~127ull;
        prefetch_l2_p(rp <= n, reinterpret_cast<const void*>(ga + 128u * ln));
      }
    }
  };
  // the compute warp's ring holds the gap-normalised S' = S + (i + j) p: the
  // store converts back, one IADD3 per value: S = S' - r p - (c0 + 32 I + t) p
  int colp[K];
#pragma unroll
  for (int I = 0; I < K; ++I) colp[I] = -(g.c0 + 32 * I + t) * g.p;
  int cp16[K];  // 16-byte path: column terms of words 4t + j (+128)
#pragma unroll
  for (int j = 0; j < K; ++j) cp16[j] = -(g.c0 + 4 * t + (j & 3) + 128 * (j >> 2)) * g.p;
  uint64_t gS = gS0 + lds4 + (half > 0 ? CH * lds4 : 0ull);  // (row CH*ks+1, word t) of the next score chunk
  auto store_chunk = [&](int k) {
    const uint32_t a0 = g.scR + static_cast<uint32_t>((CH * k) & (SR - 1)) * RS4 + 4u * t;
    uint64_t ga = gS;
    gS += static_cast<uint64_t>(kstep * CH) * lds4;
    int rp = -(CH * k + 1) * g.p;
    if (!RAGGED && vec16 && CH * k + CH <= n) {
      // 16-byte path: LDS.128 of ring words 4t..4t+3 (+128), one IADD3 per value, STG.128
      const uint32_t av = g.scR + static_cast<uint32_t>((CH * k) & (SR - 1)) * RS4 + 16u * t;
      uint64_t gv = ga - 4ull * t + 16ull * t;
#pragma unroll
      for (int i = 0; i < CH; ++i) {
        [&]<int... H>(std::integer_sequence<int, H...>) {
          ((void)[&] {
             int4 v = lds128_imm<H * 512>(av + static_cast<uint32_t>(i) * RS4);
             v.x += rp + cp16[4 * H], v.y += rp + cp16[4 * H + 1], v.z += rp + cp16[4 * H + 2], v.w += rp + cp16[4 * H + 3];
             stg128_imm<H * 512>(gv, v);
           }(), ...);
        }(std::make_integer_sequence<int, K / 4>{});
        gv += lds4;
        rp -= g.p;
      }
    } else if (!RAGGED && CH * k + CH <= n) {
      // the common case: K LDS + K IADD3 + K unpredicated coalesced STG per row
      int v[CH][K];
      [&]<int... R>(std::integer_sequence<int, R...>) { (lds_row<R * 4 * C::RS, K>(a0, v[R]), ...); }(std::make_integer_sequence<int, CH>{});
      // all conversions first, then the stores back to back (an IADD3 -> STG pair per value
      // serialises on the ALU latency: measured 11 cycles per value)
#pragma unroll
      for (int i = 0; i < CH; ++i) {
#pragma unroll
        for (int I = 0; I < K; ++I) v[i][I] += rp + colp[I];
        rp -= g.p;
      }
#pragma unroll
      for (int i = 0; i < CH; ++i) {
        [&]<int... I>(std::integer_sequence<int, I...>) { (stg32_imm<128 * I>(ga, v[i][I]), ...); }(std::make_integer_sequence<int, K>{});
        ga += lds4;
      }
    } else {
#pragma unroll
      for (int i = 0; i < CH; ++i) {
        const int ro = CH * k + 1 + i;
        const uint32_t a = a0 + static_cast<uint32_t>(i) * RS4;
        int v[K];
        [&]<int... I>(std::integer_sequence<int, I...>) { ((v[I] = lds32_imm<128 * I>(a)), ...); }(std::make_integer_sequence<int, K>{});
        [&]<int... I>(std::integer_sequence<int, I...>) {
          (stg32_imm_p<128 * I>(ro <= n && (!RAGGED || ((wmask >> I) & 1u)), ga, v[I] + rp + colp[I]), ...);
        }(std::make_integer_sequence<int, K>{});
        ga += lds4;
        rp -= g.p;
      }
    }
  };

  // Event loop (never blocks on one side while the other could progress): issue ref chunk kr
  // once rows <= CH*kr+CH-RR are consumed (ring space), store score chunk ks once complete, and
  // publish the ref chunks landed (all but the LAG most recent) and the score chunks stored.  The
  // compute warp, at event Q (step CE*Q), has consumed ref rows <= CE*Q-30 and completed score
  // rows <= CE*Q-31, and needs ref rows <= CE*Q+CE+1 landed and score rows <= CE*Q+CE-SR stored:
  // with RR = 128 the ref stream runs about RR/2 rows ahead, so both waits are satisfiable
  // (no deadlock) and normally already satisfied.
  constexpr int LAG = 3;
  const bool tracing = kTrace && P.trace2 != nullptr && task < P.trace_cap;
  long long st_busy = 0, st_gap_sum = 0, st_last = tracing ? clock64() : 0;  // (trace) store-warp cycles
  int kr = (SEQ || !DO_REF) ? nch : 0, ks = DO_ST ? max(half, 0) : nch;
  unsigned rdy = 0;  // host pipeline: cached arrived row blocks
  long long sig_c = P.rows_done != nullptr ? (g.pair * (P.n + 1) + 1) / P.chunk_rows : 0;  // next block to release
  const uint64_t tw0 = globaltimer_ns();
  uint64_t tw = tw0;
  unsigned idle = 0;
  for (;;) {
    bool did = false;
    if (!SEQ && kr < nch) {
      const int need = CH * kr + CH - RR;
      if (consumed < need) prog_read(from_c, consumed, complete);
      // host pipeline (nw_fill[_batch]_host): the chunk's ref rows must have arrived; the copy
      // stream publishes arrived row blocks in *ref_ready (after each copy, stream-ordered)
      bool arrived = true;
      if (P.ref_ready != nullptr) {
        const long long rhi = g.pair * (P.n + 1) + min(n, CH * kr + CH);
        const unsigned need_c = static_cast<unsigned>(rhi / P.chunk_rows) + 1u;
        if (rdy < need_c) rdy = ld_acquire_gpu_u32(P.ref_ready);
        arrived = rdy >= need_c;
      }
      if (consumed >= need && arrived) {
        if constexpr (!(NW_DEBUG_SKIP & 5u)) issue_chunk(kr);  // (experiment builds only: results invalid)
        if (kr + C::PFC < nch) prefetch_chunk(kr + C::PFC);
        cp_async_commit();
        ++kr;
        did = true;
      }
    }
    if (ks < nch) {
      const int need = min(n, CH * ks + CH);  // (chunk ks complete)
      if (complete < need) prog_read(from_c, consumed, complete);
      if (complete >= need) {
        const long long cs0 = tracing ? clock64() : 0;
        if constexpr (!(NW_DEBUG_SKIP & 9u)) store_chunk(ks);
        if (tracing) st_busy += clock64() - cs0, st_gap_sum += cs0 - st_last, st_last = clock64();
        ks += kstep;
        if (P.rows_done != nullptr) {
          // host pipeline: every row block of the stacked matrix below this warp's next chunk is
          // stored (as far as this warp's chunks go): release it to the device->host copy stream
          const long long gb = g.pair * (P.n + 1);
          const long long c_end = ks < nch ? (gb + CH * ks + 1) / P.chunk_rows : (gb + n) / P.chunk_rows + 1;
          if (sig_c < c_end) {
            __threadfence();  // this lane's score stores before the counter (gpu scope)
            __syncwarp();
            if (t == 0)
              for (long long c = sig_c; c < c_end; ++c) atomicAdd(P.rows_done + c, 1u);
            sig_c = c_end;
          }
        }
        did = true;
      }
    }
    bool done = true;
    if constexpr (DO_REF) {
      int nl;
      if (SEQ || kr == nch) {
        cp_async_wait<0>();
        nl = n;
      } else {
        cp_async_wait<LAG>();  // chunks <= kr-1-LAG landed (this lane's copies)
        nl = min(n, max(0, CH * (kr - LAG)));
      }
      if (nl > landed) {
        landed = nl;
        // release: every lane's copies have completed (wait_group) before the __syncwarp and
        // this store; the compute warp's acquire load orders its ring reads after them
        prog_publish(to_ref, landed, 0, !strict);
      }
      done = landed == n;
    }
    if constexpr (DO_ST) {
      const int ns = min(ks, nch);  // my chunks below ns are stored
      if (ns > stored) {
        stored = ns;
        // release: the ring slots were READ (every STG above consumed its LDS result) before the
        // compute warp, after its acquire load, rewrites them
        prog_publish(to_st, stored, 0, !strict);
      }
      done = done && ks >= nch;
    }
    if (done) break;
    if (did) {
      idle = 0;
    } else {
      // idle: back off (a tight poll of the progress words competes with the compute warp's
      // shared-memory / shuffle traffic in the SM's MIO pipe)
      if constexpr (NW_STAGE_SLEEP_NS > 0) __nanosleep(NW_STAGE_SLEEP_NS);
      if ((++idle & 255u) == 0) {
        const uint64_t now = globaltimer_ns();
        if (idle == 256) tw = now;
        else if (now - tw > P.spin_limit_ns) watchdog_trap(P.err);
      }
    }
  }
  (void)tw0;
  if constexpr (DO_ST) {
    if (tracing && t == 0) {
      P.trace2[8 * task + 4] = static_cast<unsigned long long>(st_busy);
      P.trace2[8 * task + 5] = static_cast<unsigned long long>(st_gap_sum);
    }
  }
}

// The compute warp of a band: the wavefront sweep (no staging instructions in the step).
// SRC (compile time): where the band's left border column comes from.
// HALO_OUT (compile time): the band pushes its last column into a strip halo, whose entries
// hold the true S (nw.h), not the kernel's gap-normalised S'.
template <class C, bool RAGGED, int SRC, bool HALO_OUT, bool REMOTE = false>
__device__ __forceinline__ void wave_band(const StripParams& P, const long long task, const int w, const int t,
                                          unsigned char* const smem, unsigned char* const wsm, const uint32_t gen,
                                          const int sink) {
  constexpr int K = C::K, CE = C::CE, RR = C::RR, SR = C::SR;
  constexpr uint32_t RS4 = 4u * C::RS;
  constexpr bool SEQ = C::SEQ;
  constexpr unsigned FULL = 0xffffffffu;
  // border prefetch distance (blocks): a polled global source (the previous band still running)
  // is copied one block ahead -- an older snapshot would add its age to the band-to-band lag; a
  // complete source (the input column, or in pair mode the finished previous band, whose entries
  // come back from HBM) three blocks ahead so the copy's latency is hidden (one block ahead exposed
  // ~350 cycles per event on config 4)
  const int BD = (SRC == kSrcGlobal && !P.pair_mode) ? NW_BD_GLOBAL : 3;
  const bool tracing = kTrace && P.trace != nullptr;
  const unsigned long long t_task0 = tracing ? globaltimer_ns() : 0ull;
  long long spin_cyc = 0, wait_cyc = 0, bp_cyc = 0, steady_cyc = 0, steady_blocks = 0;
  long long ph_cyc[3] = {0, 0, 0}, st_wait_cyc = 0, pub_cyc = 0;  // event phases: publish + staging wait, border (+ spin), back-pressure + misc
  constexpr bool strict = (NW_DEBUG_SKIP & 16u) == 0;  // release-stored progress words (above)

  const BandGeo<C> g(P, task, wsm);
  const int n = g.n, p = g.p, band = g.band, c0 = g.c0, ws = g.ws;
  const long long pair = g.pair;
  const long long lds = P.lds;
  const uint32_t to_s = g.hdr, from_r = opaque(g.hdr + 8), from_t = opaque(g.hdr + 16);
  const uint32_t s_prog = opaque(smem_u32(smem + 8));     // [4w]: rows consumed by warp w (shared source)
  const uint32_t s_bring = opaque(smem_u32(smem + 128));  // [w * BR * 8]: ring warp w -> w+1

  // ---- border source (left)
  const uint64_t* lin = nullptr;
  uint32_t lin_epoch = 0;
  bool lin_sys = false;
  if (band == 0) {
    lin = P.halo_in;
    lin_sys = true;
    lin_epoch = P.halo_epoch;
  } else if (SRC == kSrcGlobal) {
    lin = P.xbuf + (pair * (P.nbands - 1) + band - 1) * xstride(n);
    lin_epoch = P.epoch;
  }
  // CL > 1 (NW = 1): the incoming ring at s_bring is written by the previous CTA of the cluster;
  // REMOTE: this band's out-ring / consumer progress live in the next CTA (DSMEM addresses)
  const uint32_t bring_in = C::CL > 1 ? s_bring : s_bring + (w - 1) * C::BR * 8;
  const uint32_t prog_in = s_prog + 4 * w;  // written by this warp (consumer of the previous band)
  uint32_t bring_out = s_bring + w * C::BR * 8, prog_out = s_prog + 4 * (w + 1);
  if constexpr (REMOTE) {
    const uint32_t nxt = cluster_ctarank() + 1;
    bring_out = mapa_u32(s_bring, nxt);
    prog_out = mapa_u32(s_prog, nxt);
  }
  const int32_t* const colp = g.S + (c0 - 1);      // plain left border column
  // ---- sink (right)
  uint64_t* lout = nullptr;
  uint32_t lout_tag = 0;
  const bool sink_smem = sink == kSinkSmem;
  bool sink_gpu = false, sink_sys = false;
  if (sink == kSinkGlobal) {
    if (g.last_band) {
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
  const int out_m = (ws - 1) - out_lane * K;  // the band's last column within the out lane
  const bool do_out = t == out_lane && sink != kSinkNone;

  // ---- border blocks: lane j < CE of block q holds the entry of row CE*q + 1 + j
  auto load_block = [&](int q) -> uint64_t {  // synchronous (shared source / re-poll)
    const int row = CE * q + 1 + t;
    if (t >= CE || row > n) return 0ull;
    if constexpr (SRC == kSrcGlobal) return lin_sys ? ld_relaxed_sys(lin + row) : ld_relaxed_gpu(lin + row);
    if constexpr (SRC == kSrcSmem) return lds64_volatile(bring_in + 8u * (row & (C::BR - 1)));
    return static_cast<uint32_t>(__ldg(colp + static_cast<long long>(row) * lds));
  };
  // Global / plain sources: block q is copied by cp.async BD blocks ahead (one commit group per
  // event) into slot q & 3 of a shared ring -- a polled global source ONE block ahead (an older
  // snapshot would add its age to the band-to-band lag), the plain input column three blocks
  // ahead: rows CE*q .. CE*q+CE+1 (global: 16-byte pairs (2k, 2k+1) through L2 only, never via L1
  // since the entries are polled; plain: the 4-byte values of score column c0-1).  No register
  // holds an in-flight load across an event (a register move of one stalls for the latency).
  auto prefetch_block = [&](int q) {
    const uint32_t slot = g.bpre + 8u * (CE + 2) * static_cast<uint32_t>(q & 3);
    if constexpr (SRC == kSrcGlobal) {
      const int row = CE * q + 2 * t;
      cp_async16_cg_p(t <= CE / 2 && row <= n, slot + 16u * t, lin + row);
    } else if constexpr (SRC == kSrcPlain) {
      const int row = CE * q + 1 + t;
      cp_async4_p(t < CE && row <= n, slot + 8u * (1 + t), colp + static_cast<long long>(row) * lds);
    }
  };
  auto read_block = [&](int q) -> uint64_t {
    const uint32_t slot = g.bpre + 8u * (CE + 2) * static_cast<uint32_t>(q & 3);
    return t < CE ? lds64_volatile(slot + 8u * (1 + t)) : 0ull;
  };
  // number of leading rows of block q whose entries in e are valid (uniform)
  auto leading_valid = [&](uint64_t e, int q) -> int {
    const int row = CE * q + 1 + t;
    bool ok = true;
    if (t < CE && row <= n) {
      const uint32_t hi = static_cast<uint32_t>(e >> 32);
      if constexpr (SRC == kSrcGlobal)
        ok = hi == lin_epoch;
      else if constexpr (SRC == kSrcSmem)
        ok = hi == (gen | static_cast<uint32_t>(row));
    }
    const unsigned bad = ~__ballot_sync(FULL, ok);
    return bad ? __ffs(bad) - 1 : 32;
  };

  // ---- prologue: top border row, first border blocks
  // gap-normalised values S' = S + (i + j) p; row 0: S'(0, j) = S(0, j) + j p
  int Pv[K];
#pragma unroll
  for (int m = 0; m < K; ++m) Pv[m] = (t * K + m < ws) ? __ldg(g.S + c0 + t * K + m) + (c0 + t * K + m) * p : 0;
  int Lprev = (t * K < ws) ? __ldg(g.S + c0 + t * K - 1) + (c0 + t * K - 1) * p : 0;  // diag input of the first row
  uint64_t e1 = 0ull;                                           // shared source: the next block's entries
  if (SRC == kSrcSmem || (SRC == kSrcGlobal && BD == 1 && NW_BORDER_REG)) {
    e1 = load_block(0);
  } else {
    for (int q = 0; q < BD; ++q) prefetch_block(q);
    cp_async_commit();
  }

  // SEQ: per-band substitution profile prof[x][t][m] = subst[x][b[c0-1+tK+m]] + 2p (int32, the
  // diagonal move of the gap-normalised recurrence).  K = 8: lane t's two 16-byte halves are
  // swapped when bit 2 of t is set, so the 8 lanes of an LDS.128 phase cover all 32 banks.
  const uint8_t* const A = SEQ ? P.seq_a + pair * P.psa : nullptr;
  int a_cur = 0, a_nxt = 0;  // residues of this lane's current / next row (software pipeline)
  const uint32_t sw = K == 8 ? ((t >> 2) & 1u) : 0u;
  if constexpr (SEQ) {
    int* const prof = reinterpret_cast<int*>(wsm + (g.prof - g.hdr));
    const uint8_t* const Bq = P.seq_b + pair * P.psb;
    int bj[K];
#pragma unroll
    for (int m = 0; m < K; ++m) bj[m] = (t * K + m < ws) ? (Bq[c0 - 1 + t * K + m] & 31) : 0;
    for (int x = 0; x < 32; ++x) {
#pragma unroll
      for (int m = 0; m < K; ++m)
        prof[(x * 32 + t) * K + 4 * ((m >> 2) ^ sw) + (m & 3)] = static_cast<int>(P.subst[x * 32 + bj[m]]) + 2 * p;
    }
    a_cur = A[min(max(1 - t, 0), n - 1)] & 31;  // row 2-t (row 1-t's profile row is loaded at event 0)
    a_nxt = A[min(max(2 - t, 0), n - 1)] & 31;  // row 3-t
    __syncwarp();
  }
  const uint32_t profA = opaque(g.prof + 4u * K * t + 16u * sw);

  uint32_t tok = 0;  // produced after each event's acquire, consumed by the ref loads
  int rvn[K];        // ref of the lane's NEXT row (loaded one step ahead)
#pragma unroll
  for (int m = 0; m < K; ++m) rvn[m] = 0;
  int bp_cache = 0;            // last consumer progress read (back-pressure, shared sink)
  int landed = 0, stored = 0;  // cached staging-warp progress
  // store warps publish chunk indices (SPB = 3: two warps, even / odd chunks): rows stored
  auto read_stored = [&]() -> int {
    int a, unused;
    prog_read(from_t, a, unused);
    if constexpr (C::SPB == 3) {
      int b;
      prog_read(from_t + 8, b, unused);
      a = min(a, b);
    }
    return min(n, C::CH * a);
  };
  uint64_t cur = 0ull;
  int curv = 0;  // lane j < CE: S' of the border entry of row CE*Q+1+j (the current block)
  // band 0's border (score column 0 or a strip halo) holds the true S: S'(r, 0) = S(r, 0) + r p
  const bool conv_in = SRC == kSrcPlain || (SRC == kSrcGlobal && band == 0);
  // HALO_OUT: S(r, c_last) = S'(r, c_last) - (r + c_last) p, c_last = c0 + ws - 1
  const int out_adj = HALO_OUT ? (c0 + ws - 1 + 1 - out_lane) * p : 0;  // + s p = (r + c_last) p at step s
  int vlast = Pv[K - 1];
  const uint32_t laneR = opaque(g.refR + 16u * (K / 4) * t), laneS = opaque(g.scR + 16u * (K / 4) * t);
  auto load_prof_row = [&](int a) {  // SEQ: this lane's K profile values for residue a
    const uint32_t a0 = profA + (static_cast<uint32_t>(a) << (7 + (K == 8 ? 3 : 2)));  // + a * 32 lanes * 4K bytes
    const int4 u = lds128_tok<0>(a0, tok);
    rvn[0] = u.x, rvn[1] = u.y, rvn[2] = u.z, rvn[3] = u.w;
    if constexpr (K == 8) {
      const int4 v = lds128_tok<0>(a0 ^ 16u, tok);
      rvn[4] = v.x, rvn[5] = v.y, rvn[6] = v.z, rvn[7] = v.w;
    }
  };
  auto load_ref_row = [&](uint32_t a) {  // K/4 LDS.128 of this lane's K ref values
    const int4 u = lds128_tok<0>(a, tok);
    rvn[0] = u.x, rvn[1] = u.y, rvn[2] = u.z, rvn[3] = u.w;
    if constexpr (K == 8) {
      const int4 v = lds128_tok<16>(a, tok);
      rvn[4] = v.x, rvn[5] = v.y, rvn[6] = v.z, rvn[7] = v.w;
    }
  };

  // one wavefront step s (entry jj of the block's border window); ALL = every lane's row is in
  // 1..n (no predicates)
  constexpr int kPfAt = NW_PF_AT;  // mid-block work (border copy, progress pre-read) this many steps into the block
  static_assert(kPfAt >= 0 && kPfAt < CE, "mid-block point");
  // step of the block at which the staging progress is pre-read (A/B: late for the K = 8 kernel,
  // early for the K = 4 kernels, whose two-band CTA measured 235 vs 204 GCUPS at 4 vs 14)
  constexpr int kPreAt = K == 8 ? NW_PRE_AT : NW_PRE_AT4;
  static_assert(kPreAt >= 0 && kPreAt < CE, "pre-read point");
  // the staging warps' progress words for the NEXT event, read kPfAt steps into the block
  // (the result is first used at that event; cached values that already suffice are kept)
  int cur_sig0 = 0;
  auto pre_read = [&]() {
    const int nl = SEQ ? 0 : min(n, cur_sig0 + 2 * CE + 1), ns = cur_sig0 + 2 * CE - SR;
    if (landed < nl) {
      int unused;
      prog_read(from_r, landed, unused);
    }
    if (stored < ns) stored = read_stored();
  };
  int vprev = 0;  // the out lane's previous row value (paired border-entry stores)
  int vbuf[8];    // steady blocks: the out lane's last 8 row values, published as 4 pairs per 8 steps
  auto step = [&](const int s, auto jj_tag, auto all_tag) {
    constexpr int jj = decltype(jj_tag)::value;  // step within the block (an immediate)
    constexpr bool ALL = decltype(all_tag)::value;
    const int r = s + 1 - t;  // this lane's row
    // ---- ref of this step's row (loaded last step) and the next row's loads
    int rv[K];
    if constexpr (SEQ) {
      // the profile row of row r was loaded last step; load row r+1's now (its residue was
      // fetched two steps ago) and fetch row r+3's residue
#pragma unroll
      for (int m = 0; m < K; ++m) rv[m] = rvn[m];
      load_prof_row(a_cur);
      a_cur = a_nxt;
      a_nxt = __ldg(A + min(max(r + 2, 0), n - 1)) & 31;  // residue of row r+3
    } else {
      // ref' = ref + 2p (the diagonal move of the gap-normalised recurrence); off the
      // recurrence's critical path (the row was loaded one step ahead)
#pragma unroll
      for (int m = 0; m < K; ++m) rv[m] = rvn[m] + P.p2;
      if constexpr (!(ALL && (NW_STEP_EXP & 4))) load_ref_row(laneR + static_cast<uint32_t>(r & (RR - 1)) * RS4);  // ring row of row r+1
    }
    // ---- left value: lane t-1's last column of this row, lane 0: the border entry
    const int bval = (ALL && (NW_STEP_EXP & 8)) ? curv + jj : __shfl_sync(FULL, curv, jj);
    const int from_left = (ALL && (NW_STEP_EXP & 128)) ? vlast + 1 : __shfl_up_sync(FULL, vlast, 1);
    if constexpr (jj == kPreAt) pre_read();  // (its acquire load waits in the shuffles' shadow)
    const int L = (ALL && (NW_STEP_EXP & 16)) ? from_left + bval : (t == 0) ? bval : from_left;
    bool active = true;
    if (!ALL) active = r >= 1 && r <= n;
    if (active) {
      // gap-normalised cell: S'(r,j) = max(S'(r-1,j-1) + ref'(r,j), S'(r-1,j), S'(r,j-1))
      // x_m = max(diag + ref', up); the row's left chain is a plain prefix max and the left
      // value L enters with one max per cell.
      int x[K];
      if constexpr (ALL && (NW_STEP_EXP & 32)) {
#pragma unroll
        for (int m = 0; m < K; ++m) x[m] = 0;
      }
      x[0] = __viaddmax_s32(Lprev, rv[0], Pv[0]);
#pragma unroll
      for (int m = 1; m < K; ++m) x[m] = __viaddmax_s32(Pv[m - 1], rv[m], Pv[m]);
      // (written as a sequential chain: ptxas schedules it better than a hand-built max3 tree;
      // scripts/ubench_sp.cu V=2 vs V=0: 80 vs 94 cycles per K = 8 step)
      int Y[K];
      Y[0] = x[0];
#pragma unroll
      for (int m = 1; m < K; ++m) Y[m] = max(Y[m - 1], x[m]);
#pragma unroll
      for (int m = 0; m < K; ++m) Pv[m] = max(L, Y[m]);
      if constexpr (ALL && (NW_STEP_EXP & 32)) {  // (timing only) no recurrence chain: each cell independent
#pragma unroll
        for (int m = 0; m < K; ++m) Pv[m] = __viaddmax_s32(Pv[m], rv[m], L);
      }
      if constexpr (ALL && (NW_STEP_EXP & 64)) {  // (timing only) chain-free L path: S'_7 = max(L + 0, Y_7)
        Pv[K - 1] = __viaddmax_s32(L, P.zero0, Y[K - 1]);
      }
      Lprev = L;
      const uint32_t aS = laneS + static_cast<uint32_t>((r - 1) & (SR - 1)) * RS4;
      [&]<int... I>(std::integer_sequence<int, I...>) {
        if constexpr (!(ALL && (NW_STEP_EXP & 2))) (sts128_ring<16 * I>(aS, Pv[4 * I], Pv[4 * I + 1], Pv[4 * I + 2], Pv[4 * I + 3]), ...);
      }(std::make_integer_sequence<int, K / 4>{});
      int vo = Pv[K - 1];
      if constexpr (RAGGED) {
#pragma unroll
        for (int m = 0; m < K - 1; ++m) vo = out_m == m ? Pv[m] : vo;
      }
      if constexpr (HALO_OUT) vo -= out_adj + s * p;
      if constexpr (ALL && (NW_STEP_EXP & 1)) {
      } else if constexpr (!RAGGED && kPairs && ALL) {
        // steady block (every row in 1..n, full band: the out lane is lane 31 at row r = s - 30):
        // the out lane's values are buffered and published as four 16-byte pairs at the end of
        // each 8-step half (rows r-7 .. r, r-7 even); one store per step held a register quad
        // that the next step's store rewrote (ncu: long-scoreboard stalls behind the LSU queue)
        vbuf[jj & 7] = vo;
        if constexpr ((jj & 7) == 7) {
#pragma unroll
          for (int k = 0; k < 4; ++k) {
            const int r0 = r - 7 + 2 * k;
            const uint32_t u0 = static_cast<uint32_t>(r0);
            if constexpr (REMOTE)
              st_pair_dsmem_p(do_out && sink_smem, bring_out + 8u * (r0 & (C::BR - 1)), static_cast<uint32_t>(vbuf[2 * k]), gen | u0,
                              static_cast<uint32_t>(vbuf[2 * k + 1]), gen | (u0 + 1));
            else
              st_pair_smem_p(do_out && sink_smem, bring_out + 8u * (r0 & (C::BR - 1)), static_cast<uint32_t>(vbuf[2 * k]), gen | u0,
                             static_cast<uint32_t>(vbuf[2 * k + 1]), gen | (u0 + 1));
            if constexpr (HALO_OUT)
              st_pair_sys_p(do_out, lout + r0, static_cast<uint32_t>(vbuf[2 * k]), lout_tag, static_cast<uint32_t>(vbuf[2 * k + 1]), lout_tag);
            else
              st_pair_gpu_p(do_out && sink_gpu, lout + r0, static_cast<uint32_t>(vbuf[2 * k]), lout_tag, static_cast<uint32_t>(vbuf[2 * k + 1]),
                            lout_tag);
          }
        }
        vprev = vo;
      } else if constexpr (!RAGGED && kPairs) {
        // full band: the out lane is lane 31, so its row r = s - 30 has the parity of J.  Odd
        // rows publish the pair (r-1, r) in one 16-byte store; an even last row is flushed alone.
        constexpr bool ODD = (jj & 1) != 0;
        const uint32_t ur = static_cast<uint32_t>(r);
        if constexpr (ODD) {
          if constexpr (REMOTE)
            st_pair_dsmem_p(do_out && sink_smem, bring_out + 8u * ((r - 1) & (C::BR - 1)), static_cast<uint32_t>(vprev), gen | (ur - 1),
                            static_cast<uint32_t>(vo), gen | ur);
          else
            st_pair_smem_p(do_out && sink_smem, bring_out + 8u * ((r - 1) & (C::BR - 1)), static_cast<uint32_t>(vprev), gen | (ur - 1),
                           static_cast<uint32_t>(vo), gen | ur);
          if constexpr (HALO_OUT)
            st_pair_sys_p(do_out, lout + (r - 1), static_cast<uint32_t>(vprev), lout_tag, static_cast<uint32_t>(vo), lout_tag);
          else
            st_pair_gpu_p(do_out && sink_gpu, lout + (r - 1), static_cast<uint32_t>(vprev), lout_tag, static_cast<uint32_t>(vo), lout_tag);
        } else if constexpr (!ALL) {
          const bool fl = do_out && r == n;
          if constexpr (REMOTE)
            st_pair_dsmem_p(fl && sink_smem, bring_out + 8u * (r & (C::BR - 1)), static_cast<uint32_t>(vo), gen | ur, static_cast<uint32_t>(vo),
                            gen | (ur + 1));
          else
            st_pair_smem_p(fl && sink_smem, bring_out + 8u * (r & (C::BR - 1)), static_cast<uint32_t>(vo), gen | ur, static_cast<uint32_t>(vo),
                           gen | (ur + 1));
          if constexpr (HALO_OUT)
            st_pair_sys_p(fl, lout + r, static_cast<uint32_t>(vo), lout_tag, static_cast<uint32_t>(vo), lout_tag);
          else
            st_pair_gpu_p(fl && sink_gpu, lout + r, static_cast<uint32_t>(vo), lout_tag, static_cast<uint32_t>(vo), lout_tag);
        }
        vprev = vo;
      } else {
        if constexpr (REMOTE)
          st_entry_dsmem_p(do_out && sink_smem, bring_out + 8u * (r & (C::BR - 1)), static_cast<uint32_t>(vo), gen | static_cast<uint32_t>(r));
        else
          st_entry_smem_p(do_out && sink_smem, bring_out + 8u * (r & (C::BR - 1)), static_cast<uint32_t>(vo), gen | static_cast<uint32_t>(r));
        if constexpr (HALO_OUT)
          st_entry_sys_p(do_out, lout + r, static_cast<uint32_t>(vo), lout_tag);
        else
          st_entry_gpu_p(do_out && sink_gpu, lout + r, static_cast<uint32_t>(vo), lout_tag);
      }
    }
    vlast = Pv[K - 1];
  };

  const int nsteps = n + 31;  // compute steps 0 .. n+30
  const int nblk = (nsteps + CE - 1) / CE;
  for (int Q = 0; Q < nblk; ++Q) {
    const int sig0 = Q * CE;
    cur_sig0 = sig0;
    // ---- event Q.  To the staging warp: ref rows <= sig0-30 consumed (lane 31 read row sig0-30
    // at step sig0-1), score rows <= sig0-31 complete (lane 31 wrote row sig0-31 at step sig0-1).
    const long long ce0 = tracing ? clock64() : 0;
    // release after __syncwarp: every lane's ring writes (score) and reads (ref) of the earlier
    // steps happen before the staging warps' acquire of this word
    prog_publish(to_s, max(0, sig0 - 30), max(0, sig0 - 31), !strict);
    if (tracing) pub_cyc += clock64() - ce0;
    {
      // this block reads ref rows <= sig0+CE+1 and rewrites score slots of rows <= sig0+CE
      const int need_l = SEQ ? 0 : min(n, sig0 + CE + 1), need_s = sig0 + CE - SR;
      // one direct read of each stale progress word first (the staging warps normally run ahead:
      // the timed spin below is the exception, and its timer reads are not free)
      if (landed < need_l || stored < need_s) {
        int unused;
        if (landed < need_l) prog_read(from_r, landed, unused);
        if (stored < need_s) stored = read_stored();
      }
      if (landed < need_l || stored < need_s) {
        const bool landed_short = !(landed < need_l);  // (trace) waiting on the store warp only
        const long long c0c = clock64();
        const uint64_t tw = globaltimer_ns();
        unsigned spins = 0;
        int unused;
        for (;;) {
          if (landed < need_l) prog_read(from_r, landed, unused);
          if (stored < need_s) stored = read_stored();
          if (landed >= need_l && stored >= need_s) break;
          if ((++spins & 255u) == 0 && globaltimer_ns() - tw > P.spin_limit_ns) watchdog_trap(P.err);
        }
        wait_cyc += clock64() - c0c;
        if (landed_short) st_wait_cyc += clock64() - c0c;
      }
    }
    const long long ce1 = tracing ? clock64() : 0;
    if constexpr (SRC == kSrcSmem) {
      cur = e1;
      if (sig0 + CE < nsteps) e1 = load_block(Q + 1);
      if (t == 0) sts32_volatile(prog_in, sig0);  // rows <= sig0 consumed (block Q-1 validated)
    } else if (SRC == kSrcGlobal && BD == 1 && NW_BORDER_REG) {
      cur = e1;  // the polled producer column: loaded into registers at the previous mid-block
    } else {
      // block Q's copy is in the prologue's group (Q < BD) or in the one committed at the half
      // point of block Q-BD; the groups committed after it may still be in flight
      const int newer = min(Q, BD - 1);
      if (newer == 0)
        cp_async_wait<0>();
      else if (newer == 1)
        cp_async_wait<1>();
      else
        cp_async_wait<2>();
      __syncwarp();  // landed by lanes 0..CE-1, visible to the warp
      cur = read_block(Q);
    }
    if constexpr (SRC != kSrcPlain) {
      // the whole block must be published before its first step (a row-by-row re-poll at the
      // producer's frontier costs one round trip per row: measured slower)
      if (leading_valid(cur, Q) < CE) {
        const long long c0c = clock64();
        const uint64_t tw = globaltimer_ns();
        unsigned spins = 0;
        do {
          cur = load_block(Q);
          if ((++spins & 255u) == 0 && globaltimer_ns() - tw > P.spin_limit_ns) watchdog_trap(P.err);
        } while (leading_valid(cur, Q) < CE);
        spin_cyc += clock64() - c0c;
      }
    }
    curv = static_cast<int>(static_cast<uint32_t>(cur));
    if (conv_in) curv += (CE * Q + 1 + t) * p;
    const long long ce2 = tracing ? clock64() : 0;
    if (sink_smem) {
      // rows written in this block are <= sig0+CE; the slot of row x held row x-BR
      const int need = sig0 + CE - C::BR;
      auto read_bp = [&]() -> int { return REMOTE ? ld_dsmem_b32(prog_out) : lds32_volatile(prog_out); };
      if (need > bp_cache && need > (bp_cache = read_bp())) {
        const long long c0c = clock64();
        const uint64_t tw = globaltimer_ns();
        while (need > (bp_cache = read_bp()))
          if (globaltimer_ns() - tw > P.spin_limit_ns) watchdog_trap(P.err);
        bp_cyc += clock64() - c0c;
      }
    }
    asm volatile("mov.u32 %0, 0;" : "=r"(tok)::"memory");  // the block's ref loads stay below
    if constexpr (!SEQ) {
      if (Q == 0) load_ref_row(laneR + static_cast<uint32_t>((-t) & (RR - 1)) * RS4);  // row 1-t
    } else {
      if (Q == 0) load_prof_row(A[min(max(-t, 0), n - 1)] & 31);  // row 1-t
    }
    if (tracing) {
      const long long ce3 = clock64();
      ph_cyc[0] += ce1 - ce0, ph_cyc[1] += ce2 - ce1, ph_cyc[2] += ce3 - ce2;
    }
    // ---- CE steps, fully unrolled (the border entry index jj is an immediate), in two parts
    // around the mid-block work at step kPfAt: the border copy of block Q + BD (global / plain
    // sources) and a read of the staging warps' progress words for the NEXT event, whose result
    // is consumed only there (its latency hides behind the second part's steps instead of
    // stalling the event; measured ~200 cycles per event when read at the event itself)
    auto mid_block = [&]() {
      if constexpr (SRC == kSrcGlobal && NW_BORDER_REG) {
        if (BD == 1) {
          // a polled producer column: the next block's entries straight into registers (lanes
          // 0..CE-1, relaxed 8-byte loads, first used at the next event) -- no copy to wait for,
          // no shared-memory round trip at the event
          if (sig0 + CE < nsteps) e1 = load_block(Q + 1);
          return;
        }
      }
      if constexpr (SRC != kSrcSmem) {
        // a fresher snapshot of the producer's column than at the event (less band-to-band lag);
        // later than the half point the L2 round trip is exposed at the event
        if (sig0 + CE * BD < nsteps) prefetch_block(Q + BD);
        cp_async_commit();
      }
    };
    auto block_steps = [&](auto all_tag) {
      [&]<int... J>(std::integer_sequence<int, J...>) {
        (step(sig0 + J, std::integral_constant<int, J>{}, all_tag), ...);
      }(std::make_integer_sequence<int, kPfAt>{});
      mid_block();
      [&]<int... J>(std::integer_sequence<int, J...>) {
        (step(sig0 + kPfAt + J, std::integral_constant<int, kPfAt + J>{}, all_tag), ...);
      }(std::make_integer_sequence<int, CE - kPfAt>{});
    };
    if (sig0 >= 31 && sig0 + CE <= n) {
      const long long c0c = tracing ? clock64() : 0;
      block_steps(std::true_type{});
      if (tracing) steady_cyc += clock64() - c0c, ++steady_blocks;
    } else {
      block_steps(std::false_type{});
    }
  }
  prog_publish(to_s, n, n, !strict);  // every row consumed and complete
  if (tracing && t == 0 && task < P.trace_cap) {
    unsigned smid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    unsigned long long* e = P.trace + 8 * task;
    e[0] = static_cast<unsigned long long>(task);
    e[1] = t_task0;
    e[2] = globaltimer_ns();
    e[3] = smid;
    e[4] = static_cast<unsigned long long>(steady_cyc) | (static_cast<unsigned long long>(steady_blocks) << 44);
    if (kTrace && P.trace2 != nullptr)
      for (int k = 0; k < 3; ++k) P.trace2[8 * task + k] = static_cast<unsigned long long>(ph_cyc[k]);
    if (P.trace2 != nullptr) P.trace2[8 * task + 3] = static_cast<unsigned long long>(st_wait_cyc);
    if (P.trace2 != nullptr) P.trace2[8 * task + 6] = static_cast<unsigned long long>(pub_cyc);
    e[5] = static_cast<unsigned long long>(bp_cyc);
    e[6] = static_cast<unsigned long long>(spin_cyc);
    e[7] = static_cast<unsigned long long>(wait_cyc);
  }
}

template <class C>
__global__ void __launch_bounds__(32 * C::NWARPS, 1) nw_wave_kernel(const __grid_constant__ StripParams P) {
  constexpr int NW = C::NW;
  extern __shared__ __align__(128) unsigned char smem[];
  const int t = threadIdx.x & 31;
  // warps 0..NW-1 compute; SPB = 1: NW..2NW-1 ref + store staging; SPB = 2: NW..2NW-1 ref,
  // 2NW..3NW-1 store staging
  const int wa = threadIdx.x >> 5;
  const bool staging = wa >= NW;
  int role = wa < NW ? 0 : (C::SPB == 1 ? (kRoleRef | kRoleStore) : (wa < 2 * NW ? kRoleRef : kRoleStore));
  const int half = C::SPB == 3 && wa >= 2 * NW ? (wa >= 3 * NW ? 1 : 0) : -1;  // SPB = 3: even / odd score chunks
  if (C::SPREAD && wa >= 2 * NW) role = wa >= 6 ? kRoleStore : kRoleIdle;
  const int w = wa % NW;  // the band slot this warp serves
  // CTA header: [0] group ticket, [8 + 4w] consumer progress of warp w, [128..] border rings
  unsigned long long* const s_group = reinterpret_cast<unsigned long long*>(smem);
  const uint32_t s_prog = smem_u32(smem + 8);
  unsigned char* const wsm = smem + C::kCtaHdr + w * C::kWarpSmem;
  // shared border rings start invalid (tag 0xFFFFFFFF never equals gen | row, row < 2^30)
  for (int i = threadIdx.x; i < (C::CL > 1 ? 1 : NW - 1) * C::BR; i += 32 * C::NWARPS) reinterpret_cast<unsigned long long*>(smem + 128)[i] = ~0ull;
  if (threadIdx.x < NW) sts32_volatile(s_prog + 4 * threadIdx.x, 0);
  if (!staging && t == 0) {  // band progress words
    st_release_cta_v2(smem_u32(wsm), 0u, 0u);
    st_release_cta_v2(smem_u32(wsm) + 8, 0u, 0u);
    st_release_cta_v2(smem_u32(wsm) + 16, 0u, 0u);
    st_release_cta_v2(smem_u32(wsm) + 24, C::SPB == 3 ? 1u : 0x3fffffffu, 0u);  // odd-chunk store warp: next chunk 1
  }
  __syncthreads();

  int gcount = 0;  // groups processed by this CTA (generation of the shared border tags)
  const uint32_t crank = C::CL > 1 ? cluster_ctarank() : 0u;
  if constexpr (C::CL > 1) cluster_sync_all();  // every CTA's rings initialised before any remote store
  for (;;) {
    long long group;
    if constexpr (C::CL > 1) {
      // one ticket per cluster (rank 0 draws it); the cluster takes CL consecutive bands
      if (crank == 0 && threadIdx.x == 0) *s_group = atomicAdd(P.ticket, 1ull);
      cluster_sync_all();
      unsigned long long tk;
      asm volatile("ld.relaxed.cluster.shared::cluster.b64 %0, [%1];" : "=l"(tk) : "r"(mapa_u32(smem_u32(s_group), 0)) : "memory");
      cluster_sync_all();  // every CTA read the ticket before rank 0 may draw the next one
      group = static_cast<long long>(tk - P.ticket_base);
    } else {
      if (threadIdx.x == 0) *s_group = atomicAdd(P.ticket, 1ull);
      __syncthreads();
      group = static_cast<long long>(*s_group - P.ticket_base);
    }
    if (group < 0 || group >= P.ngroups) break;  // (< 0: a stale ticket base; never draw a negative task)
    // pair mode (many independent pairs, NW = 1): a ticket is a whole pair and the CTA sweeps its
    // bands one after the other -- band k's border column is already complete when it starts
    // (no band-to-band pipeline fill, no polling)
    const int nsub = P.pair_mode ? P.nbands : 1;
    for (int sub = 0; sub < nsub; ++sub) {
    const long long task = P.pair_mode ? group * P.nbands + sub : (C::CL > 1 ? group * C::CL + crank : group * NW + w);
    const uint32_t gen = static_cast<uint32_t>(gcount & 3) << 30;
    if (task < P.ntasks) {
      const int band = static_cast<int>(task % P.nbands);
      const bool full = band_ws(P.width, band, C::W) == C::W;
      if (role == kRoleIdle) {
      } else if (C::SPB == 1 && staging) {
        if (full)
          wave_stage<C, false, kRoleRef | kRoleStore>(P, task, t, wsm);
        else
          wave_stage<C, true, kRoleRef | kRoleStore>(P, task, t, wsm);
      } else if (role == kRoleRef) {
        if (full)
          wave_stage<C, false, kRoleRef>(P, task, t, wsm);
        else
          wave_stage<C, true, kRoleRef>(P, task, t, wsm);
      } else if (role == kRoleStore) {
        if (full)
          wave_stage<C, false, kRoleStore>(P, task, t, wsm, half);
        else
          wave_stage<C, true, kRoleStore>(P, task, t, wsm, half);
      } else {
        const bool last_band = band == P.nbands - 1;
        // position of the band in its group: the previous / next band of the group is in this CTA
        // (NW > 1: warps w -1 / w + 1) or, with clusters, in the previous / next CTA
        const int jpos = C::CL > 1 ? static_cast<int>(crank) : w, jlast = C::CL > 1 ? C::CL - 1 : NW - 1;
        int sink;
        if (last_band)
          sink = P.halo_out ? kSinkGlobal : kSinkNone;
        else
          sink = (jpos < jlast) ? kSinkSmem : kSinkGlobal;
        const int src = band == 0 ? (P.halo_in ? kSrcGlobal : kSrcPlain) : (jpos > 0 ? kSrcSmem : kSrcGlobal);
        const bool halo_out = last_band && P.halo_out;  // validated: such a band is full width
        if (C::CL > 1 && sink == kSinkSmem) {
          if (!full) __trap();  // (unreachable: only the last band of a pair can be ragged)
          if (src == kSrcGlobal)
            wave_band<C, false, kSrcGlobal, false, true>(P, task, w, t, smem, wsm, gen, sink);
          else if (src == kSrcSmem)
            wave_band<C, false, kSrcSmem, false, true>(P, task, w, t, smem, wsm, gen, sink);
          else
            wave_band<C, false, kSrcPlain, false, true>(P, task, w, t, smem, wsm, gen, sink);
        } else if (halo_out) {
          if (src == kSrcGlobal)
            wave_band<C, false, kSrcGlobal, true>(P, task, w, t, smem, wsm, gen, sink);
          else if (src == kSrcSmem)
            wave_band<C, false, kSrcSmem, true>(P, task, w, t, smem, wsm, gen, sink);
          else
            wave_band<C, false, kSrcPlain, true>(P, task, w, t, smem, wsm, gen, sink);
        } else if (full) {
          if (src == kSrcGlobal)
            wave_band<C, false, kSrcGlobal, false>(P, task, w, t, smem, wsm, gen, sink);
          else if (src == kSrcSmem)
            wave_band<C, false, kSrcSmem, false>(P, task, w, t, smem, wsm, gen, sink);
          else
            wave_band<C, false, kSrcPlain, false>(P, task, w, t, smem, wsm, gen, sink);
        } else {
          if (src == kSrcGlobal)
            wave_band<C, true, kSrcGlobal, false>(P, task, w, t, smem, wsm, gen, sink);
          else if (src == kSrcSmem)
            wave_band<C, true, kSrcSmem, false>(P, task, w, t, smem, wsm, gen, sink);
          else
            wave_band<C, true, kSrcPlain, false>(P, task, w, t, smem, wsm, gen, sink);
        }
      }
    }
    __syncthreads();  // group end: every warp done (shared rings / progress words reusable)
    if (threadIdx.x < NW) sts32_volatile(s_prog + 4 * threadIdx.x, 0);
    if (!staging && t == 0) {
      st_release_cta_v2(smem_u32(wsm), 0u, 0u);
      st_release_cta_v2(smem_u32(wsm) + 8, 0u, 0u);
      st_release_cta_v2(smem_u32(wsm) + 16, 0u, 0u);
    st_release_cta_v2(smem_u32(wsm) + 24, C::SPB == 3 ? 1u : 0x3fffffffu, 0u);  // odd-chunk store warp: next chunk 1
    }
    __syncthreads();
    ++gcount;
    }
  }
}

}  // namespace nwb200
