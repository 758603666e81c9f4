// nw_strip.cuh — the persistent NW wavefront kernel for sm_100a.
//
// What it computes (Fig. 2, with Rodinia's cell function, R1):
//     score[i][j] = max(score[i-1][j-1] + ref[i][j], score[i-1][j] - p, score[i][j-1] - p)
// for every interior cell, each value written ONCE, in place, into score (the short-circuited
// update of P:512-516 / P:616-656: no temporary, no copy).
//
// How (B200 design; the paper's per-diagonal kernels are prior art, see nw_diag.cuh):
//   * Columns are cut into tile-column bands of W = 32*K columns (P:487-501's tiles stacked
//     into a column; the "a CTA owns a band" lever of SURVEY §7).  A CTA of NW warps claims a
//     GROUP of NW consecutive bands through one atomic ticket; warp w sweeps band
//     group*NW + w from row 1 to row n.  Tickets enumerate (pair, band) in wavefront order and
//     band k waits only on band k-1 — held by the same CTA or by a CTA that claimed earlier —
//     so there is no deadlock without co-residency (a 1-CTA grid is tested).
//   * Intra-band wavefront: lane t owns K adjacent columns; at step s it computes row s+1-t
//     (the intra-tile anti-diagonals of P:498-501, skewed one row per lane).  The left value
//     arrives from lane t-1 by one warp shuffle per step; each cell is two DPX VIADDMNMX.
//   * Inside a band the paper's Rvert / Rhoriz slices never touch memory: the row
//     above is in registers, the left column arrives by shuffle.
//   * Staging (per warp, 64-row shared rings, events every CH steps): ref rows arrive by
//     16-byte cp.async (LDGSTS, whole warp, completion on an mbarrier) LOOK chunks ahead;
//     finished score rows leave by LDS.128 + STG.128 (16-byte aligned interior) plus scalar
//     stores for the <= 3 unaligned head/tail words — the Rodinia pitch n+1 puts every row at a
//     different 16-byte phase (SURVEY §7 hard part 3).  Element x of row r sits at
//     ring((r-1) & 63) + (G(r) & 31) + x, G(r) = global word address of the row's first
//     column: smem and global 16-byte phases agree and, for an odd pitch, the 32 skewed rows a
//     warp touches fall in 32 different banks.  (Per-row cp.async.bulk copies
//     were measured first: ~64 small copies per SM per event serialise in the TMA unit.)
//   * Band handoff (the paper's "successive anti-diagonals are computed sequentially" and
//     Fig. 9's W ∩ R = ∅): the lane holding a band's last column publishes every row as a
//     64-bit entry {value, tag} — the ready flag fused with the value, one row granularity.
//       - between warps of one CTA: a shared-memory ring (tag = gen << 30 | row, 256 entries,
//         back-pressure on the consumer's published progress);
//       - between CTAs / GPUs: a global buffer (tag = launch epoch; relaxed gpu/sys scope).
//     The consumer keeps a 32-row window of entries in registers and, once per CH-step block,
//     checks (one vote) that the block's rows are published, re-polling if not; the steps
//     themselves are branch free.
//   * Every spin is bounded by a %globaltimer watchdog: on expiry the kernel records
//     kErrWatchdog and traps, so a broken protocol surfaces as a CUDA error.
#pragma once
#include <cstdint>
#include <type_traits>

#include "nw_ptx.cuh"

namespace nwb200 {

// per band pair header: ev mbarriers [0,128), progress word [128], global-sink staging ring
// [256,512), border prefetch ring [512,1280)
constexpr int kBarBytes = 2048;
constexpr int kHdrEv = 0, kHdrState = 128, kHdrGstage = 256, kHdrBpre = 512;
constexpr int kBR = 256;      // shared border ring entries between consecutive warps of a CTA
constexpr int kNEv = 16;      // event mbarrier slots (compute leads staging by <= 2 events)
constexpr int kPF = 4;        // ref chunks prefetched into L2 beyond the smem lookahead
constexpr unsigned kErrWatchdog = 0xBADB0001u;

// Geometry of one kernel instance.  Events happen every CH steps (event Q starts step CH*Q).
// In block Q lane t touches rows CH*Q+1-t .. CH*Q+CH-t: chunks Q-SKEW .. Q (the 31-row skew).
template <int K_, bool SEQ_, int NW_, int CH_, int RR_, int SR_>
struct StripCfg {
  static constexpr int K = K_, NW = NW_, CH = CH_;
  static constexpr bool SEQ = SEQ_;
  static constexpr int W = 32 * K;   // warp band width (columns)
  static constexpr int RS = W + 36;  // row slot (words): W + 3 head + 3 tail + 28 swizzle, 16B multiple
  static constexpr int SKEW = (31 + CH - 1) / CH;
  static constexpr int RR = SEQ ? CH : RR_;           // ref ring rows
  static constexpr int SR = SR_;                      // score ring rows
  static constexpr int REF_SLOTS = RR / CH;           // ref chunks per ring
  static constexpr int SLOTS = SR / CH;               // score chunks per ring
  static constexpr int STORE_DELAY = SKEW + 1;        // chunk c complete after step CH*c+CH-1+31
  static constexpr int LOOKW = REF_SLOTS - SKEW - 1;  // ref chunks the staging warp runs ahead
  static constexpr int MAXR = W / 4 + 2;              // 16-byte chunks of a ref row superset
  static constexpr int MAXS = W / 4;                  // 16-byte chunks of a score row interior
  static constexpr int ITER_R = (CH * MAXR + 31) / 32;
  static constexpr int ITER_S = (CH * MAXS + 31) / 32;
  static constexpr int REF_ROWS = SEQ ? 0 : RR;
  static constexpr int PROF_WORDS = SEQ ? 32 * 32 : 0;
  static constexpr size_t kWarpSmem = kBarBytes + 4ull * ((size_t)REF_ROWS * RS + (size_t)SR * RS + PROF_WORDS);
  static constexpr size_t kCtaHdr = 128 + (size_t)(NW - 1) * kBR * 8;
  static constexpr size_t kSmem = kCtaHdr + NW * kWarpSmem;
  static_assert(32 % CH == 0 && CH <= 16, "events must align with the 32-row border windows");
  static_assert(RR % CH == 0 && SR % CH == 0, "rings hold whole chunks");
  static_assert(SEQ || LOOKW >= 1, "ref ring too small for any lookahead");
  static_assert(SLOTS >= STORE_DELAY + 1, "score ring too small for the store delay");
  static_assert(RS % 4 == 0 && kWarpSmem % 16 == 0, "16-byte aligned rings");
  static_assert(((size_t)RR * RS) % 32 == 0 && ((size_t)SR * RS) % 32 == 0, "ring wrap keeps banks");
  static_assert(NW <= 8, "header space");
  static_assert(2 * CH * 8 <= 256 && 4 * (CH + 2) * 8 <= 768, "per-band header regions");
};

// ---- the schedule (shared by the kernel and the host export nw_strip_map, pin P7) --------
// Band k of a pair covers columns [band_c0, band_c0 + band_ws); at wavefront step s lane t
// computes row lane_row(s, t) (if 1 <= row <= n), columns band_c0 + t*K .. + K - 1 (clipped).
__host__ __device__ __forceinline__ int band_c0(int band, int W) { return 1 + band * W; }
__host__ __device__ __forceinline__ int band_ws(long long width, int band, int W) {
  const long long r = width - static_cast<long long>(band) * W;
  return static_cast<int>(r < W ? r : W);
}
__host__ __device__ __forceinline__ int lane_row(int step, int lane) { return step + 1 - lane; }
// entries per band-border slot in the global border buffer: >= n+2 (16-byte pair reads may touch
// row n+1) and even (every slot starts 16-byte aligned)
__host__ __device__ __forceinline__ long long xstride(long long n) { return (n + 3) & ~1ll; }

struct StripParams {
  int32_t* score;
  int64_t lds, pss;  // pitch, pair stride (elements)
  const int32_t* ref;
  int64_t ldr, psr;
  int64_t n;       // rows 1..n
  int64_t width;   // interior columns 1..width
  int32_t p;
  int32_t nbands;  // bands per pair
  int64_t ntasks;  // pairs * nbands
  int64_t ngroups; // ceil(ntasks / NW)
  uint64_t* xbuf;  // [pairs][nbands-1][n+1] epoch-tagged right borders (inter-CTA handoffs)
  uint32_t epoch;  // tag of this launch (xbuf)
  const uint64_t* halo_in;  // left border of band 0 (sharded rank > 0) or null (use score col 0)
  uint64_t* halo_out;       // right border of the last band (sharded, peer) or null
  uint32_t halo_epoch;
  int32_t halo_out_sys;
  unsigned long long* ticket;
  unsigned long long ticket_base;
  unsigned int* err;
  unsigned long long spin_limit_ns;
  unsigned long long* trace;  // debug: per task 8 x u64 (see nw.h nw_debug_set_trace) or null
  long long trace_cap;
  unsigned long long* trace2;  // debug: per task {store cycles, ref-issue cycles} or null
  unsigned int dbg_skip;       // timing experiments only (results invalid when nonzero)
  unsigned int stage_sleep_ns; // staging-warp back-off when idle (NW_STAGE_SLEEP_NS, default below)
  // NEXT-2 (SEQ kernels): ref[i][j] = subst[a[i-1]][b[j-1]] generated on chip
  const uint8_t* seq_a;
  const uint8_t* seq_b;
  int64_t psa, psb;  // pair strides of a / b (bytes)
  int8_t subst[32 * 32];
};

__device__ __forceinline__ int prmt_sext(uint32_t w, uint32_t sel) {
  uint32_t d;
  asm("prmt.b32 %0, %1, 0, %2;" : "=r"(d) : "r"(w), "r"(sel));
  return static_cast<int>(d);
}
// opaque copy: keeps a value in a register (stops the compiler re-deriving smem bases per step)
__device__ __forceinline__ uint32_t opaque(uint32_t x) {
  asm volatile("mov.b32 %0, %0;" : "+r"(x));
  return x;
}
// ref-ring load: not volatile (the compiler may hoist it inside a staging block for ILP), but it
// consumes the token produced after the chunk's mbarrier wait, so it never moves above it
__device__ __forceinline__ int lds_tok(uint32_t a, uint32_t tok) {
  int v;
  asm("ld.shared.b32 %0, [%1];" : "=r"(v) : "r"(a), "r"(tok));
  return v;
}
__device__ __forceinline__ uint32_t mbar_wait_tok(uint32_t bar, uint32_t parity) {
  mbar_wait(bar, parity);
  uint32_t tk;
  asm volatile("mov.u32 %0, 0;" : "=r"(tk)::"memory");
  return tk;
}
__device__ __forceinline__ uint64_t lds64_volatile(uint32_t a) {
  uint64_t v;
  asm volatile("ld.volatile.shared.b64 %0, [%1];" : "=l"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ int lds32_volatile(uint32_t a) {
  int v;
  asm volatile("ld.volatile.shared.b32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ void sts32_volatile(uint32_t a, int v) {
  asm volatile("st.volatile.shared.b32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
// predicated border-entry publishes (no branch in the step)
__device__ __forceinline__ void st_entry_smem(bool pred, uint32_t a, uint32_t lo, uint32_t hi) {
  asm volatile("{ .reg .pred q; .reg .b64 e; setp.ne.b32 q, %0, 0; mov.b64 e, {%2, %3}; @q st.volatile.shared.b64 [%1], e; }" ::"r"(
                   static_cast<int>(pred)),
               "r"(a), "r"(lo), "r"(hi)
               : "memory");
}
__device__ __forceinline__ void st_entry_gpu(bool pred, uint64_t* p, uint32_t lo, uint32_t hi) {
  asm volatile("{ .reg .pred q; .reg .b64 e; setp.ne.b32 q, %0, 0; mov.b64 e, {%2, %3}; @q st.relaxed.gpu.global.b64 [%1], e; }" ::"r"(
                   static_cast<int>(pred)),
               "l"(p), "r"(lo), "r"(hi)
               : "memory");
}
__device__ __forceinline__ void st_entry_sys(bool pred, uint64_t* p, uint32_t lo, uint32_t hi) {
  asm volatile("{ .reg .pred q; .reg .b64 e; setp.ne.b32 q, %0, 0; mov.b64 e, {%2, %3}; @q st.relaxed.sys.global.b64 [%1], e; }" ::"r"(
                   static_cast<int>(pred)),
               "l"(p), "r"(lo), "r"(hi)
               : "memory");
}

__device__ __noinline__ void watchdog_trap(unsigned int* err) {
  atomicExch(err, kErrWatchdog);
  __trap();
}

// Border sources/sinks of one band (uniform per task)
enum : int { kSrcPlain = 0, kSrcGlobal = 1, kSrcSmem = 2 };
enum : int { kSinkNone = 0, kSinkSmem = 1, kSinkGlobal = 2 };

// One band (task) of the persistent kernel; SINK is specialised so the steady-state step has no
// branches.
template <class C>
__device__ __forceinline__ void nw_band(const StripParams& P, const long long task, const int w, const int t,
                                        unsigned char* const smem, unsigned char* const wsm, const uint32_t gen,
                                        uint32_t& cbase, const int SINK) {
  constexpr int K = C::K, RS = C::RS, CH = C::CH;
  constexpr bool SEQ = C::SEQ;
  constexpr unsigned FULL = 0xffffffffu;
  const unsigned long long t_task0 = globaltimer_ns();
  const long long c_task0 = clock64();
  const bool tracing = P.trace != nullptr;
  long long ev_cyc = 0, spin_cyc = 0, wait_cyc = 0;  // debug cycle accounting (trace only)
  long long blk_cyc = 0;                              // steady-state step blocks
  long long ph_cyc[5] = {0, 0, 0, 0, 0};              // event sub-phases (trace only)

  const uint32_t s_prog = smem_u32(smem + 8);
  const uint32_t s_bring = smem_u32(smem + 128);
  const uint32_t bar_ev = smem_u32(wsm) + kHdrEv, s_state = smem_u32(wsm) + kHdrState;
  int32_t* const ref_ring = reinterpret_cast<int32_t*>(wsm + kBarBytes);
  int32_t* const sc_ring = ref_ring + C::REF_ROWS * RS;
  uint32_t* const prof = reinterpret_cast<uint32_t*>(sc_ring + C::SR * RS);

  const int n = static_cast<int>(P.n);
  const int nch = (n + CH - 1) / CH;
  const int nsteps = n + 31;
  const int p = P.p;
  const long long pair = task / P.nbands;
  const int band = static_cast<int>(task - pair * P.nbands);
  const bool last_band = band == P.nbands - 1;
  const int c0 = band_c0(band, C::W);
  const int ws = band_ws(P.width, band, C::W);
  int32_t* const S = P.score + pair * P.pss;
  const int32_t* const R = SEQ ? nullptr : P.ref + pair * P.psr;

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
    src = kSrcSmem;  // band-1 is warp w-1 of this CTA
  } else {
    src = kSrcGlobal;
    lin = P.xbuf + (pair * (P.nbands - 1) + band - 1) * xstride(n);
    lin_epoch = P.epoch;
  }
  // ---- sink (right)
  uint64_t* lout = nullptr;
  uint32_t lout_tag = 0;
  bool lout_sys = false;
  if (SINK == kSinkGlobal) {
    if (last_band) {
      lout = P.halo_out;
      lout_tag = P.halo_epoch;
      lout_sys = P.halo_out_sys != 0;
    } else {
      lout = P.xbuf + (pair * (P.nbands - 1) + band) * xstride(n);
      lout_tag = P.epoch;
    }
  } else if (SINK == kSinkSmem) {
    lout_tag = gen;
  }
  const uint32_t bring_in = s_bring + (w - 1) * kBR * 8;   // src == kSrcSmem
  const uint32_t bring_out = s_bring + w * kBR * 8;        // SINK == kSinkSmem
  const uint32_t prog_out = s_prog + 4 * (w + 1);          // consumer's progress (SINK smem)
  const uint32_t prog_in = s_prog + 4 * w;                 // my progress (src smem)
  const int32_t* const colp = S + (c0 - 1);                // plain left border column
  const int out_lane = (ws - 1) / K;
  const uintptr_t GR0 = SEQ ? 0 : (reinterpret_cast<uintptr_t>(R) >> 2) + c0;  // word addr of (0, c0)
  const uintptr_t GS0 = (reinterpret_cast<uintptr_t>(S) >> 2) + c0;
  const uintptr_t rend =
      SEQ ? 0 : reinterpret_cast<uintptr_t>(R + static_cast<long long>(n) * P.ldr + P.width + 1);  // past the last element
  const uint32_t refR0 = opaque(smem_u32(ref_ring));
  const uint32_t scR0 = opaque(smem_u32(sc_ring));

  auto load_entry = [&](int row) -> uint64_t {
    if (row > n) return 0ull;
    if (src == kSrcGlobal) return lin_sys ? ld_relaxed_sys(lin + row) : ld_relaxed_gpu(lin + row);
    if (src == kSrcSmem) return lds64_volatile(bring_in + 8u * (row & (kBR - 1)));
    return static_cast<uint32_t>(__ldg(colp + static_cast<long long>(row) * P.lds));
  };
  auto entry_ok = [&](uint64_t e, int row) -> bool {
    const uint32_t hi = static_cast<uint32_t>(e >> 32);
    if (src == kSrcGlobal) return hi == lin_epoch;
    if (src == kSrcSmem) return hi == (gen | static_cast<uint32_t>(row));
    return true;
  };

  // ---- prologue: top border (row 0 is input), left-border window, first ref chunks
  int Pv[K];
#pragma unroll
  for (int m = 0; m < K; ++m) Pv[m] = (t * K + m < ws) ? __ldg(S + c0 + t * K + m) : 0;
  int Lprev = (t * K < ws) ? __ldg(S + c0 + t * K - 1) : 0;  // diag input of the first row
  int vlast = Pv[K - 1];
  // left border, per CH-row block: lane j < CH holds the entry of row sig0+1+j (`cur`).
  // Global / plain sources are prefetched D blocks ahead by cp.async into a 4-block shared ring
  // (no register scoreboard on the in-flight loads); a shared-ring source (warp w-1) is read
  // directly at the event.  Ring slot of block q: entries of rows CH*q .. CH*q+CH+1.
  constexpr int D = 2;
  constexpr uint32_t kSlotB = 8u * (CH + 2);
  const uint32_t bpre = smem_u32(wsm) + kHdrBpre;
  auto prefetch_block = [&](int q) {  // block q = rows CH*q+1 .. CH*q+CH
    const uint32_t slot = bpre + kSlotB * static_cast<uint32_t>(q & 3);
    if (src == kSrcGlobal) {
      // 16-byte pairs (rows 2k, 2k+1) through L2 only (entries are polled: never via L1)
      const int row = CH * q + 2 * t;
      cp_async16_cg_p(t <= CH / 2 && row <= n, slot + 16u * t, lin + row);
    } else if (src == kSrcPlain) {
      const int row = CH * q + 1 + t;
      cp_async4_p(t < CH && row <= n, slot + 8u * (1 + t), colp + static_cast<long long>(row) * P.lds);
    }
    cp_async_commit();
  };
  uint64_t cur = 0ull;
  if (src != kSrcSmem)
    for (int q = 0; q < D; ++q) prefetch_block(q);
  // per-lane ring addressing: row r (= step + 1 - t) lives at ring row (r-1) & 63
  const int r0 = 1 - t;
  int rowR = (((r0 - 1) % C::RR) + C::RR) % C::RR;  // ring rows of this lane's current row
  int rowS = (((r0 - 1) % C::SR) + C::SR) % C::SR;
  int gR = static_cast<int>((GR0 + static_cast<uintptr_t>(static_cast<intptr_t>(r0) * P.ldr)) & 31);
  int gS = static_cast<int>((GS0 + static_cast<uintptr_t>(static_cast<intptr_t>(r0) * P.lds)) & 31);
  const int ldr32 = static_cast<int>(P.ldr & 31), lds32 = static_cast<int>(P.lds & 31);
  const uint32_t laneR = refR0 + 4u * t * K, laneS = scR0 + 4u * t * K;
  // right-border publish (lane out_lane holds the band's last column in Pv[K-1]; every band
  // with a right neighbour is full width)
  const bool do_out = t == out_lane && SINK != kSinkNone;
  uint32_t sout_hi = (SINK == kSinkSmem ? lout_tag : 0u) + static_cast<uint32_t>(r0);  // tag | row (row for global)
  const uint32_t gstage = smem_u32(wsm) + kHdrGstage;  // [2*CH] x 8 bytes: global-sink entries awaiting publish
  const uint32_t out_base = SINK == kSinkSmem ? bring_out : gstage;
  const uint32_t out_mask = SINK == kSinkSmem ? kBR - 1 : 2 * CH - 1;
  // SEQ: per-band substitution profile prof[x][t] = pack_m subst[x][b[c0-1+tK+m]] (int8 x K)
  const uint8_t* const A = SEQ ? P.seq_a + pair * P.psa : nullptr;
  int a0 = 0, a1 = 0;  // residues of this lane's current and next row (software pipeline)
  if constexpr (SEQ) {
    const uint8_t* const Bq = P.seq_b + pair * P.psb;
    int bj[K];
#pragma unroll
    for (int m = 0; m < K; ++m) bj[m] = (t * K + m < ws) ? (Bq[c0 - 1 + t * K + m] & 31) : 0;
    for (int x = 0; x < 32; ++x) {
      uint32_t wv = 0;
#pragma unroll
      for (int m = 0; m < K; ++m)
        wv |= static_cast<uint32_t>(static_cast<uint8_t>(P.subst[x * 32 + bj[m]])) << (8 * m);
      prof[x * 32 + t] = wv;
    }
    a0 = A[min(max(r0 - 1, 0), n - 1)] & 31;
    a1 = A[min(max(r0, 0), n - 1)] & 31;
    __syncwarp();
  }
  const uint32_t* const profp = prof + t;
  uint32_t tok = 0;  // produced by each chunk's mbarrier wait, consumed by the ref loads
  uint64_t st_cache = 0;  // last staging progress word read (acquired) by this warp
  int bp_cache = 0;       // last consumer progress read (back-pressure)
  int negp[K];       // -(m+1) p
#pragma unroll
  for (int m = 0; m < K; ++m) negp[m] = -(m + 1) * p;

  // ref values are software-pipelined one step ahead: rvn holds row r's values when step s
  // (row r) starts, and the loads for row r+1 are issued before the step's arithmetic, so the
  // LDS latency hides behind the step's shuffle chain.
  int rvn[K];
  auto load_ref = [&](int out[K], int rr_, int gR_) {
    if constexpr (SEQ) {
      (void)rr_;
      (void)gR_;
    } else {
      const uint32_t aR = laneR + 4u * RS * static_cast<uint32_t>(rr_) + 4u * static_cast<uint32_t>(gR_ & 31);
#pragma unroll
      for (int m = 0; m < K; ++m) out[m] = lds_tok(aR + 4 * m, tok);
    }
  };
  bool rvn_valid = false;  // rvn must be (re)loaded after each chunk event (new token)
#pragma unroll
  for (int m = 0; m < K; ++m) negp[m] = static_cast<int>(opaque(static_cast<uint32_t>(negp[m])));

  // one wavefront step; ALL = every lane's row is in 1..n (steady state, no predicates)
  auto step = [&](const int sig, auto all_tag) {
    constexpr bool ALL = decltype(all_tag)::value;
    const int rowR1 = rowR + 1 == C::RR ? 0 : rowR + 1;  // ring row of the next row
    const uint32_t soff = 4u * RS * static_cast<uint32_t>(rowS);
    int rv[K];
    if constexpr (SEQ) {
      const uint32_t pw = profp[32 * a0];
#pragma unroll
      for (int m = 0; m < K; ++m) rv[m] = prmt_sext(pw, 0x8880u + 0x1111u * m);  // sign-extended byte m
    } else {
      if (!rvn_valid) load_ref(rvn, rowR, gR);
#pragma unroll
      for (int m = 0; m < K; ++m) rv[m] = rvn[m];
      load_ref(rvn, rowR1, gR + ldr32);  // next row (same chunk block or ring-resident)
      rvn_valid = true;
    }
    const int bval = __shfl_sync(FULL, static_cast<int>(static_cast<uint32_t>(cur)), sig & (CH - 1));  // lane 0's left
    const int from_left = __shfl_up_sync(FULL, vlast, 1);
    const int L = (t == 0) ? bval : from_left;
    bool active = true;
    if (!ALL) {
      const int r = lane_row(sig, t);
      active = r >= 1 && r <= n;
    }
    if (active) {
      // Lane-local max-plus prefix form of the K-cell row segment:
      //   x_m = max(up_m - p, diag_m + ref_m),  Y_m = max(Y_{m-1} - p, x_m),
      //   v_m = max(Y_m, L - (m+1) p)  ==  max(x_m, v_{m-1} - p) with v_{-1} = L.
      // x and Y need only the row above, so the left value L (one shuffle away) enters the
      // step's critical path through a single VIADDMNMX per cell.
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
      const uint32_t aS = laneS + soff + 4u * static_cast<uint32_t>(gS & 31);
#pragma unroll
      for (int m = 0; m < K; ++m) sts_s32(aS + 4 * m, Pv[m]);
      // publish the band's last column (lane out_lane, Pv[K-1]): straight into warp w+1's
      // shared ring, or into the local staging ring flushed to global memory at each event
      st_entry_smem(do_out, out_base + 8u * (sout_hi & out_mask), static_cast<uint32_t>(Pv[K - 1]), sout_hi);
    }
    vlast = Pv[K - 1];
    // advance this lane to row r+1
    if constexpr (SEQ) {
      a0 = a1;
      a1 = __ldg(A + min(max(lane_row(sig, t) + 1, 0), n - 1)) & 31;  // residue of row r+2
    }
    rowR = rowR1;
    rowS = rowS + 1 == C::SR ? 0 : rowS + 1;
    gR += ldr32;
    gS += lds32;
    ++sout_hi;
  };

  for (int Q = 0; Q <= nch + C::STORE_DELAY - 1; ++Q) {
    const int sig0 = Q * CH;
    const long long c_ev0 = tracing ? clock64() : 0;
    // ---- chunk events (warp-uniform).  The paired staging warp stores finished score chunks
    // and prefetches ref chunks; this warp only synchronises with it.
    if (Q < nch && !(P.dbg_skip & 2u)) {
      // staging progress: ref chunk Q in shared memory, score chunk Q-SLOTS stored (its slot
      // is about to be rewritten)
      const long long c_w0 = tracing ? clock64() : 0;
      const uint32_t need_rd = cbase + static_cast<uint32_t>(Q) + 1u;
      const uint32_t need_st = Q >= C::SLOTS ? cbase + static_cast<uint32_t>(Q - C::SLOTS) + 1u : 0u;
      auto ok = [&](uint64_t v) {
        return (SEQ || static_cast<int>(static_cast<uint32_t>(v) - need_rd) >= 0) &&
               static_cast<int>(static_cast<uint32_t>(v >> 32) - need_st) >= 0;
      };
      // the last progress word seen usually still covers this event (the staging warp runs
      // LOOKW chunks ahead): re-read it only when it does not
      uint64_t stt = st_cache;
      if (!ok(stt)) stt = ld_acquire_cta(s_state);
      if (!ok(stt)) {
        const uint64_t t0 = globaltimer_ns();
        unsigned spins = 0;
        do {
          stt = ld_acquire_cta(s_state);
          if ((++spins & 1023u) == 0 && globaltimer_ns() - t0 > P.spin_limit_ns) watchdog_trap(P.err);
        } while (!ok(stt));
      }
      st_cache = stt;
      // token (always 0) data-dependent on the acquire: the ref loads cannot move above it
      asm volatile("and.b32 %0, %1, 0;" : "=r"(tok) : "r"(static_cast<uint32_t>(stt)));
      if (tracing) wait_cyc += clock64() - c_w0;
    }
    // event Q reached: score chunk Q-STORE_DELAY is complete, ref chunk Q-SKEW-1 no longer read
    const long long c_p1 = tracing ? clock64() : 0;
    if (tracing) ph_cyc[0] += c_p1 - c_ev0;
    rvn_valid = false;  // rows of the new chunk may be read only after this event's check
    __syncwarp();
    if (t == 0 && !(P.dbg_skip & 4u)) mbar_arrive(bar_ev + 8 * (Q % kNEv));
    const long long c_p2 = tracing ? clock64() : 0;
    if (tracing) ph_cyc[1] += c_p2 - c_p1;
    if (SINK == kSinkGlobal) {
      // publish the rows the out lane finished during block Q-1 (rows CH*(Q-1)+1-out_lane ..
      // CH*Q-out_lane), CH entries at once
      if (Q > 0) {
        const int row = CH * (Q - 1) + 1 - out_lane + t;
        const bool go = t < CH && row >= 1 && row <= n;
        const uint32_t v = go ? static_cast<uint32_t>(lds64_volatile(gstage + 8u * (row & (2 * CH - 1)))) : 0u;
        st_entry_gpu(go && !lout_sys, lout + row, v, lout_tag);
        st_entry_sys(go && lout_sys, lout + row, v, lout_tag);
      }
    }
    if (sig0 >= nsteps) {
      if (tracing) ev_cyc += clock64() - c_ev0;
      continue;
    }
    if (src == kSrcSmem && t == 0) sts32_volatile(prog_in, sig0);  // rows <= sig0 consumed
    if (src == kSrcSmem) {
      cur = t < CH ? lds64_volatile(bring_in + 8u * ((sig0 + 1 + t) & (kBR - 1))) : 0ull;
    } else {
      cp_async_wait<D - 1>();  // block Q's entries landed (one group per block, D in flight)
      __syncwarp();
      cur = t < CH ? lds64_volatile(bpre + kSlotB * static_cast<uint32_t>(Q & 3) + 8u * (1 + t)) : 0ull;
      __syncwarp();
      prefetch_block(Q + D);  // into the slot of block Q+D-4, consumed two events ago
    }
    const long long c_p3 = tracing ? clock64() : 0;
    if (tracing) ph_cyc[2] += c_p3 - c_p2;
    if (src != kSrcPlain && !(P.dbg_skip & 8u)) {
      // the block needs rows sig0+1 .. sig0+CH of the left border (lanes 0 .. CH-1)
      auto ready = [&]() {
        const int row = sig0 + 1 + t;
        const bool need = t < CH && row <= n;
        return __all_sync(FULL, !need || entry_ok(cur, row)) != 0;
      };
      if (!ready()) {
        const long long c_0 = clock64();
        const uint64_t t0 = globaltimer_ns();
        unsigned spins = 0;
        do {
          cur = t < CH ? load_entry(sig0 + 1 + t) : 0ull;  // synchronous re-poll
          if ((++spins & 255u) == 0 && globaltimer_ns() - t0 > P.spin_limit_ns) watchdog_trap(P.err);
        } while (!ready());
        spin_cyc += clock64() - c_0;
      }
    }
    const long long c_p4 = tracing ? clock64() : 0;
    if (tracing) ph_cyc[3] += c_p4 - c_p3;
    if (SINK == kSinkSmem) {
      // back-pressure: rows written in this block are <= sig0+CH-31; their ring slots must hold
      // rows the consumer (warp w+1) already consumed
      const int rmax = sig0 + CH - 31;
      if (rmax - kBR > bp_cache && rmax - kBR > (bp_cache = lds32_volatile(prog_out))) {
        const uint64_t t0 = globaltimer_ns();
        while (rmax - kBR > (bp_cache = lds32_volatile(prog_out)))
          if (globaltimer_ns() - t0 > P.spin_limit_ns) watchdog_trap(P.err);
      }
    }
    if (tracing) {
      const long long c_p5 = clock64();
      ph_cyc[4] += c_p5 - c_p4;
      ev_cyc += c_p5 - c_ev0;
    }
    // ---- CH wavefront steps: lane t computes row sig+1-t, columns c0+tK .. c0+tK+K-1
    if (sig0 >= 31 && sig0 + CH <= n) {  // steady state: all 32 lanes on rows 1..n
      const long long c_b0 = tracing ? clock64() : 0;
      // 4-step unrolled body: keeps the hot loop inside the L0 instruction cache
#pragma unroll 4
      for (int j = 0; j < CH; ++j) step(sig0 + j, std::true_type{});
      if (tracing) blk_cyc += clock64() - c_b0;
    } else {
#pragma unroll 1
      for (int j = 0; j < CH; ++j) {
        if (sig0 + j >= nsteps) break;
        step(sig0 + j, std::false_type{});
      }
    }
  }
  cbase += static_cast<uint32_t>(nch);
  __syncwarp();
  if (P.trace != nullptr && t == 0 && task < P.trace_cap) {
    unsigned smid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    unsigned long long* e = P.trace + 8 * task;
    e[0] = static_cast<unsigned long long>(task);
    e[1] = t_task0;
    e[2] = globaltimer_ns();
    e[3] = (static_cast<unsigned long long>(blk_cyc) << 16) | smid;  // steady-block cycles << 16 | smid
    e[4] = static_cast<unsigned long long>(ev_cyc);    // cycles in chunk events (incl. waits)
    e[5] = static_cast<unsigned long long>(wait_cyc);  // of which: waits on the staging warp
    e[6] = static_cast<unsigned long long>(spin_cyc);  // of which: left-border spins
    e[7] = static_cast<unsigned long long>(clock64() - c_task0);
    if (P.trace2 != nullptr)
      for (int k = 0; k < 5; ++k) P.trace2[8 * task + 2 + k] = static_cast<unsigned long long>(ph_cyc[k]);
  }
}


// The staging warp paired with a compute warp: prefetches ref chunks (LOOKW ahead) and stores
// finished score chunks, driven by the compute warp's per-event mbarrier arrivals.
template <class C>
__device__ __forceinline__ void nw_stage(const StripParams& P, const long long task, const int t,
                                         unsigned char* const wsm, uint32_t& ph_ev, uint32_t& cbase) {
  constexpr int RS = C::RS, CH = C::CH;
  constexpr bool SEQ = C::SEQ;
  const long long c_task0 = clock64();
  long long wait_cyc = 0;
  const uint32_t bar_ev = smem_u32(wsm) + kHdrEv, s_state = smem_u32(wsm) + kHdrState;
  int32_t* const ref_ring = reinterpret_cast<int32_t*>(wsm + kBarBytes);
  int32_t* const sc_ring = ref_ring + C::REF_ROWS * RS;
  const int n = static_cast<int>(P.n);
  const int nch = (n + CH - 1) / CH;
  const long long pair = task / P.nbands;
  const int band = static_cast<int>(task - pair * P.nbands);
  const bool last_band = band == P.nbands - 1;
  const int c0 = band_c0(band, C::W);
  const int ws = band_ws(P.width, band, C::W);
  int32_t* const S = P.score + pair * P.pss;
  const int32_t* const R = SEQ ? nullptr : P.ref + pair * P.psr;
  const uintptr_t GR0 = SEQ ? 0 : (reinterpret_cast<uintptr_t>(R) >> 2) + c0;  // word addr of (0, c0)
  const uintptr_t GS0 = (reinterpret_cast<uintptr_t>(S) >> 2) + c0;
  const uintptr_t rend =
      SEQ ? 0 : reinterpret_cast<uintptr_t>(R + static_cast<long long>(n) * P.ldr + P.width + 1);  // past the last element
  const uint32_t refR0 = opaque(smem_u32(ref_ring));
  const uint32_t scR0 = opaque(smem_u32(sc_ring));

  // Per-lane staging assignments, fixed for the whole task: in iteration it lane t moves the
  // 16-byte chunk k of row i of a CH-row chunk (f = t + 32*it, i = f / MAX, k = f % MAX).  Chunk c
  // is chunk 0 moved by c*CH rows: global addresses by c*CH*ld words, ring rows by c*CH, and the
  // swizzle G & 31 by D_c = c*CH*ld mod 32; with CH a multiple of 4 the 16-byte phase of row i
  // (G & 3) is the same in every chunk, so every per-lane offset below is precomputed once.
  uintptr_t rsrc[C::ITER_R];  // chunk-0 source byte address (16-byte aligned)
  uint32_t rdst[C::ITER_R];   // ring byte offset within a chunk: i*RS*4 + 16k
  int rg[C::ITER_R];          // G(row i of chunk 0) & 31
  bool rok[C::ITER_R];        // (row i, chunk k) exists for a full chunk
  int rrow[C::ITER_R];        // i (row within chunk)
  if constexpr (!SEQ) {
#pragma unroll
    for (int it = 0; it < C::ITER_R; ++it) {
      const int f = t + 32 * it;
      const int i = f / C::MAXR, k = f - (f / C::MAXR) * C::MAXR;
      const uintptr_t G = GR0 + static_cast<uintptr_t>((1 + i) * P.ldr);
      const int a = static_cast<int>(G & 3);
      rsrc[it] = 4u * (G - a) + 16u * k;
      rdst[it] = 4u * (i * RS) + 16u * k;
      rg[it] = static_cast<int>(G & 31);
      rok[it] = i < CH && 4 * k < a + ws;  // chunk k starts inside [G - a, align4(G + ws))
      rrow[it] = i;
    }
  }
  const uintptr_t rstride = 4u * static_cast<uintptr_t>(CH * P.ldr);
  const int rDc = static_cast<int>((CH * P.ldr) & 31);
  const int last_chunk = (n - 1) / CH;

  // ref chunk c (rows CH*c+1 .. CH*c+CH): predicated cp.async (LDGSTS) from precomputed offsets,
  // then every lane arrives on the chunk's mbarrier when its copies have landed.
  auto issue_ref = [&](int c) {
    const uintptr_t cb = static_cast<uintptr_t>(c) * rstride;
    const uint32_t db = refR0 + 4u * ((c * CH) % C::RR) * RS;
    const int Dc = (c * rDc) & 31;
    const int rlim = n - c * CH;  // row i valid iff i < rlim
    if (!(last_band && c == last_chunk)) {
#pragma unroll
      for (int it = 0; it < C::ITER_R; ++it) {
        const uint32_t dst = db + rdst[it] + 4u * ((rg[it] + Dc) & 28);
        cp_async16_p(rok[it] && rrow[it] < rlim, dst, reinterpret_cast<const void*>(rsrc[it] + cb));
      }
    } else {  // the matrix's last rows: never read past the final element
#pragma unroll
      for (int it = 0; it < C::ITER_R; ++it) {
        const uint32_t dst = db + rdst[it] + 4u * ((rg[it] + Dc) & 28);
        const uintptr_t ca = rsrc[it] + cb;
        if (rok[it] && rrow[it] < rlim) {
          if (ca + 16 <= rend) {
            cp_async16(dst, reinterpret_cast<const void*>(ca));
          } else {
            for (int x = 0; x < 4; ++x)
              if (ca + 4u * x < rend) cp_async4(dst + 4u * x, reinterpret_cast<const void*>(ca + 4u * x));
          }
        }
      }
    }
  };

  // score stores, same scheme: interior 16-byte chunks (all LDS.128 first, then STG.128) and
  // the <= 3 unaligned head (lanes 0..CH-1) / tail (lanes CH..2CH-1) words of each row
  uintptr_t sdst[C::ITER_S];  // chunk-0 destination byte address (16-byte aligned)
  uint32_t ssrc[C::ITER_S];   // ring byte offset within a chunk (without the swizzle)
  int sg[C::ITER_S];          // G_S(row i of chunk 0) & 31
  bool sok[C::ITER_S];
  int srow_i[C::ITER_S];
#pragma unroll
  for (int it = 0; it < C::ITER_S; ++it) {
    const int f = t + 32 * it;
    const int i = f / C::MAXS, k = f - (f / C::MAXS) * C::MAXS;
    const uintptr_t G = GS0 + static_cast<uintptr_t>((1 + i) * P.lds);
    const int a = static_cast<int>(G & 3);
    const int h = (4 - a) & 3;                                   // unaligned head words
    const int nint = ws > h ? (ws - h) >> 2 : 0;                 // aligned 16-byte chunks
    sdst[it] = 4u * (G + h) + 16u * k;
    ssrc[it] = 4u * (i * RS + h) + 16u * k;
    sg[it] = static_cast<int>(G & 31);
    sok[it] = i < CH && k < nint;
    srow_i[it] = i;
  }
  // head / tail words of row ht_i = t % CH (lanes < 2CH)
  int ht_x0, ht_x1;
  uintptr_t ht_g;
  int ht_gsw;
  {
    const int i = t % CH;
    const uintptr_t G = GS0 + static_cast<uintptr_t>((1 + i) * P.lds);
    const int a = static_cast<int>(G & 3);
    const int h = min((4 - a) & 3, ws);
    const int nint = ws > h ? (ws - h) >> 2 : 0;
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
  const uintptr_t sstride = 4u * static_cast<uintptr_t>(CH * P.lds);
  const int sDc = static_cast<int>((CH * P.lds) & 31);

  auto store_sc = [&](int c) {
    const uintptr_t cb = static_cast<uintptr_t>(c) * sstride;
    const uint32_t sb = scR0 + 4u * ((c * CH) % C::SR) * RS;
    const int Dc = (c * sDc) & 31;
    const int rlim = n - c * CH;
    int4 v[C::ITER_S];
#pragma unroll
    for (int it = 0; it < C::ITER_S; ++it)
      v[it] = lds128_p(sok[it] && srow_i[it] < rlim, sb + ssrc[it] + 4u * ((sg[it] + Dc) & 31));
#pragma unroll
    for (int it = 0; it < C::ITER_S; ++it)
      stg128_p(sok[it] && srow_i[it] < rlim, reinterpret_cast<void*>(sdst[it] + cb), v[it]);
    // head / tail
    const bool row_ok = (t % CH) < rlim;
    const uint32_t hb = sb + 4u * ((t % CH) * RS + ((ht_gsw + Dc) & 31));
    if (ht_x1 - ht_x0 <= 3) {
      int hv[3];
#pragma unroll
      for (int x = 0; x < 3; ++x) hv[x] = lds32_p(row_ok && ht_x0 + x < ht_x1, hb + 4u * (ht_x0 + x));
#pragma unroll
      for (int x = 0; x < 3; ++x)
        stg32_p(row_ok && ht_x0 + x < ht_x1, reinterpret_cast<void*>(ht_g + cb + 4u * (ht_x0 + x)), hv[x]);
    } else if (row_ok) {  // narrow band (< 16 bytes of aligned interior): every word scalar
      for (int x = ht_x0; x < ht_x1; ++x) stg32_p(true, reinterpret_cast<void*>(ht_g + cb + 4u * x), lds_s32(hb + 4u * x));
    }
  };

  if (P.dbg_skip & 1u) {
    cbase += static_cast<uint32_t>(nch);
    return;
  }
  // progress published to the compute warp: ref chunks < rd are in shared memory, score
  // chunks < sd are stored (absolute chunk numbers, cbase = chunks of earlier tasks)
  uint32_t rd = cbase, sd = cbase;
  if constexpr (!SEQ) {
    for (int c = 0; c < C::LOOKW; ++c) {
      if (c < nch) issue_ref(c);
      cp_async_commit();  // one group per chunk (possibly empty)
    }
    cp_async_wait<C::LOOKW - 1>();  // chunk 0 landed
    rd = cbase + 1;
  }
  __syncwarp();
  if (t == 0) st_release_cta_v2(s_state, rd, sd);
  for (int Q = 0; Q <= nch + C::STORE_DELAY - 1; ++Q) {
    const int sl = Q % kNEv;
    const long long c_w0 = clock64();
    mbar_wait(bar_ev + 8 * sl, (ph_ev >> sl) & 1u);
    ph_ev ^= 1u << sl;
    wait_cyc += clock64() - c_w0;
    if constexpr (!SEQ) {
      if (Q + C::LOOKW < nch) issue_ref(Q + C::LOOKW);
      cp_async_commit();
      // warm L2 with the ref rows kPF chunks further ahead (every 128-byte line of each row)
      const int cp = Q + C::LOOKW + kPF;
      if (cp < nch) {
        constexpr int LINES = (4 * C::W + 8 + 127) / 128 + 1;  // lines touched by one row segment
#pragma unroll
        for (int it = 0; it < (CH * LINES + 31) / 32; ++it) {
          const int f = t + 32 * it;
          const int i = f / LINES, ln = f - (f / LINES) * LINES;
          const int r = cp * CH + 1 + i;
          const uintptr_t g0 = reinterpret_cast<uintptr_t>(R + static_cast<long long>(r) * P.ldr + c0) & ~static_cast<uintptr_t>(127);
          prefetch_l2_p(i < CH && r <= n, reinterpret_cast<const void*>(g0 + 128u * ln));
        }
      }
    }
    if constexpr (!SEQ) {
      cp_async_wait<C::LOOKW - 1>();  // chunks <= Q+1 landed: publish before the stores
      rd = cbase + static_cast<uint32_t>(min(Q + 2, nch));
      __syncwarp();
      if (t == 0) st_release_cta_v2(s_state, rd, sd);
    }
    const int cs = Q - C::STORE_DELAY;
    if (cs >= 0 && cs < nch) {
      store_sc(cs);
      sd = cbase + static_cast<uint32_t>(cs) + 1u;
      __syncwarp();  // every lane's stores of this chunk read their slots
      if (t == 0) st_release_cta_v2(s_state, rd, sd);
    }
  }
  cbase += static_cast<uint32_t>(nch);
  if (P.trace2 != nullptr && t == 0 && task < P.trace_cap) {
    P.trace2[8 * task] = static_cast<unsigned long long>(clock64() - c_task0);
    P.trace2[8 * task + 1] = static_cast<unsigned long long>(wait_cyc);
  }
}

template <class C>
__global__ void __launch_bounds__(64 * C::NW, 1) nw_strip_kernel(const __grid_constant__ StripParams P) {
  constexpr int NW = C::NW;
  extern __shared__ __align__(128) unsigned char smem[];
  const int t = threadIdx.x & 31;
  const int wa = threadIdx.x >> 5;           // 0..NW-1 compute warps, NW..2NW-1 staging warps
  const bool staging = wa >= NW;
  const int w = staging ? wa - NW : wa;      // the band slot this warp serves
  // CTA header: [0] group ticket, [8 + 4w] consumer progress of warp w, [128..] border rings
  unsigned long long* const s_group = reinterpret_cast<unsigned long long*>(smem);
  const uint32_t s_prog = smem_u32(smem + 8);
  unsigned char* const wsm = smem + C::kCtaHdr + w * C::kWarpSmem;
  if (!staging && t == 0) {
    const uint32_t b = smem_u32(wsm);
    for (int i = 0; i < kNEv; ++i) mbar_init(b + kHdrEv + 8 * i, 1);  // ev: the compute warp reached an event
    st_release_cta_v2(b + kHdrState, 0u, 0u);                            // staging progress word
  }
  fence_mbar_init();
  // shared border rings start invalid (tag 0xFFFFFFFF never equals gen | row, row < 2^30)
  for (int i = threadIdx.x; i < (NW - 1) * kBR; i += 64 * NW) reinterpret_cast<unsigned long long*>(smem + 128)[i] = ~0ull;
  if (threadIdx.x < NW) sts32_volatile(s_prog + 4 * threadIdx.x, 0);
  __syncthreads();

  uint32_t ph_a = 0;   // mbarrier phase bits this warp waits on (staging: ev)
  uint32_t cbase = 0;  // chunks of earlier tasks (absolute chunk numbering shared by a warp pair)
  int gcount = 0;               // groups processed by this CTA (generation of the shared border tags)
  for (;;) {
    if (threadIdx.x == 0) *s_group = atomicAdd(P.ticket, 1ull);
    __syncthreads();
    const long long group = static_cast<long long>(*s_group - P.ticket_base);
    if (group >= P.ngroups) break;
    const long long task = group * NW + w;
    const uint32_t gen = static_cast<uint32_t>(gcount & 3) << 30;
    if (task < P.ntasks) {
      if (staging) {
        nw_stage<C>(P, task, t, wsm, ph_a, cbase);
      } else {
        const int band = static_cast<int>(task % P.nbands);
        const bool last_band = band == P.nbands - 1;
        int sink;
        if (last_band)
          sink = P.halo_out ? kSinkGlobal : kSinkNone;
        else
          sink = (w < NW - 1) ? kSinkSmem : kSinkGlobal;
        nw_band<C>(P, task, w, t, smem, wsm, gen, cbase, sink);
      }
    }
    __syncthreads();  // group end: every warp done (shared border rings / progress reusable)
    if (!staging && t == 0) sts32_volatile(s_prog + 4 * w, 0);  // ordered before the next group
    ++gcount;
  }
}

}  // namespace nwb200
