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
//   * Staging: ref rows are fetched CH at a time with cp.async.bulk (one row per lane, mbarrier
//     transaction count) LOOK chunks ahead into a per-warp shared ring; finished score rows are
//     written from a per-warp ring with cp.async.bulk stores (16-byte aligned interior) plus
//     scalar stores for the <= 3 unaligned head/tail words (the Rodinia pitch n+1 puts every
//     row at a different 16-byte phase, SURVEY §7 hard part 3).  Element x of row r sits at
//     slot(r) + (G(r) & 31) + x, G(r) = global word address of the row's first column: smem and
//     global 16-byte phases agree (bulk copies) and, for an odd pitch, the 32 skewed rows a warp
//     touches fall in 32 different banks.
//   * Band handoff (the paper's "successive anti-diagonals are computed sequentially" and
//     Fig. 9's W ∩ R = ∅): the lane holding a band's last column publishes every row as a
//     64-bit entry {value, tag} — the ready flag fused with the value, one row granularity.
//       - between warps of one CTA: a shared-memory ring (tag = row | gen << 30, 256 entries,
//         back-pressure on the consumer's published progress); the consumer reads the row it
//         needs each step (~30-cycle latency instead of an L2 round trip);
//       - between CTAs / GPUs: a global buffer (tag = launch epoch; relaxed gpu/sys scope),
//         polled 32 rows per load one window ahead; a stale entry is re-polled.
//   * Every spin is bounded by a %globaltimer watchdog: on expiry the kernel records
//     kErrWatchdog and traps, so a broken protocol surfaces as a CUDA error.
#pragma once
#include <cstdint>
#include <type_traits>

#include "nw_ptx.cuh"

namespace nwb200 {

constexpr int kBarBytes = 128;
constexpr int kBR = 256;  // shared border ring entries between consecutive warps of a CTA
constexpr unsigned kErrWatchdog = 0xBADB0001u;

// Geometry of one kernel instance.  Events happen every CH steps (event Q starts step CH*Q).
// In block Q lane t touches rows CH*Q+1-t .. CH*Q+CH-t: chunks Q-SKEW .. Q (the 31-row skew).
template <int K_, bool SEQ_, int NW_, int CH_, int LOOK_>
struct StripCfg {
  static constexpr int K = K_, NW = NW_, CH = CH_, LOOK = LOOK_;
  static constexpr bool SEQ = SEQ_;
  static constexpr int W = 32 * K;   // warp band width (columns)
  static constexpr int RS = W + 36;  // row slot (words): W + 3 head + 3 tail + 28 swizzle, 16B multiple
  static constexpr int SKEW = (31 + CH - 1) / CH;
  static constexpr int REF_SLOTS = LOOK + SKEW + 1;  // ref chunks live at once
  static constexpr int STORE_DELAY = SKEW + 1;       // chunk c complete after step CH*c+CH-1+31
  static constexpr int SC_SLOTS = STORE_DELAY + 1;   // incl. the one being stored
  static constexpr int REF_ROWS = SEQ ? 0 : REF_SLOTS * CH;
  static constexpr int SC_ROWS = SC_SLOTS * CH;
  static constexpr int SEQ_MOD = 2 * REF_SLOTS;      // ref-chunk sequence modulus (slot + parity)
  static constexpr int PROF_WORDS = SEQ ? 32 * 32 : 0;
  static constexpr size_t kWarpSmem = kBarBytes + 4ull * ((size_t)REF_ROWS * RS + (size_t)SC_ROWS * RS + PROF_WORDS);
  static constexpr size_t kCtaHdr = 128 + (size_t)(NW - 1) * kBR * 8;
  static constexpr size_t kSmem = kCtaHdr + NW * kWarpSmem;
  static_assert(32 % CH == 0, "events must align with the 32-row border windows");
  static_assert(RS % 4 == 0 && kWarpSmem % 16 == 0, "16-byte aligned rings for cp.async.bulk");
  static_assert(((size_t)REF_ROWS * RS) % 32 == 0 && ((size_t)SC_ROWS * RS) % 32 == 0, "ring wrap keeps banks");
  static_assert(NW <= 8, "group header holds 8 progress counters");
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
  unsigned long long* trace;  // debug: per task {task, t_start, t_end, smid} (globaltimer ns) or null
  long long trace_cap;
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
enum : int { kSinkNone = 0, kSinkGlobal = 1, kSinkSys = 2, kSinkSmem = 3 };

template <class C>
__global__ void __launch_bounds__(32 * C::NW, 1) nw_strip_kernel(const __grid_constant__ StripParams P) {
  constexpr int K = C::K, RS = C::RS, CH = C::CH, NW = C::NW;
  constexpr bool SEQ = C::SEQ;
  constexpr unsigned FULL = 0xffffffffu;
  extern __shared__ __align__(128) unsigned char smem[];
  const int t = threadIdx.x & 31;
  const int w = threadIdx.x >> 5;
  // CTA header: [0] group ticket, [8 + 4w] consumer progress of warp w, [128..] border rings
  unsigned long long* const s_group = reinterpret_cast<unsigned long long*>(smem);
  const uint32_t s_prog = smem_u32(smem + 8);
  const uint32_t s_bring = smem_u32(smem + 128);
  unsigned char* const wsm = smem + C::kCtaHdr + w * C::kWarpSmem;
  const uint32_t bar0 = smem_u32(wsm);
  int32_t* const ref_ring = reinterpret_cast<int32_t*>(wsm + kBarBytes);
  int32_t* const sc_ring = ref_ring + C::REF_ROWS * RS;
  uint32_t* const prof = reinterpret_cast<uint32_t*>(sc_ring + C::SC_ROWS * RS);

  if (t == 0 && !SEQ) {
    for (int i = 0; i < C::REF_SLOTS; ++i) mbar_init(bar0 + 8 * i, 32);
  }
  fence_mbar_init();
  // shared border rings start invalid (tag 0xFFFFFFFF never equals gen | row, row < 2^30)
  for (int i = threadIdx.x; i < (NW - 1) * kBR; i += 32 * NW)
    reinterpret_cast<unsigned long long*>(smem + 128)[i] = ~0ull;
  if (threadIdx.x < NW) sts32_volatile(s_prog + 4 * threadIdx.x, 0);
  __syncthreads();

  const int n = static_cast<int>(P.n);
  const int nch = (n + CH - 1) / CH;
  const int nsteps = n + 31;
  const int p = P.p;
  const int ldr32 = static_cast<int>(P.ldr & 31), lds32 = static_cast<int>(P.lds & 31);
  int seqm = 0;   // ref-chunk sequence number mod SEQ_MOD (ring slot + mbarrier parity), across tasks
  int gcount = 0; // groups processed by this CTA (generation of the shared border tags)

  for (;;) {
    if (threadIdx.x == 0) *s_group = atomicAdd(P.ticket, 1ull);
    __syncthreads();
    const long long group = static_cast<long long>(*s_group - P.ticket_base);
    if (group >= P.ngroups) break;
    const long long task = group * NW + w;
    const uint32_t gen = static_cast<uint32_t>(gcount & 3) << 30;
    if (task < P.ntasks) {
      const unsigned long long t_task0 = globaltimer_ns();
      const long long c_task0 = clock64();
      const long long pair = task / P.nbands;
      const int band = static_cast<int>(task - pair * P.nbands);
      const bool last_band = band == P.nbands - 1;
      const int c0 = band_c0(band, C::W);
      const int ws = band_ws(P.width, band, C::W);
      int32_t* const S = P.score + pair * P.pss;
      const int32_t* const R = SEQ ? nullptr : P.ref + pair * P.psr;

      // ---- border source (left) and sink (right), uniform per task
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
        lin = P.xbuf + (pair * (P.nbands - 1) + band - 1) * static_cast<long long>(n + 1);
        lin_epoch = P.epoch;
      }
      int sink;
      uint64_t* lout = nullptr;
      uint32_t lout_tag = 0;
      if (last_band) {
        sink = P.halo_out ? (P.halo_out_sys ? kSinkSys : kSinkGlobal) : kSinkNone;
        lout = P.halo_out;
        lout_tag = P.halo_epoch;
      } else if (w < NW - 1) {
        sink = kSinkSmem;  // band+1 is warp w+1 of this CTA
        lout_tag = gen;
      } else {
        sink = kSinkGlobal;
        lout = P.xbuf + (pair * (P.nbands - 1) + band) * static_cast<long long>(n + 1);
        lout_tag = P.epoch;
      }
      const uint32_t bring_in = s_bring + (w - 1) * kBR * 8;   // valid when src == kSrcSmem
      const uint32_t bring_out = s_bring + w * kBR * 8;        // valid when sink == kSinkSmem
      const uint32_t prog_out = s_prog + 4 * (w + 1);          // consumer progress (sink smem)
      const uint32_t prog_in = s_prog + 4 * w;                 // my progress (src smem)
      const int32_t* const colp = S + (c0 - 1);  // plain left border column
      const int out_lane = (ws - 1) / K;
      const int ref_row_base = (seqm % C::REF_SLOTS) * CH;
      const uintptr_t GR0 = SEQ ? 0 : (reinterpret_cast<uintptr_t>(R) >> 2) + c0;  // word addr of (0, c0)
      const uintptr_t GS0 = (reinterpret_cast<uintptr_t>(S) >> 2) + c0;

      auto load_border = [&](int row) -> uint64_t {
        if (row > n) return 0ull;
        if (src == kSrcGlobal) return lin_sys ? ld_relaxed_sys(lin + row) : ld_relaxed_gpu(lin + row);
        return static_cast<uint32_t>(__ldg(colp + static_cast<long long>(row) * P.lds));
      };

      // ref chunk c (rows CH*c+1 .. CH*c+CH): lane t < CH bulk-copies row CH*c+1+t.
      auto issue_ref = [&](int c) {
        const int sl = (seqm + c) % C::REF_SLOTS;
        const uint32_t bar = bar0 + 8 * sl;
        const int r = c * CH + 1 + (t & (CH - 1));
        uint32_t bytes = 0, dst = 0;
        const void* src_p = nullptr;
        if (t < CH && r <= n) {
          const int32_t* g = R + static_cast<long long>(r) * P.ldr + c0;
          const uintptr_t gs = reinterpret_cast<uintptr_t>(g), ge = gs + 4u * ws;
          const uintptr_t s0 = gs & ~static_cast<uintptr_t>(15);
          // never read past the matrix end: the final row of the last band loads its tail scalar
          const bool tail_scalar = (r == n) && last_band;
          const uintptr_t e0 = tail_scalar ? (ge & ~static_cast<uintptr_t>(15)) : ((ge + 15) & ~static_cast<uintptr_t>(15));
          const int gw = static_cast<int>((gs >> 2) & 31);
          int32_t* drow = ref_ring + ((ref_row_base + r - 1) % (C::REF_ROWS ? C::REF_ROWS : 1)) * RS + (gw & ~3);
          if (e0 > s0) {
            bytes = static_cast<uint32_t>(e0 - s0);
            src_p = reinterpret_cast<const void*>(s0);
            dst = smem_u32(drow);
          }
          if (tail_scalar) {
            const int a = gw & 3;
            for (int x = e0 > gs ? static_cast<int>((e0 - gs) >> 2) : 0; x < ws; ++x) drow[a + x] = __ldg(g + x);
          }
        }
        mbar_arrive_expect_tx(bar, bytes);
        if (bytes) bulk_g2s(dst, src_p, bytes, bar);
      };

      // score chunk c: lanes < CH bulk-store the aligned interior of row CH*c+1+t, lanes >= CH
      // (or all lanes for CH < 16, second pass) store the unaligned head/tail words.
      auto store_sc = [&](int c) {
        const int r = c * CH + 1 + (t % CH);
        if (r > n) return;
        int32_t* g = S + static_cast<long long>(r) * P.lds + c0;
        const uintptr_t gs = reinterpret_cast<uintptr_t>(g), ge = gs + 4u * ws;
        const uintptr_t as = (gs + 15) & ~static_cast<uintptr_t>(15), ae = ge & ~static_cast<uintptr_t>(15);
        const int32_t* srow = sc_ring + ((r - 1) % C::SC_ROWS) * RS + static_cast<int>((gs >> 2) & 31);
        if (t < CH) {
          if (ae > as) bulk_s2g(reinterpret_cast<void*>(as), smem_u32(srow) + static_cast<uint32_t>(as - gs),
                                static_cast<uint32_t>(ae - as));
        }
        if (t >= 32 - CH) {
          const int xh = ae > as ? static_cast<int>((as - gs) >> 2) : ws;
          for (int x = 0; x < xh; ++x) g[x] = srow[x];
          if (ae > as)
            for (int x = static_cast<int>((ae - gs) >> 2); x < ws; ++x) g[x] = srow[x];
        }
      };

      // ---- prologue: top border (row 0 is input), left-border window, first ref chunks
      int Pv[K];
#pragma unroll
      for (int m = 0; m < K; ++m) Pv[m] = (t * K + m < ws) ? __ldg(S + c0 + t * K + m) : 0;
      int Lprev = (t * K < ws) ? __ldg(S + c0 + t * K - 1) : 0;  // diag input of the first row
      int vlast = Pv[K - 1];
      uint64_t cur = 0, nxt = 0;
      if (src != kSrcSmem) {
        cur = load_border(1 + t);
        nxt = load_border(33 + t);
      }
      int win_base = 1;  // cur holds border rows win_base + t
      // true when every row of the window is published (or beyond n): no per-step tag checks
      auto window_valid = [&]() -> bool {
        if (src != kSrcGlobal) return true;
        return __all_sync(FULL, static_cast<uint32_t>(cur >> 32) == lin_epoch || win_base + t > n) != 0;
      };
      bool wvalid = window_valid();
      // per-lane 32-bit shared byte addresses of this lane's first column in its current row
      const int r0 = 1 - t;
      int gR = static_cast<int>((GR0 + static_cast<uintptr_t>(static_cast<intptr_t>(r0) * P.ldr)) & 31);
      int gS = static_cast<int>((GS0 + static_cast<uintptr_t>(static_cast<intptr_t>(r0) * P.lds)) & 31);
      const uint32_t refR0 = opaque(smem_u32(ref_ring)), refR1 = opaque(refR0 + 4u * C::REF_ROWS * RS);
      const uint32_t scR0 = opaque(smem_u32(sc_ring)), scR1 = opaque(scR0 + 4u * C::SC_ROWS * RS);
      uint32_t aR = refR0 + 4u * ((C::REF_ROWS ? (((ref_row_base + r0 - 1) % C::REF_ROWS + C::REF_ROWS) % C::REF_ROWS) : 0) * RS +
                                  gR + t * K);
      uint32_t aS = scR0 + 4u * ((((r0 - 1) % C::SC_ROWS + C::SC_ROWS) % C::SC_ROWS) * RS + gS + t * K);
      const uint32_t stepR = 4u * (RS + ldr32), stepS = 4u * (RS + lds32);
      // right-border publish: generic running pointer (global) or shared ring slot
      const bool do_out = sink != kSinkNone && t == out_lane;
      uint64_t* gout = lout != nullptr ? lout + r0 : nullptr;
      uint32_t sout_hi = lout_tag + (sink == kSinkSmem ? static_cast<uint32_t>(r0) : 0u);
      const uint32_t sout_inc = sink == kSinkSmem ? 1u : 0u;
      fence_proxy_async();
      __syncwarp();
      if constexpr (!SEQ) {
        for (int c = 0; c < C::LOOK && c < nch; ++c) issue_ref(c);
      }
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
      const bool tracing = P.trace != nullptr;
      long long ev_cyc = 0, spin_cyc = 0, wait_cyc = 0;  // debug cycle accounting (trace only)

      // one wavefront step; ALL = every lane's row is in 1..n (steady state, no predicates)
      auto step = [&](const int sig, auto all_tag, auto src_tag) {
        constexpr bool ALL = decltype(all_tag)::value;
        constexpr bool SMEMSRC = decltype(src_tag)::value;
        // loads first (addresses known from the previous step)
        int rv[K];
        if constexpr (SEQ) {
          const uint32_t pw = profp[32 * a0];
#pragma unroll
          for (int m = 0; m < K; ++m) rv[m] = prmt_sext(pw, 0x8880u + 0x1111u * m);  // sign-extended byte m
        } else {
#pragma unroll
          for (int m = 0; m < K; ++m) rv[m] = lds_tok(aR + 4 * m, tok);
        }
        int bval;
        if constexpr (SMEMSRC) {
          // the row this step needs (lane 0: row sig+1) from warp w-1's shared ring
          uint64_t be = lds64_volatile(bring_in + 8u * ((sig + 1) & (kBR - 1)));
          const uint32_t want = gen | static_cast<uint32_t>(sig + 1);
          if (static_cast<uint32_t>(be >> 32) != want && sig < n) {
            const long long c_0 = clock64();
            const uint64_t t0 = globaltimer_ns();
            do {
              be = lds64_volatile(bring_in + 8u * ((sig + 1) & (kBR - 1)));
              if (globaltimer_ns() - t0 > P.spin_limit_ns) watchdog_trap(P.err);
            } while (static_cast<uint32_t>(be >> 32) != want);
            spin_cyc += clock64() - c_0;
          }
          bval = static_cast<int>(static_cast<uint32_t>(be));
        } else {
          const int idx = sig & 31;
          bval = __shfl_sync(FULL, static_cast<int>(static_cast<uint32_t>(cur)), idx);
          if (!wvalid) {
            uint32_t bep = __shfl_sync(FULL, static_cast<uint32_t>(cur >> 32), idx);
            if (bep != lin_epoch && sig < n) {  // left band has not published row sig+1 yet
              const long long c_0 = clock64();
              const int rowb = win_base + t;
              const uint64_t t0 = globaltimer_ns();
              for (;;) {
                cur = load_border(rowb);
                bep = __shfl_sync(FULL, static_cast<uint32_t>(cur >> 32), idx);
                if (bep == lin_epoch) break;
                if (globaltimer_ns() - t0 > P.spin_limit_ns) watchdog_trap(P.err);
              }
              bval = __shfl_sync(FULL, static_cast<int>(static_cast<uint32_t>(cur)), idx);
              wvalid = window_valid();
              spin_cyc += clock64() - c_0;
            }
          }
        }
        const int from_left = __shfl_up_sync(FULL, vlast, 1);
        const int L = (t == 0) ? bval : from_left;
        bool active = true;
        if (!ALL) {
          const int r = lane_row(sig, t);
          active = r >= 1 && r <= n;
        }
        if (active) {
          int d = Lprev, l = L;
#pragma unroll
          for (int m = 0; m < K; ++m) {
            const int x = __viaddmax_s32(Pv[m], -p, d + rv[m]);  // max(up - p, diag + ref)
            const int v = __viaddmax_s32(l, -p, x);              // max(left - p, .)
            d = Pv[m];
            Pv[m] = v;
            l = v;
          }
          Lprev = L;
#pragma unroll
          for (int m = 0; m < K; ++m) sts_s32(aS + 4 * m, Pv[m]);
          // publish the band's last column (lane out_lane holds it in Pv[K-1]; every band with
          // a right neighbour is full width)
          const uint32_t vo = static_cast<uint32_t>(Pv[K - 1]);
          if (sink == kSinkSmem) {
            st_entry_smem(do_out, bring_out + 8u * (static_cast<uint32_t>(sout_hi) & (kBR - 1)), vo, sout_hi);
          } else if (sink == kSinkGlobal) {
            st_entry_gpu(do_out, gout, vo, lout_tag);
          } else if (sink == kSinkSys) {
            st_entry_sys(do_out, gout, vo, lout_tag);
          }
        }
        vlast = Pv[K - 1];
        // advance this lane to row r+1
        if constexpr (SEQ) {
          a0 = a1;
          a1 = __ldg(A + min(max(lane_row(sig, t) + 1, 0), n - 1)) & 31;  // residue of row r+2
        } else {
          aR += stepR;  // next row slot + swizzle advance (G(r+1) = G(r) + ld)
          gR += ldr32;
          if (gR >= 32) {
            gR -= 32;
            aR -= 128;
          }
          if (aR >= refR1) aR -= refR1 - refR0;
        }
        aS += stepS;
        gS += lds32;
        if (gS >= 32) {
          gS -= 32;
          aS -= 128;
        }
        if (aS >= scR1) aS -= scR1 - scR0;
        ++gout;
        sout_hi += sout_inc;
      };

      auto run_block = [&](const int sig0, auto src_tag) {
        if (sig0 >= 31 && sig0 + CH <= n) {  // steady state: all 32 lanes on rows 1..n
#pragma unroll
          for (int j = 0; j < CH; ++j) step(sig0 + j, std::true_type{}, src_tag);
        } else {
#pragma unroll 1
          for (int j = 0; j < CH; ++j) {
            if (sig0 + j >= nsteps) break;
            step(sig0 + j, std::false_type{}, src_tag);
          }
        }
      };

      for (int Q = 0; Q <= nch + C::STORE_DELAY - 1; ++Q) {
        const int sig0 = Q * CH;
        const long long c_ev0 = tracing ? clock64() : 0;
        // ---- chunk events (warp-uniform)
        bulk_wait_read<0>();  // stores issued at earlier events have read their slots
        __syncwarp();
        if (Q >= C::STORE_DELAY && Q - C::STORE_DELAY < nch) {
          fence_proxy_async();  // this lane's STS of rows in the finished chunk -> async proxy
          __syncwarp();
          store_sc(Q - C::STORE_DELAY);
        }
        bulk_commit();
        if constexpr (!SEQ) {
          if (Q + C::LOOK < nch) {
            fence_proxy_async();
            __syncwarp();
            issue_ref(Q + C::LOOK);
          }
          const long long c_w0 = tracing ? clock64() : 0;
          if (Q < nch) tok = mbar_wait_tok(bar0 + 8 * ((seqm + Q) % C::REF_SLOTS), ((seqm + Q) / C::REF_SLOTS) & 1);
          if (tracing) wait_cyc += clock64() - c_w0;
        }
        if (sig0 >= nsteps) continue;
        if (src == kSrcSmem) {
          // publish my consumed frontier (rows <= sig0), throttle my own shared ring producer
          if (t == 0) sts32_volatile(prog_in, sig0);
        } else if ((sig0 & 31) == 0 && sig0 > 0) {
          cur = nxt;
          win_base = sig0 + 1;
          nxt = load_border(sig0 + 33 + t);
          wvalid = window_valid();
        }
        if (sink == kSinkSmem) {
          // back-pressure: rows written in this block are <= sig0+CH-31; their ring slots must
          // hold rows the consumer (warp w+1) already consumed
          const int rmax = sig0 + CH - 31;
          if (rmax - kBR > 0 && rmax - kBR > lds32_volatile(prog_out)) {
            const uint64_t t0 = globaltimer_ns();
            while (rmax - kBR > lds32_volatile(prog_out)) {
              if (globaltimer_ns() - t0 > P.spin_limit_ns) watchdog_trap(P.err);
            }
          }
        }
        if (tracing) ev_cyc += clock64() - c_ev0;
        if (src == kSrcSmem)
          run_block(sig0, std::true_type{});
        else
          run_block(sig0, std::false_type{});
      }
      bulk_wait_all<0>();
      __syncwarp();
      if (!SEQ) seqm = (seqm + nch) % C::SEQ_MOD;
      if (P.trace != nullptr && t == 0 && task < P.trace_cap) {
        unsigned smid;
        asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
        unsigned long long* e = P.trace + 8 * task;
        e[0] = static_cast<unsigned long long>(task);
        e[1] = t_task0;
        e[2] = globaltimer_ns();
        e[3] = smid;
        e[4] = static_cast<unsigned long long>(ev_cyc);    // cycles in chunk events (incl. ref wait)
        e[5] = static_cast<unsigned long long>(wait_cyc);  // of which: ref mbarrier waits
        e[6] = static_cast<unsigned long long>(spin_cyc);  // cycles spinning on the left border
        e[7] = static_cast<unsigned long long>(clock64() - c_task0);
      }
    }
    __syncthreads();  // group end: every warp done (shared border rings / progress reusable)
    if (t == 0) sts32_volatile(s_prog + 4 * w, 0);  // ordered before the next group by its barrier
    ++gcount;
  }
}

}  // namespace nwb200
