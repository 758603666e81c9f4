// nw_strip.cuh — the persistent NW wavefront kernel for sm_100a.
//
// What it computes (Fig. 2, with Rodinia's cell function, R1):
//     score[i][j] = max(score[i-1][j-1] + ref[i][j], score[i-1][j] - p, score[i][j-1] - p)
// for every interior cell, each value written ONCE, in place, into score (the short-circuited
// update of P:512-516 / P:616-656: no temporary, no copy).
//
// How (B200 design; the paper's per-diagonal kernels are prior art, see nw_diag.cuh):
//   * The n columns are cut into tile-column bands of W = 32*K columns (P:487-501's b x b tiles
//     stacked vertically; the band is the "CTA owns a band" lever of SURVEY §7).  A one-warp
//     CTA claims a band through an atomic ticket (tickets enumerate (pair, band) in wavefront
//     order: band k waits only on band k-1, which a running CTA already holds, so there is no
//     deadlock without co-residency) and sweeps it from row 1 to row n.
//   * Intra-band wavefront: lane t owns K adjacent columns; at step s it computes row s+1-t
//     (the intra-tile anti-diagonals of P:498-501, skewed one row per lane).  The left value
//     arrives from lane t-1 by one warp shuffle per step; the K cells of a lane are a
//     dependent chain of one VIADDMNMX (DPX add+max) each.
//   * Read set of a row segment = its ref (4 B/cell, HBM stream) + the row above (registers)
//     + the left column (shuffle / band handoff): the LMAD slices Rvert / Rhoriz of P:546-566
//     never leave the chip inside a band.
//   * Staging: ref rows are fetched 16 at a time with cp.async.bulk (one row per lane,
//     mbarrier transaction count) two chunks ahead into a 5-chunk shared ring; finished score
//     rows are written from a 4-chunk shared ring with cp.async.bulk stores (16-byte aligned
//     interior) plus scalar stores for the <= 3 unaligned head/tail words (the Rodinia pitch
//     n+1 makes every row start at a different 16-byte phase, SURVEY §7 hard part 3).  Row
//     slots are swizzled ((r>>2)&7)*16 bytes so the per-lane 4-byte shared accesses of 32
//     skewed rows are bank-conflict free.
//   * Band handoff (the paper's "successive anti-diagonals are computed sequentially" +
//     Fig. 9's W ∩ R = ∅ argument): the lane holding the band's last column stores
//     (epoch << 32 | value) for every row into a border buffer; the next band polls 32 rows
//     at a time with relaxed 64-bit loads and re-polls a row whose tag is stale.  The ready
//     flag is fused with the value (one L2 round trip instead of flag + data), and its
//     granularity is one row instead of one tile.
//   * A stale border entry is re-polled under a %globaltimer watchdog: after
//     spin_limit_ns the kernel records kErrWatchdog and traps, so a broken protocol surfaces
//     as a CUDA error instead of a hung GPU.
#pragma once
#include <cstdint>
#include <type_traits>

#include "nw_ptx.cuh"

namespace nwb200 {

// Ring geometry.  Events happen every kCH steps (event Q starts step kCH*Q).  In block Q lane t
// touches rows kCH*Q+1-t .. kCH*Q+kCH-t, i.e. chunks Q-kSkewCh .. Q (the 31-row lane skew).
constexpr int kCH = 16;                              // rows per staging chunk (<= 32, divides 32)
constexpr int kSkewCh = (31 + kCH - 1) / kCH;        // chunks behind the newest one still in use
constexpr int kLook = 2;                             // ref chunks fetched ahead (event Q issues Q+kLook)
constexpr int kRefSlots = kLook + kSkewCh + 1;       // ref chunks live at once
constexpr int kStoreDelay = kSkewCh + 1;             // chunk c complete after step kCH*c+kCH-1+31
constexpr int kScSlots = kStoreDelay + 1;            // score chunks live (incl. the one being stored)
constexpr int kRefRows = kRefSlots * kCH;
constexpr int kScRows = kScSlots * kCH;
constexpr int kSeqMod = 2 * kRefSlots;               // ref-chunk sequence modulus (slot + parity)
static_assert(32 % kCH == 0, "events must align with the 32-row border windows");
constexpr int kBarBytes = 128;
constexpr unsigned kErrWatchdog = 0xBADB0001u;

template <int K, bool SEQ = false>
struct StripGeom {
  static constexpr int W = 32 * K;   // band width (columns)
  static constexpr int RS = W + 36;  // row slot (words): W + 3 head + 3 tail + 28 swizzle, 16B multiple
  static constexpr int kProfWords = 32 * 32;  // SEQ: prof[x][lane] = K packed int8 subst[x][b_j]
  static constexpr size_t kSmem =
      kBarBytes + 4ull * ((SEQ ? 0 : (size_t)kRefRows * RS) + (size_t)kScRows * RS + (SEQ ? kProfWords : 0));
  static_assert(RS % 4 == 0, "row slots must be 16-byte multiples for cp.async.bulk");
  static_assert((kRefRows * RS) % 32 == 0 && (kScRows * RS) % 32 == 0, "ring wrap must keep banks");
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
  uint64_t* xbuf;  // [pairs][nbands-1][n+1] epoch-tagged right borders of bands 0..nbands-2
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

template <int K, bool SEQ>
__global__ void __launch_bounds__(32, 1) nw_strip_kernel(const __grid_constant__ StripParams P) {
  using G = StripGeom<K, SEQ>;
  constexpr int RS = G::RS;
  constexpr unsigned FULL = 0xffffffffu;
  extern __shared__ __align__(128) unsigned char smem[];
  const int t = threadIdx.x;
  const uint32_t bar0 = smem_u32(smem);
  int32_t* const ref_ring = reinterpret_cast<int32_t*>(smem + kBarBytes);
  int32_t* const sc_ring = ref_ring + (SEQ ? 0 : kRefRows * RS);
  uint32_t* const prof = reinterpret_cast<uint32_t*>(sc_ring + kScRows * RS);

  if (t == 0) {
    for (int i = 0; i < kRefSlots; ++i) mbar_init(bar0 + 8 * i, 32);
  }
  fence_mbar_init();
  __syncwarp();

  const int n = static_cast<int>(P.n);
  const int nch = (n + kCH - 1) / kCH;
  const int nsteps = n + 31;
  const int p = P.p;
  int seq10 = 0;  // ref-chunk sequence number mod kSeqMod (ring slot + mbarrier parity), across tasks

  for (;;) {
    unsigned long long tk = 0;
    if (t == 0) tk = atomicAdd(P.ticket, 1ull);
    tk = __shfl_sync(FULL, tk, 0);
    const long long task = static_cast<long long>(tk - P.ticket_base);
    if (task >= P.ntasks) break;
    const unsigned long long t_task0 = globaltimer_ns();
    const long long pair = task / P.nbands;
    const int band = static_cast<int>(task - pair * P.nbands);
    const bool last_band = band == P.nbands - 1;
    const int c0 = band_c0(band, G::W);
    const int ws = band_ws(P.width, band, G::W);
    int32_t* const S = P.score + pair * P.pss;
    const int32_t* const R = P.ref + pair * P.psr;

    const uint64_t* lin;
    bool lin_sys;
    uint32_t lin_epoch;
    if (band > 0) {
      lin = P.xbuf + (pair * (P.nbands - 1) + band - 1) * static_cast<long long>(n + 1);
      lin_sys = false;
      lin_epoch = P.epoch;
    } else {
      lin = P.halo_in;
      lin_sys = true;
      lin_epoch = P.halo_epoch;
    }
    uint64_t* lout;
    bool lout_sys;
    uint32_t lout_epoch;
    if (!last_band) {
      lout = P.xbuf + (pair * (P.nbands - 1) + band) * static_cast<long long>(n + 1);
      lout_sys = false;
      lout_epoch = P.epoch;
    } else {
      lout = P.halo_out;
      lout_sys = P.halo_out_sys != 0;
      lout_epoch = P.halo_epoch;
    }
    const int32_t* const colp = S + (c0 - 1);  // plain left border column (band 0 without halo)
    const int out_lane = (ws - 1) / K;
    const int ref_row_base = (seq10 % kRefSlots) * kCH;
    // Row slots are swizzled by the row's own global word address: element x of row r sits at
    // slot(r) + (G(r) & 31) + x, G(r) = word address of (r, c0).  The 16-byte phase G & 3 keeps
    // smem and global 16-byte alignment identical (bulk copies), and for an odd pitch the
    // 32 skewed rows a warp touches hit 32 different banks.
    const uintptr_t GR0 = (reinterpret_cast<uintptr_t>(R) >> 2) + c0;  // word address of (0, c0)
    const uintptr_t GS0 = (reinterpret_cast<uintptr_t>(S) >> 2) + c0;
    const int ldr32 = static_cast<int>(P.ldr & 31), lds32 = static_cast<int>(P.lds & 31);

    auto load_border = [&](int row) -> uint64_t {
      if (row > n) return 0ull;
      if (lin != nullptr) return lin_sys ? ld_relaxed_sys(lin + row) : ld_relaxed_gpu(lin + row);
      return static_cast<uint32_t>(__ldg(colp + static_cast<long long>(row) * P.lds));
    };

    // ref chunk c (rows 16c+1 .. 16c+16): lane t < 16 bulk-copies row 16c+1+t.
    auto issue_ref = [&](int c) {
      const int sl = (seq10 + c) % kRefSlots;
      const uint32_t bar = bar0 + 8 * sl;
      const int r = c * kCH + 1 + (t & (kCH - 1));
      uint32_t bytes = 0, dst = 0;
      const void* src = nullptr;
      if (t < kCH && r <= n) {
        const int32_t* g = R + static_cast<long long>(r) * P.ldr + c0;
        const uintptr_t gs = reinterpret_cast<uintptr_t>(g), ge = gs + 4u * ws;
        const uintptr_t s0 = gs & ~static_cast<uintptr_t>(15);
        // never read past the matrix end: the final row of the last band loads its tail scalar
        const bool tail_scalar = (r == n) && last_band;
        const uintptr_t e0 = tail_scalar ? (ge & ~static_cast<uintptr_t>(15)) : ((ge + 15) & ~static_cast<uintptr_t>(15));
        const int gw = static_cast<int>((gs >> 2) & 31);
        int32_t* drow = ref_ring + ((ref_row_base + r - 1) % kRefRows) * RS + (gw & ~3);
        if (e0 > s0) {
          bytes = static_cast<uint32_t>(e0 - s0);
          src = reinterpret_cast<const void*>(s0);
          dst = smem_u32(drow);
        }
        if (tail_scalar) {
          const int a = gw & 3;
          for (int x = e0 > gs ? static_cast<int>((e0 - gs) >> 2) : 0; x < ws; ++x) drow[a + x] = __ldg(g + x);
        }
      }
      mbar_arrive_expect_tx(bar, bytes);
      if (bytes) bulk_g2s(dst, src, bytes, bar);
    };

    // score chunk c: lanes < 16 bulk-store the aligned interior of row 16c+1+t, lanes >= 16
    // store the unaligned head/tail words of row 16c+1+(t-16).
    auto store_sc = [&](int c) {
      const int r = c * kCH + 1 + (t & (kCH - 1));
      if (r > n) return;
      int32_t* g = S + static_cast<long long>(r) * P.lds + c0;
      const uintptr_t gs = reinterpret_cast<uintptr_t>(g), ge = gs + 4u * ws;
      const uintptr_t as = (gs + 15) & ~static_cast<uintptr_t>(15), ae = ge & ~static_cast<uintptr_t>(15);
      const int32_t* srow = sc_ring + ((r - 1) % kScRows) * RS + static_cast<int>((gs >> 2) & 31);
      if (t < kCH) {
        if (ae > as) bulk_s2g(reinterpret_cast<void*>(as), smem_u32(srow) + static_cast<uint32_t>(as - gs),
                              static_cast<uint32_t>(ae - as));
      } else {
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
    uint64_t cur = load_border(1 + t), nxt = load_border(33 + t);
    int win_base = 1;  // cur holds border rows win_base + t
    // true when every row of the window is published (or beyond n): no per-step tag checks
    auto window_valid = [&]() -> bool {
      if (lin == nullptr) return true;
      return __all_sync(FULL, static_cast<uint32_t>(cur >> 32) == lin_epoch || win_base + t > n) != 0;
    };
    bool wvalid = window_valid();
    // per-lane incremental addressing for row r = step + 1 - t (starts at r0 = 1 - t)
    const int r0 = 1 - t;
    // 32-bit shared byte addresses of this lane's first column in its current row:
    //   ring + 4*(row_slot*RS + (G(r) & 31) + t*K); one add + two wrap fix-ups per step.
    int gR = static_cast<int>((GR0 + static_cast<uintptr_t>(static_cast<intptr_t>(r0) * P.ldr)) & 31);
    int gS = static_cast<int>((GS0 + static_cast<uintptr_t>(static_cast<intptr_t>(r0) * P.lds)) & 31);
    const uint32_t refR0 = smem_u32(ref_ring), refR1 = refR0 + 4u * kRefRows * RS;
    const uint32_t scR0 = smem_u32(sc_ring), scR1 = scR0 + 4u * kScRows * RS;
    uint32_t aR = refR0 + 4u * ((((ref_row_base + r0 - 1) % kRefRows + kRefRows) % kRefRows) * RS + gR + t * K);
    uint32_t aS = scR0 + 4u * ((((r0 - 1) % kScRows + kScRows) % kScRows) * RS + gS + t * K);
    const uint32_t stepR = 4u * (RS + ldr32), stepS = 4u * (RS + lds32);
    uint64_t* lout_row = lout != nullptr ? lout + r0 : nullptr;
    const bool do_out = lout != nullptr && t == out_lane;
    fence_proxy_async();
    __syncwarp();
    if constexpr (!SEQ) {
      for (int c = 0; c < kLook && c < nch; ++c) issue_ref(c);
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
        uint32_t w = 0;
#pragma unroll
        for (int m = 0; m < K; ++m) w |= static_cast<uint32_t>(static_cast<uint8_t>(P.subst[x * 32 + bj[m]])) << (8 * m);
        prof[x * 32 + t] = w;
      }
      a0 = A[min(max(r0 - 1, 0), n - 1)] & 31;
      a1 = A[min(max(r0, 0), n - 1)] & 31;
      __syncwarp();
    }

    // one wavefront step; ALL = every lane's row is in 1..n (steady state, no predicates)
    auto step = [&](const int sig, auto all_tag) {
      constexpr bool ALL = decltype(all_tag)::value;
      const int from_left = __shfl_up_sync(FULL, vlast, 1);
      const int idx = sig & 31;
      int bval = __shfl_sync(FULL, static_cast<int>(static_cast<uint32_t>(cur)), idx);
      if (!wvalid) {
        uint32_t bep = __shfl_sync(FULL, static_cast<uint32_t>(cur >> 32), idx);
        if (bep != lin_epoch && sig < n) {  // left band has not published row sig+1 yet
          const int rowb = win_base + t;
          const uint64_t t0 = globaltimer_ns();
          for (;;) {
            cur = load_border(rowb);
            bep = __shfl_sync(FULL, static_cast<uint32_t>(cur >> 32), idx);
            if (bep == lin_epoch) break;
            if (globaltimer_ns() - t0 > P.spin_limit_ns) {
              if (t == 0) atomicExch(P.err, kErrWatchdog);
              __trap();
            }
          }
          bval = __shfl_sync(FULL, static_cast<int>(static_cast<uint32_t>(cur)), idx);
          wvalid = window_valid();
        }
      }
      const int L = (t == 0) ? bval : from_left;
      bool active = true;
      if (!ALL) {
        const int r = lane_row(sig, t);
        active = r >= 1 && r <= n;
      }
      if (active) {

        int rv[K];
        if constexpr (SEQ) {
          const uint32_t pw = prof[a0 * 32 + t];
#pragma unroll
          for (int m = 0; m < K; ++m) rv[m] = prmt_sext(pw, 0x8880u + 0x1111u * m);  // sign-extended byte m
        } else {
#pragma unroll
          for (int m = 0; m < K; ++m) rv[m] = lds_s32(aR + 4 * m);
        }
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
        if (do_out) {
          // the publishing lane holds the band's last column in Pv[K-1]: every band with a right
          // neighbour is full width (only a pair's / the last rank's final band is ragged)
          const int vo = Pv[K - 1];
          if (lout_sys)
            st_relaxed_sys_v2(lout_row, static_cast<uint32_t>(vo), lout_epoch);
          else
            st_relaxed_gpu_v2(lout_row, static_cast<uint32_t>(vo), lout_epoch);
        }
      }
      vlast = Pv[K - 1];
      // advance this lane to row r+1
      if constexpr (SEQ) {
        a0 = a1;
        a1 = __ldg(A + min(max(lane_row(sig, t) + 1, 0), n - 1)) & 31;  // residue of row r+2
      }
      aR += stepR;  // next row slot + swizzle advance (G(r+1) = G(r) + ld)
      gR += ldr32;
      if (gR >= 32) {
        gR -= 32;
        aR -= 128;
      }
      if (aR >= refR1) aR -= refR1 - refR0;
      aS += stepS;
      gS += lds32;
      if (gS >= 32) {
        gS -= 32;
        aS -= 128;
      }
      if (aS >= scR1) aS -= scR1 - scR0;
      ++lout_row;
    };

    for (int Q = 0; Q <= nch + kStoreDelay - 1; ++Q) {
      const int sig0 = Q * kCH;
      // ---- chunk events (warp-uniform)
      bulk_wait_read<0>();  // stores issued at earlier events have read their slots
      __syncwarp();
      if (Q >= kStoreDelay && Q - kStoreDelay < nch) {
        fence_proxy_async();  // this lane's STS of rows in the finished chunk -> async proxy
        __syncwarp();
        store_sc(Q - kStoreDelay);
      }
      bulk_commit();
      if (!SEQ && Q + kLook < nch) {
        fence_proxy_async();
        __syncwarp();
        issue_ref(Q + kLook);
      }
      if (!SEQ && Q < nch) mbar_wait(bar0 + 8 * ((seq10 + Q) % kRefSlots), ((seq10 + Q) / kRefSlots) & 1);
      if (sig0 >= nsteps) continue;
      if ((sig0 & 31) == 0 && sig0 > 0) {
        cur = nxt;
        win_base = sig0 + 1;
        nxt = load_border(sig0 + 33 + t);
        wvalid = window_valid();
      }
      // ---- 16 wavefront steps: lane t computes row sig+1-t, columns c0+tK .. c0+tK+K-1
      if (sig0 >= 31 && sig0 + kCH <= n) {  // steady state: all 32 lanes on rows 1..n
#pragma unroll
        for (int j = 0; j < kCH; ++j) step(sig0 + j, std::true_type{});
      } else {
#pragma unroll 1
        for (int j = 0; j < kCH; ++j) {
          if (sig0 + j >= nsteps) break;
          step(sig0 + j, std::false_type{});
        }
      }
    }
    bulk_wait_all<0>();
    __syncwarp();
    seq10 = (seq10 + nch) % kSeqMod;
    if (P.trace != nullptr && t == 0 && task < P.trace_cap) {
      unsigned smid;
      asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
      unsigned long long* e = P.trace + 4 * task;
      e[0] = static_cast<unsigned long long>(task);
      e[1] = t_task0;
      e[2] = globaltimer_ns();
      e[3] = smid;
    }
  }
}

}  // namespace nwb200
