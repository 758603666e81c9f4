// nw_common.cuh — definitions shared by the wavefront kernel (nw_wave.cuh) and the host side:
// the band schedule (exported by nw_strip_map for pin P7), the kernel parameter block, the
// border-source / sink kinds, the volatile shared-memory accessors and the spin watchdog.
//
// What the path computes (Fig. 2, with Rodinia's cell function, R1):
//     score[i][j] = max(score[i-1][j-1] + ref[i][j], score[i-1][j] - p, score[i][j-1] - p)
// for every interior cell, each value written ONCE, in place (the short-circuited update of
// P:512-516 / P:616-656: no temporary, no copy).
#pragma once
#include <cstdint>
#include <type_traits>

#include "nw_ptx.cuh"

namespace nwb200 {

constexpr unsigned kErrWatchdog = 0xBADB0001u;

// Per-band timing instrumentation (nw_debug_set_trace / bench.py --trace) is compiled in only
// with -DNW_TRACE=1 (NW_TRACE=1 python -m paper_conf_sc_munksgaardhso22_b200._build): its
// runtime checks re-load the trace pointer from the constant bank at every event.
#ifndef NW_TRACE
#define NW_TRACE 0
#endif
constexpr bool kTrace = NW_TRACE != 0;
// full bands publish their border entries two rows per 16-byte store (NW_PAIRS=0: one per row)
#ifndef NW_PAIRS
#define NW_PAIRS 1
#endif
constexpr bool kPairs = NW_PAIRS != 0;

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
  // host pipeline (nw_fill[_batch]_host, pinned buffers): the stacked matrix's rows (pair * (n+1)
  // + r) in blocks of chunk_rows; ref block arrivals counted in *ref_ready by the copy-in stream,
  // score block completions counted per block in rows_done by the store warps (null: off)
  const unsigned* ref_ready;
  unsigned* rows_done;
  int64_t chunk_rows;
  int32_t vec16;  // 1: score and ref interior rows start 16-byte aligned (16-byte staging copies)
  int32_t zero0;  // 0 (experiment builds: an operand the compiler cannot fold)
  int32_t p2;  // 2p, read straight from the parameter bank by the step (a uniform operand, no register)
  int32_t nbands;  // bands per pair
  int64_t ntasks;  // pairs * nbands
  int64_t ngroups; // ceil(ntasks / NW) (pair mode: pairs)
  int32_t pair_mode;  // 1: a ticket is a whole pair, its bands swept one after the other (NW = 1)
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
  // NEXT-2 (SEQ kernels): ref[i][j] = subst[a[i-1]][b[j-1]] generated on chip
  const uint8_t* seq_a;
  const uint8_t* seq_b;
  int64_t psa, psb;  // pair strides of a / b (bytes)
  int8_t subst[32 * 32];
};

// opaque copy: keeps a value in a register (stops the compiler re-deriving smem bases per step)
__device__ __forceinline__ uint32_t opaque(uint32_t x) {
  asm volatile("mov.b32 %0, %0;" : "+r"(x));
  return x;
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
__device__ __noinline__ void watchdog_trap(unsigned int* err) {
  atomicExch(err, kErrWatchdog);
  __trap();
}

// Border sources/sinks of one band (uniform per task)
enum : int { kSrcPlain = 0, kSrcGlobal = 1, kSrcSmem = 2 };
enum : int { kSinkNone = 0, kSinkSmem = 1, kSinkGlobal = 2 };

}  // namespace nwb200
