// nw_lib.cu — host side of libnwb200.so: the C ABI declared in include/nw.h.
//
// Synchronous validation, a per-(device, stream) workspace cache (ticket counter, epoch-tagged
// band-border buffer, Unopt temporary), and the launches.  Every compute step runs in the
// kernels of nw_wave.cuh / nw_diag.cuh; there is no CPU fallback: without a usable CUDA
// device the entry points return NW_ECUDA.
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdlib>
#include <map>
#include <mutex>
#include <utility>

#include "nw.h"
#include "nw_diag.cuh"
#include "nw_traceback.cuh"
#include "nw_wave.cuh"

using namespace nwb200;

namespace {

thread_local int g_last_cuda = 0;

nw_status cuda_fail(cudaError_t e) {
  g_last_cuda = static_cast<int>(e);
  (void)cudaGetLastError();  // clear a non-sticky launch error
  return NW_ECUDA;
}
#define NW_CU(x)                                    \
  do {                                              \
    cudaError_t e_ = (x);                           \
    if (e_ != cudaSuccess) return cuda_fail(e_);    \
  } while (0)

constexpr int64_t kMaxN = (int64_t{1} << 30) - 64;

// tile -> kernel variant (WaveCfg below).  Band width W = 32 K.
//   variant 0 (tile 0 / 256): K = 8, W = 256, one band per CTA (compute, ref and two store
//             warps on the four SM sub-partitions) -- measured fastest at n = 32768;
//   variant 1 (tiles 16, 128): K = 4, W = 128, two bands per CTA (border between them through
//             shared memory), ref + store warp per band;
//   variant 2 (tiles 32, 64):  K = 4, W = 128, one band per CTA with a ref and two store warps
//             -- twice the CTAs of variant 1, for n where W = 128 bands are too few to fill the
//             GPU two per SM (n = 16384: 128 bands).
// The paper's b x b tile does not exist here (a band is W columns x all rows); every tile value
// gives the same matrix (tested).
int tile_to_variant(int32_t tile) {
  switch (tile) {
    case 0:
    case 256: return 0;
    case 16:
    case 128: return 1;
    case 32:
    case 64: return 2;
    default: return -1;
  }
}
int tile_to_k(int32_t tile) {
  const int v = tile_to_variant(tile);
  return v < 0 ? 0 : (v == 0 ? 8 : 4);
}

bool aligned4(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 3) == 0; }

bool overlaps(const void* a, int64_t abytes, const void* b, int64_t bbytes) {
  const uintptr_t a0 = reinterpret_cast<uintptr_t>(a), b0 = reinterpret_cast<uintptr_t>(b);
  return a0 < b0 + static_cast<uintptr_t>(bbytes) && b0 < a0 + static_cast<uintptr_t>(abytes);
}

// bytes spanned by an (n+1) x (n+1) matrix with pitch ld (first to last element)
int64_t span_bytes(int64_t n, int64_t ld) { return 4 * (n * ld + n + 1); }

// Range contract (nw.h).  The wavefront kernels evaluate the gap-normalised S' = S + (i + j) p
// (DESIGN.md §4.2); every intermediate is bounded by max|border| + (n + 1)(2p + NW_REF_MAX) in
// absolute value (S <= max border + min(i, j) NW_REF_MAX, S >= -max|border| - n p, (i + j) p <=
// 2 n p, a diagonal candidate adds ref + 2p).  With the caller's |border| <= 2^30 the sum stays
// below 2^31 when (n + 1)(2p + NW_REF_MAX) < 2^30, which is what we require.
nw_status check_range(int64_t n, int32_t p) {
  if (p < 0) return NW_ERANGE;
  const long double worst = (static_cast<long double>(n) + 1.0L) * (2.0L * p + NW_REF_MAX);
  if (worst >= 1073741824.0L) return NW_ERANGE;
  return NW_OK;
}

// Kernel instances: K columns per lane, SEQ (ref generated from the sequences), NW warps
// (bands) per CTA (DESIGN.md §4.3 sizes the rings).
// v5 self-staging wavefront kernels (nw_wave.cuh)
#ifndef NW_K8_SPB
#define NW_K8_SPB 3
#endif
#ifndef NW_K4_SPB
#define NW_K4_SPB 2
#endif
using WCfg8 = WaveCfg<8, false, 1, NW_K8_SPB>;   // tile 0 / 256: W = 256, one band per CTA, ref + store warps
using WCfg8S = WaveCfg<8, true, 1, NW_K8_SPB>;
using WCfg4 = WaveCfg<4, false, 2, NW_K4_SPB>;   // tiles 16, 128: W = 128, two bands per CTA
using WCfg4S = WaveCfg<4, true, 2, NW_K4_SPB>;
#ifndef NW_CLUSTER
#define NW_CLUSTER 4
#endif
using WCfg8C = WaveCfg<8, false, 1, NW_K8_SPB, NW_CLUSTER>;  // variant 0, one pair: clusters (DSMEM handoff)
using WCfg41 = WaveCfg<4, false, 1, 3>;          // tiles 32, 64: W = 128, one band per CTA
using WCfg41S = WaveCfg<4, true, 1, 3>;

struct DevInfo {
  bool init = false;
  int sms = 0;
  int clusters = 0;  // co-resident clusters of the WCfg8C kernel (0: clusters unusable)
  int wocc[3][2] = {{0, 0}, {0, 0}, {0, 0}};  // resident CTAs per SM [variant][SEQ]
};

template <class C>
cudaError_t setup_wave(int* occ) {
  cudaError_t e = cudaFuncSetAttribute(nw_wave_kernel<C>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       static_cast<int>(C::kSmem));
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(occ, nw_wave_kernel<C>, 32 * C::NWARPS, C::kSmem);
}

std::mutex g_mu;
DevInfo g_dev[128];
// test / experiment switches (explicit API calls, never environment variables: nw.h)
int g_debug_grid = 0;
bool g_debug_cluster = false;
int g_debug_pair_mode = 0;
int g_host_mode = 2;  // pinned host buffers: 0 staged, 1 zero copy, 2 copy-engine pipeline
int64_t g_host_block_rows = 0;  // pipeline row-block size (0: ~64 MB)
unsigned long long* g_trace = nullptr;
long long g_trace_cap = 0;

nw_status dev_info(int dev, DevInfo** out) {
  if (dev < 0 || dev >= 128) return NW_EINVAL;
  DevInfo& d = g_dev[dev];
  if (!d.init) {
    NW_CU(cudaDeviceGetAttribute(&d.sms, cudaDevAttrMultiProcessorCount, dev));
    NW_CU((setup_wave<WCfg8>(&d.wocc[0][0])));
    NW_CU((setup_wave<WCfg8S>(&d.wocc[0][1])));
    NW_CU((setup_wave<WCfg4>(&d.wocc[1][0])));
    NW_CU((setup_wave<WCfg4S>(&d.wocc[1][1])));
    NW_CU((setup_wave<WCfg41>(&d.wocc[2][0])));
    NW_CU((setup_wave<WCfg41S>(&d.wocc[2][1])));
    {
      int occ_c = 0;
      if (setup_wave<WCfg8C>(&occ_c) == cudaSuccess) {
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3(static_cast<unsigned>(WCfg8C::CL * 16));
        cfg.blockDim = dim3(32 * WCfg8C::NWARPS);
        cfg.dynamicSmemBytes = WCfg8C::kSmem;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeClusterDimension;
        at[0].val.clusterDim.x = WCfg8C::CL;
        at[0].val.clusterDim.y = 1;
        at[0].val.clusterDim.z = 1;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        if (cudaOccupancyMaxActiveClusters(&d.clusters, nw_wave_kernel<WCfg8C>, &cfg) != cudaSuccess) d.clusters = 0;
      }
      (void)cudaGetLastError();
    }
    for (auto& r : d.wocc)
      for (int o : r)
        if (o < 1) return cuda_fail(cudaErrorInvalidConfiguration);
    d.init = true;
  }
  *out = &d;
  return NW_OK;
}

struct Workspace {
  unsigned long long* d_ticket = nullptr;
  unsigned long long ticket_next = 0;
  unsigned int* d_err = nullptr;
  uint64_t* xbuf = nullptr;
  size_t xbuf_entries = 0;
  uint32_t epoch = 0;
  int32_t* xtmp = nullptr;  // Unopt temporary X
  size_t xtmp_elems = 0;
};
std::map<std::pair<int, void*>, Workspace*> g_ws;

nw_status get_ws(int dev, cudaStream_t st, Workspace** out) {
  auto key = std::make_pair(dev, static_cast<void*>(st));
  auto it = g_ws.find(key);
  if (it != g_ws.end()) {
    *out = it->second;
    return NW_OK;
  }
  Workspace* w = new Workspace();
  cudaError_t e = cudaMalloc(reinterpret_cast<void**>(&w->d_ticket), 64);
  if (e == cudaSuccess) e = cudaMemsetAsync(w->d_ticket, 0, 64, st);
  if (e != cudaSuccess) {
    delete w;
    return cuda_fail(e);
  }
  w->d_err = reinterpret_cast<unsigned int*>(w->d_ticket + 1);
  g_ws[key] = w;
  *out = w;
  return NW_OK;
}

nw_status ensure_xbuf(Workspace* w, size_t entries, cudaStream_t st) {
  if (entries <= w->xbuf_entries && w->epoch < 0xFFFFFFF0u) return NW_OK;
  if (w->xbuf) NW_CU(cudaFreeAsync(w->xbuf, st));
  w->xbuf = nullptr;
  w->xbuf_entries = 0;
  const size_t want = entries < 1024 ? 1024 : entries;
  NW_CU(cudaMallocAsync(reinterpret_cast<void**>(&w->xbuf), want * sizeof(uint64_t), st));
  NW_CU(cudaMemsetAsync(w->xbuf, 0, want * sizeof(uint64_t), st));  // tag 0 = never written
  w->xbuf_entries = want;
  w->epoch = 0;
  return NW_OK;
}

unsigned long long spin_limit_ns() {
  static unsigned long long v = [] {
    const char* s = std::getenv("NW_SPIN_LIMIT_MS");
    const unsigned long long ms = s ? std::strtoull(s, nullptr, 10) : 20000ull;
    return (ms ? ms : 20000ull) * 1000000ull;
  }();
  return v;
}

// Host pipeline signals (nw_fill[_batch]_host on pinned buffers, see there)
struct HostPipe {
  const unsigned* ref_ready;
  unsigned* rows_done;
  int64_t chunk_rows;
};

// One launch of the persistent kernel over `pairs` x ceil(width/W) bands.
nw_status launch_strip(int32_t* score, int64_t lds, int64_t pss, const int32_t* ref, int64_t ldr, int64_t psr,
                       int64_t pairs, int64_t n, int64_t width, int32_t p, int32_t tile, const uint64_t* halo_in,
                       uint64_t* halo_out, uint32_t halo_epoch, int32_t halo_out_sys, cudaStream_t st,
                       const uint8_t* seq_a = nullptr, const uint8_t* seq_b = nullptr, int64_t psa = 0,
                       int64_t psb = 0, const int8_t* subst32 = nullptr, const HostPipe* pipe = nullptr) {
  const int K = tile_to_k(tile);
  const bool SEQ = seq_a != nullptr;
  const int W = 32 * K;
  if (pairs == 0 || n == 0 || width == 0) return NW_OK;
  int dev = 0;
  NW_CU(cudaGetDevice(&dev));
  std::lock_guard<std::mutex> lk(g_mu);
  DevInfo* di = nullptr;
  nw_status s = dev_info(dev, &di);
  if (s != NW_OK) return s;
  Workspace* w = nullptr;
  s = get_ws(dev, st, &w);
  if (s != NW_OK) return s;
  const int64_t nbands = (width + W - 1) / W;
  // +2: the kernel's 16-byte border prefetches read entry pairs (2k, 2k+1), up to row n+1
  const size_t entries = static_cast<size_t>(pairs) * static_cast<size_t>(nbands - 1) * static_cast<size_t>(xstride(n)) + 2;
  s = ensure_xbuf(w, entries, st);
  if (s != NW_OK) return s;
  StripParams P{};
  P.score = score;
  P.lds = lds;
  P.pss = pss;
  P.ref = ref;
  P.ldr = ldr;
  P.psr = psr;
  P.n = n;
  P.width = width;
  P.p = p;
  P.p2 = 2 * p;
  P.nbands = static_cast<int32_t>(nbands);
  P.ntasks = pairs * nbands;
  const int var = tile_to_variant(tile);
  const int NW = var == 0 ? WCfg8::NW : (var == 1 ? WCfg4::NW : WCfg41::NW);
  // opt-in (nw_debug_set_cluster(1)): one pair on the K = 8 kernel as clusters of CL CTAs that
  // hand the border column over through DSMEM.  Measured slower than the global-memory handoff at
  // n = 32768 (318 vs 337 GCUPS with CL = 4; CL = 8 clusters do not all fit co-resident).
  const bool use_cluster = var == 0 && !SEQ && pairs == 1 && g_debug_cluster && di->clusters > 0 && g_debug_grid == 0;
  P.ngroups = use_cluster ? (P.ntasks + WCfg8C::CL - 1) / WCfg8C::CL : (P.ntasks + NW - 1) / NW;
  // many independent pairs on a one-band-per-CTA kernel: whole pairs per ticket (pair mode);
  // nw_debug_set_pair_mode: -1 never, 1 for any batch (tests), 0 automatic
  if (!use_cluster && NW == 1 && nbands > 1 && g_debug_pair_mode >= 0 &&
      (g_debug_pair_mode == 1 ? pairs > 1 : pairs >= 2LL * di->sms)) {
    P.pair_mode = 1;
    P.ngroups = pairs;
  }
  P.xbuf = w->xbuf;
  P.epoch = ++w->epoch;
  // 16-byte staging copies when every interior row of score (and ref) starts 16-byte aligned
  auto al16 = [&](const int32_t* base, int64_t ld, int64_t ps) {
    return (reinterpret_cast<uintptr_t>(base + 1) & 15) == 0 && ld % 4 == 0 && (pairs == 1 || ps % 4 == 0);
  };
  P.vec16 = al16(score, lds, pss) && (SEQ || al16(ref, ldr, psr)) ? 1 : 0;
  if (pipe) {
    P.ref_ready = pipe->ref_ready;
    P.rows_done = pipe->rows_done;
    P.chunk_rows = pipe->chunk_rows;
  }
  P.halo_in = halo_in;
  P.halo_out = halo_out;
  P.halo_epoch = halo_epoch;
  P.halo_out_sys = halo_out_sys;
  P.ticket = w->d_ticket;
  P.err = w->d_err;
  P.spin_limit_ns = spin_limit_ns();
  P.trace = g_trace;
  P.trace_cap = g_trace_cap;
  P.trace2 = g_trace ? g_trace + 8 * g_trace_cap : nullptr;
  if (SEQ) {
    P.seq_a = seq_a;
    P.seq_b = seq_b;
    P.psa = psa;
    P.psb = psb;
    for (int i = 0; i < 32 * 32; ++i) P.subst[i] = subst32[i];
  }
  if (use_cluster) {
    const int64_t ncl = std::min<int64_t>(di->clusters, P.ngroups);
    P.ticket_base = w->ticket_next;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(static_cast<unsigned>(ncl * WCfg8C::CL));
    cfg.blockDim = dim3(32 * WCfg8C::NWARPS);
    cfg.dynamicSmemBytes = WCfg8C::kSmem;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = WCfg8C::CL;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    NW_CU(cudaLaunchKernelEx(&cfg, nw_wave_kernel<WCfg8C>, P));
    w->ticket_next += static_cast<unsigned long long>(P.ngroups + ncl);  // every cluster draws one extra ticket
    return NW_OK;
  }
  const int occ = di->wocc[var][SEQ];
  int64_t grid = static_cast<int64_t>(occ) * di->sms;
  if (g_debug_grid > 0) grid = g_debug_grid;
  if (grid > P.ngroups) grid = P.ngroups;
  P.ticket_base = w->ticket_next;
  const unsigned g = static_cast<unsigned>(grid);
  if (var == 0 && !SEQ)
    nw_wave_kernel<WCfg8><<<g, 32 * WCfg8::NWARPS, WCfg8::kSmem, st>>>(P);
  else if (var == 0)
    nw_wave_kernel<WCfg8S><<<g, 32 * WCfg8S::NWARPS, WCfg8S::kSmem, st>>>(P);
  else if (var == 1 && !SEQ)
    nw_wave_kernel<WCfg4><<<g, 32 * WCfg4::NWARPS, WCfg4::kSmem, st>>>(P);
  else if (var == 1)
    nw_wave_kernel<WCfg4S><<<g, 32 * WCfg4S::NWARPS, WCfg4S::kSmem, st>>>(P);
  else if (!SEQ)
    nw_wave_kernel<WCfg41><<<g, 32 * WCfg41::NWARPS, WCfg41::kSmem, st>>>(P);
  else
    nw_wave_kernel<WCfg41S><<<g, 32 * WCfg41S::NWARPS, WCfg41S::kSmem, st>>>(P);
  NW_CU(cudaGetLastError());
  // only a launched grid consumes tickets (every CTA draws one past the last group): a failed
  // launch leaves the device counter and the host base in step
  w->ticket_next += static_cast<unsigned long long>(P.ngroups + grid);
  return NW_OK;
}

nw_status validate_pair(const int32_t* score, int64_t lds, const int32_t* ref, int64_t ldr, int64_t n,
                        int32_t p, int32_t tile) {
  if (!score || !ref) return NW_EINVAL;
  if (n < 0 || n > kMaxN) return NW_EINVAL;
  if (tile_to_k(tile) == 0) return NW_EINVAL;
  if (lds < n + 1 || ldr < n + 1) return NW_EINVAL;
  if (!aligned4(score) || !aligned4(ref)) return NW_EINVAL;
  if (overlaps(score, span_bytes(n, lds), ref, span_bytes(n, ldr))) return NW_EINVAL;
  return check_range(n, p);
}

template <int B>
nw_status run_diag(int32_t* score, int64_t lds, const int32_t* ref, int64_t ldr, int64_t n, int32_t p, bool unopt,
                   cudaStream_t st) {
  const int q = static_cast<int>((n + B - 1) / B);
  int32_t* X = nullptr;
  if (unopt) {
    int dev = 0;
    NW_CU(cudaGetDevice(&dev));
    std::lock_guard<std::mutex> lk(g_mu);
    Workspace* w = nullptr;
    nw_status s = get_ws(dev, st, &w);
    if (s != NW_OK) return s;
    const size_t need = static_cast<size_t>(q) * B * B;
    if (need > w->xtmp_elems) {
      if (w->xtmp) NW_CU(cudaFreeAsync(w->xtmp, st));
      w->xtmp = nullptr;
      w->xtmp_elems = 0;
      NW_CU(cudaMallocAsync(reinterpret_cast<void**>(&w->xtmp), need * sizeof(int32_t), st));
      w->xtmp_elems = need;
    }
    X = w->xtmp;
  }
  for (int d = 0; d <= 2 * q - 2; ++d) {
    const DiagLmad L = diag_lmad(q, B, lds, d);
    nw_diag_kernel<B><<<static_cast<unsigned>(L.cnt), B, 0, st>>>(score, lds, ref, ldr, static_cast<int>(n), p, d,
                                                                   q, X);
    if (unopt) nw_diag_copy_kernel<B><<<static_cast<unsigned>(L.cnt), B, 0, st>>>(score, lds, static_cast<int>(n), d, q, X);
  }
  NW_CU(cudaGetLastError());
  return NW_OK;
}

nw_status diag_entry(int32_t* score, int64_t lds, const int32_t* ref, int64_t ldr, int64_t n, int32_t p,
                     int32_t tile, void* stream, bool unopt) {
  if (tile != 16 && tile != 32 && tile != 64) return NW_EINVAL;
  nw_status s = validate_pair(score, lds, ref, ldr, n, p, tile);
  if (s != NW_OK || n == 0) return s;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  switch (tile) {
    case 16: return run_diag<16>(score, lds, ref, ldr, n, p, unopt, st);
    case 32: return run_diag<32>(score, lds, ref, ldr, n, p, unopt, st);
    default: return run_diag<64>(score, lds, ref, ldr, n, p, unopt, st);
  }
}

struct HostBufs {
  int32_t* score = nullptr;
  int32_t* ref = nullptr;
  size_t elems = 0;
  cudaStream_t st = nullptr;
  cudaStream_t sin = nullptr, sout = nullptr;  // pipeline: copy-in / copy-out streams
  cudaEvent_t ev = nullptr;
  unsigned* flags = nullptr;  // pipeline: [0] ref blocks arrived, [1 + c] store signals of block c
  size_t nflags = 0;
};

// Stream memory operations (driver API, fetched at run time: the library links only cudart)
using PfnWaitValue32 = CUresult (*)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
using PfnWriteValue32 = CUresult (*)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
PfnWaitValue32 g_wait_value = nullptr;
PfnWriteValue32 g_write_value = nullptr;
bool stream_mem_ops() {
  static const bool ok = [] {
    cudaDriverEntryPointQueryResult q;
    cudaGetDriverEntryPoint("cuStreamWaitValue32", reinterpret_cast<void**>(&g_wait_value), cudaEnableDefault, &q);
    cudaGetDriverEntryPoint("cuStreamWriteValue32", reinterpret_cast<void**>(&g_write_value), cudaEnableDefault, &q);
    (void)cudaGetLastError();
    return g_wait_value != nullptr && g_write_value != nullptr;
  }();
  return ok;
}
HostBufs g_host[128];
// one staged host call per device at a time: the staging buffers and their stream are per device
// (the lock spans the reallocation, the copies, the launch and the final synchronisation)
std::mutex g_host_mu[128];

}  // namespace

extern "C" {

const char* nw_status_str(int status) {
  switch (status) {
    case NW_OK: return "NW_OK";
    case NW_EINVAL: return "NW_EINVAL: invalid argument (pointer, size, tile, pitch, alignment or overlap)";
    case NW_ERANGE: return "NW_ERANGE: penalty < 0 or int32 could overflow ((n+1)*(2*p + NW_REF_MAX) >= 2^30)";
    case NW_ECUDA: return "NW_ECUDA: a CUDA runtime call or workspace allocation failed (see nw_last_cuda_error)";
    case NW_ECOMM: return "NW_ECOMM: inconsistent sharded strip / halo description";
    default: return "NW_UNKNOWN";
  }
}

int nw_abi_version(void) { return NW_ABI_VERSION; }
int nw_last_cuda_error(void) { return g_last_cuda; }

nw_status nw_fill_ld(int32_t* score, int64_t ld_score, const int32_t* ref, int64_t ld_ref, int64_t n,
                     int32_t penalty, int32_t tile, void* stream) {
  nw_status s = validate_pair(score, ld_score, ref, ld_ref, n, penalty, tile);
  if (s != NW_OK || n == 0) return s;
  return launch_strip(score, ld_score, 0, ref, ld_ref, 0, 1, n, n, penalty, tile, nullptr, nullptr, 0, 0,
                      static_cast<cudaStream_t>(stream));
}

nw_status nw_fill(int32_t* score, const int32_t* ref, int64_t n, int32_t penalty, int32_t tile, void* stream) {
  return nw_fill_ld(score, n + 1, ref, n + 1, n, penalty, tile, stream);
}

nw_status nw_fill_batch_ld(int32_t* score, int64_t ld_score, int64_t stride_score, const int32_t* ref,
                           int64_t ld_ref, int64_t stride_ref, int64_t batch, int64_t n, int32_t penalty,
                           int32_t tile, void* stream) {
  if (batch < 0) return NW_EINVAL;
  if (!score || !ref || n < 0 || n > kMaxN || tile_to_k(tile) == 0) return NW_EINVAL;
  if (ld_score < n + 1 || ld_ref < n + 1) return NW_EINVAL;
  if (!aligned4(score) || !aligned4(ref)) return NW_EINVAL;
  const int64_t ss = span_bytes(n, ld_score) / 4, sr = span_bytes(n, ld_ref) / 4;
  if (batch > 1 && (stride_score < ss || stride_ref < sr)) return NW_EINVAL;  // pairs must not overlap
  if (batch > 0 && overlaps(score, 4 * ((batch - 1) * stride_score + ss), ref, 4 * ((batch - 1) * stride_ref + sr)))
    return NW_EINVAL;
  nw_status s = check_range(n, penalty);
  if (s != NW_OK || batch == 0 || n == 0) return s;
  return launch_strip(score, ld_score, stride_score, ref, ld_ref, stride_ref, batch, n, n, penalty, tile, nullptr,
                      nullptr, 0, 0, static_cast<cudaStream_t>(stream));
}

nw_status nw_fill_batch(int32_t* score, const int32_t* ref, int64_t batch, int64_t n, int32_t penalty,
                        int32_t tile, void* stream) {
  const int64_t st = (n + 1) * (n + 1);
  return nw_fill_batch_ld(score, n + 1, st, ref, n + 1, st, batch, n, penalty, tile, stream);
}

nw_status nw_fill_sharded(const nw_strip* sp, int32_t penalty, int32_t tile, void* stream) {
  if (!sp) return NW_EINVAL;
  const nw_strip& S = *sp;
  if (!S.score || !S.ref || S.n < 0 || S.n > kMaxN || S.w < 0 || S.w > kMaxN) return NW_EINVAL;
  if (tile_to_k(tile) == 0) return NW_EINVAL;
  if (S.ld_score < S.w + 1 || S.ld_ref < S.w + 1) return NW_EINVAL;
  if (!aligned4(S.score) || !aligned4(S.ref)) return NW_EINVAL;
  if (overlaps(S.score, 4 * (S.n * S.ld_score + S.w + 1), S.ref, 4 * (S.n * S.ld_ref + S.w + 1))) return NW_EINVAL;
  if ((S.halo_in || S.halo_out) && S.epoch == 0) return NW_ECOMM;
  if ((S.halo_in && (reinterpret_cast<uintptr_t>(S.halo_in) & 15)) ||
      (S.halo_out && (reinterpret_cast<uintptr_t>(S.halo_out) & 15)))
    return NW_ECOMM;
  // a strip that pushes a halo must end on a band boundary (its last band is then full width)
  if (S.halo_out && S.w % nw_band_width(tile) != 0) return NW_ECOMM;
  nw_status s = check_range(S.n > S.w ? S.n : S.w, penalty);
  if (s != NW_OK || S.n == 0 || S.w == 0) return s;
  return launch_strip(S.score, S.ld_score, 0, S.ref, S.ld_ref, 0, 1, S.n, S.w, penalty, tile, S.halo_in,
                      S.halo_out, S.epoch, S.halo_out_is_peer, static_cast<cudaStream_t>(stream));
}

nw_status nw_fill_seq_batch(int32_t* score, int64_t ld_score, int64_t stride_score, const uint8_t* a,
                            const uint8_t* b, int64_t stride_seq, int64_t batch, int64_t n, const int32_t* subst,
                            int32_t alphabet, int32_t penalty, int32_t tile, void* stream) {
  if (batch < 0 || !score || !a || !b || !subst || n < 0 || n > kMaxN || tile_to_k(tile) == 0) return NW_EINVAL;
  if (alphabet < 1 || alphabet > 32 || ld_score < n + 1 || !aligned4(score)) return NW_EINVAL;
  const int64_t ss = span_bytes(n, ld_score) / 4;
  if (batch > 1 && (stride_score < ss || stride_seq < n)) return NW_EINVAL;
  int8_t tab[32 * 32] = {0};
  for (int x = 0; x < alphabet; ++x)
    for (int y = 0; y < alphabet; ++y) {
      const int32_t v = subst[x * alphabet + y];
      if (v < -128 || v > 127) return NW_ERANGE;
      tab[x * 32 + y] = static_cast<int8_t>(v);
    }
  nw_status s = check_range(n, penalty);
  if (s != NW_OK || batch == 0 || n == 0) return s;
  return launch_strip(score, ld_score, stride_score, nullptr, 0, 0, batch, n, n, penalty, tile, nullptr, nullptr, 0,
                      0, static_cast<cudaStream_t>(stream), a, b, stride_seq, stride_seq, tab);
}

nw_status nw_fill_seq(int32_t* score, int64_t ld_score, const uint8_t* a, const uint8_t* b, int64_t n,
                      const int32_t* subst, int32_t alphabet, int32_t penalty, int32_t tile, void* stream) {
  return nw_fill_seq_batch(score, ld_score, 0, a, b, 0, 1, n, subst, alphabet, penalty, tile, stream);
}

nw_status nw_fill_batch_host(int32_t* score_host, const int32_t* ref_host, int64_t batch, int64_t n, int32_t penalty,
                             int32_t tile, int32_t device) {
  if (!score_host || !ref_host || batch < 0 || n < 0 || n > kMaxN || tile_to_k(tile) == 0) return NW_EINVAL;
  if (device < 0 || device >= 128) return NW_EINVAL;
  nw_status s = check_range(n, penalty);
  if (s != NW_OK || n == 0 || batch == 0) return s;
  NW_CU(cudaSetDevice(device));
  HostBufs& hb = g_host[device];
  const size_t pair_elems = static_cast<size_t>(n + 1) * static_cast<size_t>(n + 1);
  const size_t elems = pair_elems * static_cast<size_t>(batch);
  {
    std::lock_guard<std::mutex> lk(g_mu);
    if (!hb.st) NW_CU(cudaStreamCreateWithFlags(&hb.st, cudaStreamNonBlocking));
  }
  cudaPointerAttributes as{}, ar{};
  const bool pinned = cudaPointerGetAttributes(&as, score_host) == cudaSuccess &&
                      cudaPointerGetAttributes(&ar, ref_host) == cudaSuccess && as.type == cudaMemoryTypeHost &&
                      ar.type == cudaMemoryTypeHost && as.devicePointer && ar.devicePointer;
  (void)cudaGetLastError();
  // Pinned (device-mapped) host buffers, zero-copy mode: the kernel streams ref in and score out
  // over the host link itself (both directions at once, overlapped with the wavefront).
  if (pinned && g_host_mode == 1) {
    s = launch_strip(static_cast<int32_t*>(as.devicePointer), n + 1, static_cast<int64_t>(pair_elems),
                     static_cast<const int32_t*>(ar.devicePointer), n + 1, static_cast<int64_t>(pair_elems), batch, n, n,
                     penalty, tile, nullptr, nullptr, 0, 0, hb.st);
    if (s != NW_OK) return s;
    NW_CU(cudaStreamSynchronize(hb.st));
    return NW_OK;
  }
  const bool pipeline = pinned && g_host_mode == 2 && stream_mem_ops();
  std::lock_guard<std::mutex> hlk(g_host_mu[device]);
  {
    std::lock_guard<std::mutex> lk(g_mu);
    if (elems > hb.elems) {
      if (hb.score) NW_CU(cudaFree(hb.score));
      if (hb.ref) NW_CU(cudaFree(hb.ref));
      hb.score = hb.ref = nullptr;
      hb.elems = 0;
      NW_CU(cudaMalloc(reinterpret_cast<void**>(&hb.score), elems * 4));
      NW_CU(cudaMalloc(reinterpret_cast<void**>(&hb.ref), elems * 4));
      hb.elems = elems;
    }
  }
  const size_t pitch = static_cast<size_t>(n + 1) * 4;
  if (pipeline) {
    // Copy-engine pipeline over the stacked matrix's rows (pair * (n+1) + r) in blocks of CHR rows
    // (~64 MB): the copy-in stream moves the borders, then ref block by block, publishing each
    // arrival in flags[0] (stream write); the kernel's ref warps wait for the blocks they stage;
    // its store warps count, per block, the bands whose rows in it are stored (flags[1 + c]); the
    // copy-out stream waits for each block's count and copies it back.  Both link directions
    // then run at copy-engine rate while the wavefront runs (zero copy moved ~31 GB/s each way).
    const int64_t rows = batch * (n + 1);
    const int64_t chr = g_host_block_rows > 0 ? g_host_block_rows : std::max<int64_t>(64, (int64_t{64} << 20) / static_cast<int64_t>(pitch));
    const int64_t nblk = (rows + chr - 1) / chr;
    const int K = tile_to_k(tile);
    const int64_t nbands = (n + 32 * K - 1) / (32 * K);
    const int nstore = tile_to_variant(tile) == 1 ? 1 : 2;  // store warps per band (WaveCfg SPB)
    {
      std::lock_guard<std::mutex> lk(g_mu);
      if (!hb.sin) NW_CU(cudaStreamCreateWithFlags(&hb.sin, cudaStreamNonBlocking));
      if (!hb.sout) NW_CU(cudaStreamCreateWithFlags(&hb.sout, cudaStreamNonBlocking));
      if (!hb.ev) NW_CU(cudaEventCreateWithFlags(&hb.ev, cudaEventDisableTiming));
      if (static_cast<size_t>(nblk + 1) > hb.nflags) {
        if (hb.flags) NW_CU(cudaFree(hb.flags));
        hb.flags = nullptr;
        hb.nflags = 0;
        NW_CU(cudaMalloc(reinterpret_cast<void**>(&hb.flags), static_cast<size_t>(nblk + 1) * 4));
        hb.nflags = static_cast<size_t>(nblk + 1);
      }
    }
    NW_CU(cudaMemsetAsync(hb.flags, 0, static_cast<size_t>(nblk + 1) * 4, hb.sin));
    for (int64_t k = 0; k < batch; ++k) {  // borders first: row 0 and column 0 of each pair
      int32_t* d = hb.score + k * static_cast<int64_t>(pair_elems);
      const int32_t* h = score_host + k * static_cast<int64_t>(pair_elems);
      NW_CU(cudaMemcpyAsync(d, h, pitch, cudaMemcpyHostToDevice, hb.sin));
      NW_CU(cudaMemcpy2DAsync(d + (n + 1), pitch, h + (n + 1), pitch, 4, static_cast<size_t>(n), cudaMemcpyHostToDevice, hb.sin));
    }
    NW_CU(cudaEventRecord(hb.ev, hb.sin));
    NW_CU(cudaStreamWaitEvent(hb.st, hb.ev, 0));
    NW_CU(cudaStreamWaitEvent(hb.sout, hb.ev, 0));
    const HostPipe pipe{hb.flags, hb.flags + 1, chr};
    s = launch_strip(hb.score, n + 1, static_cast<int64_t>(pair_elems), hb.ref, n + 1, static_cast<int64_t>(pair_elems), batch, n,
                     n, penalty, tile, nullptr, nullptr, 0, 0, hb.st, nullptr, nullptr, 0, 0, nullptr, &pipe);
    if (s != NW_OK) {
      (void)cudaStreamSynchronize(hb.sin);
      return s;
    }
    const CUdeviceptr fl = reinterpret_cast<CUdeviceptr>(hb.flags);
    for (int64_t c = 0; c < nblk; ++c) {
      const int64_t r0 = c * chr, r1 = std::min(rows, r0 + chr);
      NW_CU(cudaMemcpyAsync(hb.ref + r0 * (n + 1), ref_host + r0 * (n + 1), static_cast<size_t>(r1 - r0) * pitch,
                            cudaMemcpyHostToDevice, hb.sin));
      if (g_write_value(hb.sin, fl, static_cast<cuuint32_t>(c + 1), 0) != CUDA_SUCCESS) return cuda_fail(cudaErrorUnknown);
    }
    for (int64_t c = 0; c < nblk; ++c) {
      const int64_t r0 = c * chr, r1 = std::min(rows, r0 + chr);
      // signals expected in block c: every band of every pair with an interior row in it
      const int64_t p_lo = r0 / (n + 1), p_hi = (r1 - 2) / (n + 1);  // pairs with an interior row in [r0, r1)
      const int64_t npairs = p_hi >= p_lo ? p_hi - p_lo + 1 : 0;
      const cuuint32_t want = static_cast<cuuint32_t>(npairs * nbands * nstore);
      if (want > 0 && g_wait_value(hb.sout, fl + 4 * (1 + c), want, CU_STREAM_WAIT_VALUE_GEQ) != CUDA_SUCCESS)
        return cuda_fail(cudaErrorUnknown);
      NW_CU(cudaMemcpyAsync(score_host + r0 * (n + 1), hb.score + r0 * (n + 1), static_cast<size_t>(r1 - r0) * pitch,
                            cudaMemcpyDeviceToHost, hb.sout));
    }
    NW_CU(cudaStreamSynchronize(hb.sout));
    NW_CU(cudaStreamSynchronize(hb.st));
    NW_CU(cudaStreamSynchronize(hb.sin));
    return NW_OK;
  }
  NW_CU(cudaMemcpyAsync(hb.ref, ref_host, elems * 4, cudaMemcpyHostToDevice, hb.st));
  for (int64_t k = 0; k < batch; ++k) {  // borders only: row 0 and column 0 of each pair
    int32_t* d = hb.score + k * static_cast<int64_t>(pair_elems);
    const int32_t* h = score_host + k * static_cast<int64_t>(pair_elems);
    NW_CU(cudaMemcpyAsync(d, h, pitch, cudaMemcpyHostToDevice, hb.st));
    NW_CU(cudaMemcpy2DAsync(d + (n + 1), pitch, h + (n + 1), pitch, 4, static_cast<size_t>(n), cudaMemcpyHostToDevice, hb.st));
  }
  s = launch_strip(hb.score, n + 1, static_cast<int64_t>(pair_elems), hb.ref, n + 1, static_cast<int64_t>(pair_elems), batch, n, n,
                   penalty, tile, nullptr, nullptr, 0, 0, hb.st);
  if (s != NW_OK) return s;
  NW_CU(cudaMemcpyAsync(score_host, hb.score, elems * 4, cudaMemcpyDeviceToHost, hb.st));
  NW_CU(cudaStreamSynchronize(hb.st));
  return NW_OK;
}

nw_status nw_fill_host(int32_t* score_host, const int32_t* ref_host, int64_t n, int32_t penalty, int32_t tile,
                       int32_t device) {
  return nw_fill_batch_host(score_host, ref_host, 1, n, penalty, tile, device);
}

nw_status nw_traceback_batch(const int32_t* score, int64_t ld_score, int64_t stride_score, const int32_t* ref,
                             int64_t ld_ref, int64_t stride_ref, int64_t batch, int64_t n, int32_t penalty,
                             uint8_t* ops, int64_t ops_stride, int32_t* len, void* stream) {
  if (batch < 0 || !score || !ref || !ops || !len || n < 0 || n > kMaxN) return NW_EINVAL;
  if (ld_score < n + 1 || ld_ref < n + 1 || !aligned4(score) || !aligned4(ref) || !aligned4(len)) return NW_EINVAL;
  if (batch > 1 && (stride_score < span_bytes(n, ld_score) / 4 || stride_ref < span_bytes(n, ld_ref) / 4 ||
                    ops_stride < 2 * n))
    return NW_EINVAL;
  if (batch > 0) {  // outputs must not overlap each other or the inputs
    const int64_t ob = (batch - 1) * ops_stride + 2 * n, lb = 4 * batch;
    const int64_t sb = 4 * ((batch - 1) * stride_score) + span_bytes(n, ld_score);
    const int64_t rb = 4 * ((batch - 1) * stride_ref) + span_bytes(n, ld_ref);
    if (overlaps(ops, ob, len, lb) || overlaps(ops, ob, score, sb) || overlaps(ops, ob, ref, rb) ||
        overlaps(len, lb, score, sb) || overlaps(len, lb, ref, rb))
      return NW_EINVAL;
  }
  nw_status s = check_range(n, penalty);
  if (s != NW_OK || batch == 0) return s;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  TbParams P{score, ld_score, stride_score, ref, ld_ref, stride_ref, batch, n, penalty, ops, ops_stride, len};
  if (batch <= kTbFewPairs)  // few pairs: kTbFewWpp warps share each window
    nw_traceback_kernel<kTbFewWpp, kTbFewWpp><<<static_cast<unsigned>(batch), 32 * kTbFewWpp, 0, st>>>(P);
  else
    nw_traceback_kernel<kTbManyWpp><<<static_cast<unsigned>((batch * kTbManyWpp + kTbWarps - 1) / kTbWarps),
                                      32 * kTbWarps, 0, st>>>(P);
  NW_CU(cudaGetLastError());
  if (n > 0) {
    const long long gx = std::min<long long>((n + 255) / 256, 1024);
    const unsigned gy = static_cast<unsigned>(std::min<long long>(batch, 65535));
    nw_traceback_reverse_kernel<<<dim3(static_cast<unsigned>(gx), gy), 256, 0, st>>>(ops, ops_stride, len, batch);
    NW_CU(cudaGetLastError());
  }
  return NW_OK;
}

nw_status nw_traceback(const int32_t* score, int64_t ld_score, const int32_t* ref, int64_t ld_ref, int64_t n,
                       int32_t penalty, uint8_t* ops, int32_t* len, void* stream) {
  return nw_traceback_batch(score, ld_score, 0, ref, ld_ref, 0, 1, n, penalty, ops, 2 * n, len, stream);
}

nw_status nw_fill_diagonal(int32_t* score, int64_t ld_score, const int32_t* ref, int64_t ld_ref, int64_t n,
                           int32_t penalty, int32_t tile, void* stream) {
  return diag_entry(score, ld_score, ref, ld_ref, n, penalty, tile, stream, false);
}

nw_status nw_fill_unopt(int32_t* score, int64_t ld_score, const int32_t* ref, int64_t ld_ref, int64_t n,
                        int32_t penalty, int32_t tile, void* stream) {
  return diag_entry(score, ld_score, ref, ld_ref, n, penalty, tile, stream, true);
}

int32_t nw_band_width(int32_t tile) { return 32 * tile_to_k(tile); }

int64_t nw_launch_count(int32_t kind, int64_t n, int32_t tile) {
  if (n <= 0) return 0;
  if (kind == 0) return tile_to_k(tile) ? 1 : -1;
  if (tile != 16 && tile != 32 && tile != 64) return -1;
  const int64_t q = (n + tile - 1) / tile;
  if (kind == 1) return 2 * q - 1;
  if (kind == 2) return 2 * (2 * q - 1);
  return -1;
}

int32_t nw_diag_lmad(int64_t n, int64_t N, int32_t tile, int64_t d, int64_t out[10]) {
  if (!out || n < 1 || tile < 1 || N < n + 1) return -1;
  const int64_t q = (n + tile - 1) / tile;
  if (d < 0 || d > 2 * q - 2) return -1;
  const DiagLmad L = diag_lmad(q, tile, N, d);
  out[0] = L.cnt;
  out[1] = L.base;
  out[2] = L.base + N + 1;  // W offset
  out[3] = L.s0;
  out[4] = N;
  out[5] = 1;
  out[6] = L.base;  // Rvert offset
  out[7] = N;
  out[8] = L.base + 1;  // Rhoriz offset
  out[9] = 1;
  return 0;
}

nw_status nw_kernel_info(int32_t tile, int32_t device, int64_t* smem_bytes, int32_t* ctas_per_sm,
                         int32_t* num_sms) {
  const int K = tile_to_k(tile);
  if (!K) return NW_EINVAL;
  const int var = tile_to_variant(tile);
  if (smem_bytes) *smem_bytes = static_cast<int64_t>(var == 0 ? WCfg8::kSmem : (var == 1 ? WCfg4::kSmem : WCfg41::kSmem));
  if (!ctas_per_sm && !num_sms) return NW_OK;
  NW_CU(cudaSetDevice(device));
  std::lock_guard<std::mutex> lk(g_mu);
  DevInfo* di = nullptr;
  nw_status s = dev_info(device, &di);
  if (s != NW_OK) return s;
  if (ctas_per_sm) *ctas_per_sm = di->wocc[var][0];
  if (num_sms) *num_sms = di->sms;
  return NW_OK;
}

int32_t nw_strip_map(int64_t n, int64_t width, int32_t tile, int32_t band, int32_t step, int32_t lane,
                     int64_t out[3]) {
  const int K = tile_to_k(tile);
  if (!out || !K || n < 0 || width < 1 || lane < 0 || lane > 31 || band < 0) return -1;
  const int W = 32 * K;
  if (static_cast<int64_t>(band) * W >= width) return -1;
  const int c0 = band_c0(band, W), ws = band_ws(width, band, W);
  const int r = lane_row(step, lane);
  int nc = ws - lane * K;
  nc = nc < 0 ? 0 : (nc > K ? K : nc);
  if (r < 1 || r > n) nc = 0;
  out[0] = r;
  out[1] = c0 + lane * K;
  out[2] = nc;
  return 0;
}

void nw_debug_set_grid(int32_t grid) { g_debug_grid = grid > 0 ? grid : 0; }
void nw_debug_set_pair_mode(int32_t mode) { g_debug_pair_mode = mode < 0 ? -1 : (mode > 0 ? 1 : 0); }
void nw_debug_set_cluster(int32_t on) { g_debug_cluster = on != 0; }
void nw_debug_set_host_zero_copy(int32_t on) { g_host_mode = on ? 1 : 2; }
void nw_debug_set_host_mode(int32_t mode) { g_host_mode = mode < 0 || mode > 2 ? 2 : mode; }
void nw_debug_set_host_block_rows(int64_t rows) { g_host_block_rows = rows > 0 ? rows : 0; }

void nw_debug_set_trace(uint64_t* dev_buf, int64_t cap_tasks) {
  std::lock_guard<std::mutex> lk(g_mu);
  g_trace = reinterpret_cast<unsigned long long*>(dev_buf);
  g_trace_cap = dev_buf ? cap_tasks : 0;
}

void nw_release_workspace(void) {
  std::lock_guard<std::mutex> lk(g_mu);
  for (auto& kv : g_ws) {
    Workspace* w = kv.second;
    cudaSetDevice(kv.first.first);
    cudaStreamSynchronize(static_cast<cudaStream_t>(kv.first.second));
    if (w->xbuf) cudaFree(w->xbuf);
    if (w->xtmp) cudaFree(w->xtmp);
    if (w->d_ticket) cudaFree(w->d_ticket);
    delete w;
  }
  g_ws.clear();
  for (int d = 0; d < 128; ++d) {
    HostBufs& hb = g_host[d];
    if (hb.score || hb.ref || hb.st) {
      cudaSetDevice(d);
      if (hb.st) cudaStreamSynchronize(hb.st);
      if (hb.sin) cudaStreamSynchronize(hb.sin);
      if (hb.sout) cudaStreamSynchronize(hb.sout);
      if (hb.score) cudaFree(hb.score);
      if (hb.ref) cudaFree(hb.ref);
      if (hb.flags) cudaFree(hb.flags);
      if (hb.ev) cudaEventDestroy(hb.ev);
      if (hb.st) cudaStreamDestroy(hb.st);
      if (hb.sin) cudaStreamDestroy(hb.sin);
      if (hb.sout) cudaStreamDestroy(hb.sout);
      hb = HostBufs();
    }
  }
}

}  // extern "C"
