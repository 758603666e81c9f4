/*
 * nw.h — C-ABI of libnwb200.so: Needleman–Wunsch score-matrix fill on B200 (sm_100a).
 *
 * THE BOUNDARY of this repository.  Everything below the entry points runs in
 * hand-written CUDA kernels (paper_conf_sc_munksgaardhso22_b200/csrc/); nothing here falls
 * back to the CPU.  No torch types: plain pointers, sizes and an opaque stream handle.
 *
 * What is computed (PAPER.md = /root/reference/PAPER.md, cited P:<line>):
 *   The paper's NW running example (Fig. 2) fills an int32 matrix
 *   whose row 0 and column 0 are given (the Fig. 2 loops start at 1), using Rodinia's cell
 *   function (BASELINE.json north_star; reading R1):
 *
 *       score[i][j] = max(score[i-1][j-1] + ref[i][j], score[i-1][j] - p, score[i][j-1] - p)
 *                                                                  for 1 <= i, j <= n.
 *
 *   The blocked anti-diagonal wavefront and the short-circuited in-place update
 *   (each tile's result written straight into its LMAD slice W of score, P:512-516,
 *   P:616-656) are how the kernels compute it; the result is the unique matrix fixed by the
 *   recurrence and the borders (reading R13), bit-identical to oracle/nw_ref.c.
 *
 * Conventions shared by every entry point
 *   - Matrices are row-major int32 with a leading dimension (pitch, in ELEMENTS):
 *     element (i, j) is at base[i * ld + j].  Default pitch is n + 1 (Rodinia layout).
 *   - score: row 0 and column 0 are READ-ONLY inputs (borders); rows/cols 1..n are
 *     WRITE-ONLY outputs — the interior is never read before it is written, so a call is
 *     idempotent and may be re-run after a failure.  ref: rows/cols 1..n are read; row 0 /
 *     column 0 are ignored.  ref must not overlap score.
 *   - Device pointers are owned by the caller and must be 4-byte aligned.
 *   - `stream` is a cudaStream_t (NULL = legacy default stream).  Work is ENQUEUED and the
 *     call returns; results are visible after the caller synchronises the stream.
 *   - `tile` b in {0, 16, 32, 64, 128, 256} selects the width W of the tile-column band one
 *     warp owns (W = 32K, K columns per lane): b in {0, 256} -> W = 256 (K = 8, the default),
 *     b in {16, 32, 64, 128} -> W = 128 (K = 4; narrower b x b tiles are processed 128/b side
 *     by side, because a lane's K ref values are 16-byte shared loads).  A CTA owns one band
 *     (b in {0, 256, 32, 64}: a compute warp, a ref-staging warp and two store warps) or two
 *     consecutive bands (b in {16, 128}: two compute warps on SM sub-partitions of their own,
 *     a ref and a store warp each on the other two).  The result does not depend on it
 *     (R8).
 *   - Layouts whose interior rows start 16-byte aligned ((base + 1) % 16 == 0, ld % 4 == 0,
 *     pair strides % 4 == 0, for score and ref) are staged with 16-byte copies and stores; any
 *     other 4-byte aligned layout (e.g. the Rodinia pitch n + 1) with 4-byte copies.  Same result.
 *   - Any n >= 0 is accepted (ragged last band: n need not be a multiple of b).
 *   - Validation is synchronous and happens before anything is enqueued.  Range contract:
 *     0 <= penalty and (n+1)*(2*penalty + NW_REF_MAX) < 2^30 (else NW_ERANGE); |ref| <= NW_REF_MAX
 *     and |border| <= 2^30 are the caller's promise.  Then every intermediate of the kernels'
 *     gap-normalised arithmetic (S + (i+j)*p, bounded by |border| + (n+1)*(2p + NW_REF_MAX))
 *     fits int32, and so does every cell (reading R14).
 *   - Asynchronous device faults (including the spin watchdog's trap) surface
 *     as CUDA errors at the caller's next synchronisation of the stream.
 *   - No exception or abort crosses the ABI.  Entry points are thread-safe; internal
 *     workspace (ticket counter + epoch-tagged border buffers) is cached per (device, stream)
 *     and released by nw_release_workspace().
 */
#ifndef NWB200_NW_H
#define NWB200_NW_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

#define NW_REF_MAX 1024
#define NW_ABI_VERSION 1

typedef enum {
  NW_OK = 0,
  NW_EINVAL = 1, /* null pointer, negative size, bad tile, ld < n+1, overlap, misaligned   */
  NW_ERANGE = 2, /* penalty < 0 or (n+1)*(2p + NW_REF_MAX) >= 2^30 (int32 could overflow)  */
  NW_ECUDA = 3,  /* a CUDA runtime call failed, including a workspace allocation            */
                 /* (nw_last_cuda_error() has the code)                                     */
  NW_ECOMM = 4   /* sharded call with inconsistent peer / halo description                  */
  /* (the numbering is SURVEY.md §8(b)'s) */
} nw_status;

const char* nw_status_str(int status);
int nw_abi_version(void);
int nw_last_cuda_error(void); /* cudaError_t of the last NW_ECUDA in this thread */

/* ---- single pair -------------------------------------------------------------------
 * Persistent wavefront kernel (DESIGN.md §4 "strip kernel"): one launch; warps claim
 * tile-column bands in wavefront order through an atomic ticket; band k+1 consumes band k's
 * right border column through epoch-tagged ready entries (ready flag fused with the value,
 * P:636-645 / Fig. 9 ordering); every tile is written in place (short-circuited).
 * score, ref: (n+1) x (n+1), pitch n+1. */
nw_status nw_fill(int32_t* score, const int32_t* ref, int64_t n, int32_t penalty, int32_t tile,
                  void* stream);

/* Same with explicit pitches (elements): ld_score >= n+1, ld_ref >= n+1. */
nw_status nw_fill_ld(int32_t* score, int64_t ld_score, const int32_t* ref, int64_t ld_ref,
                     int64_t n, int32_t penalty, int32_t tile, void* stream);

/* ---- batch of independent pairs (BASELINE.json config 4) ---------------------------
 * score, ref: [batch][n+1][n+1] contiguous (pair stride (n+1)^2 elements).  One launch;
 * tickets enumerate (pair, band) so pairs are independent and need no collective. */
nw_status nw_fill_batch(int32_t* score, const int32_t* ref, int64_t batch, int64_t n,
                        int32_t penalty, int32_t tile, void* stream);

/* General strided batch: pair k's score at score + k*stride_score, pitch ld_score. */
nw_status nw_fill_batch_ld(int32_t* score, int64_t ld_score, int64_t stride_score,
                           const int32_t* ref, int64_t ld_ref, int64_t stride_ref, int64_t batch,
                           int64_t n, int32_t penalty, int32_t tile, void* stream);

/* ---- one pair split into column strips across GPUs (BASELINE.json config 5) -------
 * SPMD: every rank calls this with its own strip.  Rank g owns global columns
 * (col0, col0 + w]; its LOCAL matrices are (n+1) x (w+1) with pitch ld:
 *   local score row 0 = global row 0 columns col0..col0+w (col 0 = the corner (0, col0));
 *   local score column 0, rows >= 1: the global left border (read only when halo_in == NULL,
 *   i.e. on rank 0); local ref column 0 unused.
 * halo_in  : n+2 uint64 entries on THIS device, 16-byte aligned, written by rank g-1's
 *            kernel (entry i = (epoch << 32) | (uint32) score[i][col0], i = 1..n; the kernel
 *            reads entries in 16-byte pairs, hence the spare entry n+1); NULL on rank 0.
 *            Must be zero-filled once before first use; never needs resetting after.
 * halo_out : rank g+1's halo_in (a peer-mapped pointer, e.g. torch symmetric memory, 16-byte
 *            aligned: entries are stored in 16-byte pairs) or NULL on the last rank.  A rank with halo_out needs w % nw_band_width(tile) == 0
 *            (else NW_ECOMM).  Written with st.relaxed.sys, one entry per row as soon
 *            as the row's last column is final — the NVLink border push is fused into the
 *            wavefront kernel (no host involvement, no separate send/recv).
 * epoch    : nonzero, identical on all ranks for one collective call, strictly increasing
 *            across calls that reuse the same halo buffers.  The caller must not start call
 *            e+1 on rank g+1... until every rank finished call e (one barrier per call). */
typedef struct {
  int32_t* score;
  int64_t ld_score;
  const int32_t* ref;
  int64_t ld_ref;
  int64_t n;   /* rows 1..n                                  */
  int64_t w;   /* local interior columns 1..w                */
  const uint64_t* halo_in;
  uint64_t* halo_out;
  uint32_t epoch;
  int32_t halo_out_is_peer; /* 1: halo_out lives on another GPU (system-scope stores) */
} nw_strip;

nw_status nw_fill_sharded(const nw_strip* strip, int32_t penalty, int32_t tile, void* stream);

/* ---- NEXT-2: ref generated on chip from the two sequences --------------------------
 * The step BEFORE the paper's path (Rodinia builds ref on the host): ref[i][j] =
 * subst[a[i-1]][b[j-1]] is never materialised; each band keeps a packed int8 profile
 * prof[x][lane] of its columns in shared memory.  HBM traffic drops from 8 to ~4 B/cell
 * (the score write).  Result identical to nw_fill on the materialised ref.
 * a, b     : DEVICE uint8 residue codes (< alphabet), n each (pair k at + k*stride_seq).
 * subst    : HOST int32 alphabet x alphabet table (row-major, |v| <= 127), alphabet <= 32;
 *            copied into the kernel parameters (no device allocation).
 * Codes >= alphabet are memory-safe but give unspecified scores. */
nw_status nw_fill_seq(int32_t* score, int64_t ld_score, const uint8_t* a, const uint8_t* b, int64_t n,
                      const int32_t* subst, int32_t alphabet, int32_t penalty, int32_t tile, void* stream);
nw_status nw_fill_seq_batch(int32_t* score, int64_t ld_score, int64_t stride_score, const uint8_t* a,
                            const uint8_t* b, int64_t stride_seq, int64_t batch, int64_t n,
                            const int32_t* subst, int32_t alphabet, int32_t penalty, int32_t tile,
                            void* stream);

/* ---- end to end from HOST memory (bench e2e) ---------------------------------------
 * Copies ref (rows 1..n) and the borders host->device, runs nw_fill, copies the full score
 * matrix device->host.  Host buffers: (n+1)x(n+1) int32, pitch n+1.  Pinned buffers take a
 * copy-engine pipeline: ref moves host->device in ~64 MB row blocks on one stream while the
 * kernel runs (its ref warps wait for the blocks they stage), and each score row block moves
 * back on a second stream as soon as every band has stored it (stream memory operations on
 * device counters), so both link directions and the wavefront overlap.  Pageable buffers are
 * staged (copy in, fill, copy out).  Synchronous: returns when score_host holds the result.
 * Device buffers are freed by nw_release_workspace(). */
nw_status nw_fill_host(int32_t* score_host, const int32_t* ref_host, int64_t n, int32_t penalty,
                       int32_t tile, int32_t device);
/* nw_fill_batch_host: the same for `batch` independent pairs stored back to back
 * ([batch][n+1][n+1] int32 host arrays, pair stride (n+1)^2), one launch (nw_fill_batch). */
nw_status nw_fill_batch_host(int32_t* score_host, const int32_t* ref_host, int64_t batch, int64_t n,
                             int32_t penalty, int32_t tile, int32_t device);

/* ---- NEXT-3: traceback (the step after the path; not in the paper) -------------------
 * Recovers the alignment a filled matrix scores.  From (n, n), each interior cell takes the
 * first move, in the order diagonal > up > left (reading R12), whose predecessor
 * reproduces its value under the cell function of Fig. 2 / BASELINE north_star:
 *   op 0 diagonal  S[i][j] == S[i-1][j-1] + ref[i][j]   (a_i aligned to b_j)
 *   op 1 up        S[i][j] == S[i-1][j] - p             (a_i against a gap)
 *   op 2 left      S[i][j] == S[i][j-1] - p             (gap against b_j)
 * On row 0 / column 0 the path follows the border to the origin (global alignment).
 * score, ref: DEVICE, read-only, the layout of nw_fill_ld (pair k at + k*stride elements).
 * ops:  DEVICE uint8, >= 2n bytes per pair (pair k at ops + k*ops_stride); on completion
 *       ops[0..len) holds the path in FORWARD order (origin first); bytes past len undefined.
 * len:  DEVICE int32 per pair: the path length (n..2n), or -1 if some cell on the walk
 *       matches none of its three moves (the matrix is not a fill for this ref / p).
 * ops/len must not overlap each other or score/ref.  Two launches (walk, reverse), enqueued
 * on `stream`; validation errors are returned synchronously (NW_EINVAL / NW_ERANGE). */
nw_status nw_traceback(const int32_t* score, int64_t ld_score, const int32_t* ref, int64_t ld_ref, int64_t n,
                       int32_t penalty, uint8_t* ops, int32_t* len, void* stream);
nw_status nw_traceback_batch(const int32_t* score, int64_t ld_score, int64_t stride_score, const int32_t* ref,
                             int64_t ld_ref, int64_t stride_ref, int64_t batch, int64_t n, int32_t penalty,
                             uint8_t* ops, int64_t ops_stride, int32_t* len, void* stream);

/* ---- the paper's / Rodinia's structure, kept as baselines ----------------------------
 * nw_fill_diagonal: one kernel launch per tile anti-diagonal d = 0..2q-2 (q = ceil(n/b)),
 *   one CTA per b x b tile, the tile staged in shared memory from its LMAD slices Rvert /
 *   Rhoriz (generalised to both halves in DESIGN.md §5) and written back in
 *   place into W (the "Opt." short-circuited form of P:503-521).  tile b in {16, 32, 64}.
 * nw_fill_unopt: the same schedule WITHOUT short-circuiting (the paper's "Unopt."
 *   column of Table I): each diagonal's tiles are written to a fresh temporary
 *   X[#tiles][b][b] and a second kernel copies X into W (A[W] = X).
 * Both: score/ref (n+1)x(n+1) with the given pitches; 2q-1 (resp. 2(2q-1)) launches. */
nw_status nw_fill_diagonal(int32_t* score, int64_t ld_score, const int32_t* ref, int64_t ld_ref,
                           int64_t n, int32_t penalty, int32_t tile, void* stream);
nw_status nw_fill_unopt(int32_t* score, int64_t ld_score, const int32_t* ref, int64_t ld_ref,
                        int64_t n, int32_t penalty, int32_t tile, void* stream);

/* ---- introspection (host only; used by tests/test_schedule.py and the bench) ---------- */
/* Band geometry the persistent kernel uses: band width W for `tile` (0 -> default). */
int32_t nw_band_width(int32_t tile);
/* Number of kernel launches one call of the given entry point enqueues (bench gpu_launches):
 * kind 0 = nw_fill/_ld/_batch/_sharded, 1 = nw_fill_diagonal, 2 = nw_fill_unopt. */
int64_t nw_launch_count(int32_t kind, int64_t n, int32_t tile);
/* Paper Appendix-C LMADs of tile anti-diagonal d for the diagonal kernels (element offsets
 * relative to element (0,0), pitch N): out[0..9] = {cnt, base, W.off, W.s0, W.s1, W.s2,
 * Rvert.off, Rvert.s1, Rhoriz.off, Rhoriz.s1} with shapes W = (cnt:s0,b:s1,b:s2),
 * Rvert = (cnt:s0, b+1:s1), Rhoriz = (cnt:s0, b:1).  Returns 0, or -1 for bad args. */
int32_t nw_diag_lmad(int64_t n, int64_t N, int32_t tile, int64_t d, int64_t out[10]);
/* The persistent kernel's schedule (the same __host__ __device__ helpers the kernel calls):
 * at wavefront step `step` of band `band`, lane `lane` computes row out[0], columns
 * out[1] .. out[1]+out[2]-1 (out[2] = 0: lane idle at this step).  Steps run 0 .. n+30;
 * band b+1 consumes band b's last column row by row.  Returns 0, or -1 for bad args. */
int32_t nw_strip_map(int64_t n, int64_t width, int32_t tile, int32_t band, int32_t step, int32_t lane,
                     int64_t out[3]);
/* Smem bytes / resident CTAs per SM of the strip kernel for `tile` on `device`. */
nw_status nw_kernel_info(int32_t tile, int32_t device, int64_t* smem_bytes, int32_t* ctas_per_sm,
                         int32_t* num_sms);

/* Test hook: cap the persistent kernel's grid at `grid` CTAs (0 = automatic, #SMs x
 * occupancy).  A 1-CTA grid must still finish (ticket order => deadlock freedom). */
void nw_debug_set_grid(int32_t grid);

/* Test / experiment switches (process-wide; explicit calls, never environment variables, and none
 * of them changes a result — only which kernel schedule computes it):
 *   nw_debug_set_pair_mode(mode): one-band-per-CTA kernels over a batch sweep whole pairs per
 *     ticket: 0 = automatic (batches of >= 2 pairs per SM), 1 = for any batch of >= 2 pairs,
 *     -1 = never;
 *   nw_debug_set_cluster(on): single pairs on the K = 8 kernel as thread-block clusters handing the
 *     border column over through distributed shared memory (measured slower; off by default);
 *   nw_debug_set_host_mode(mode): how nw_fill[_batch]_host treats PINNED host buffers: 2 = the
 *     copy-engine pipeline (default), 1 = zero copy (the kernel reads ref and writes score over the
 *     host link itself), 0 = staged (copy in, fill, copy out);
 *   nw_debug_set_host_block_rows(rows): the pipeline's row-block size (0 = automatic, ~64 MB);
 *   nw_debug_set_host_zero_copy(on): shorthand for nw_debug_set_host_mode(on ? 1 : 2). */
void nw_debug_set_pair_mode(int32_t mode);
void nw_debug_set_cluster(int32_t on);
void nw_debug_set_host_mode(int32_t mode);
void nw_debug_set_host_block_rows(int64_t rows);
void nw_debug_set_host_zero_copy(int32_t on);

/* Debug hook: persistent-kernel launches record, per task (pair, band) t < cap_tasks, eight
 * uint64 {t, start_ns, end_ns, smid, event_cycles, ref_wait_cycles, border_spin_cycles,
 * total_cycles} into the DEVICE buffer dev_buf (NULL = off); dev_buf must hold 16 * cap_tasks
 * uint64 (the tail gets 8 more counters per task: staging busy / wait cycles and the compute
 * warp's event sub-phases).
 * Used by bench.py --trace to measure the wavefront ramp and the band-to-band lag. */
void nw_debug_set_trace(uint64_t* dev_buf, int64_t cap_tasks);

/* Frees every cached workspace (device buffers, pinned staging).  Not thread-safe with
 * concurrent nw_* calls. */
void nw_release_workspace(void);

#ifdef __cplusplus
}
#endif
#endif /* NWB200_NW_H */
