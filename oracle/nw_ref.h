/*
 * nw_ref.h — CPU ORACLE for Needleman–Wunsch score-matrix fill.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg
 * may load or call this.  The product library (paper_conf_sc_munksgaardhso22_b200/) never
 * includes, links or calls it, and it shares no code with the CUDA path.
 *
 * What it computes — the paper's "Golden Sequential" NW loop, Fig. 2 (PAPER.md P:371-381,
 * P:418-420): for i = 1..n, j = 1..n
 *     score[i][j] = max(score[i-1][j-1] + ref[i][j],  score[i-1][j] - p,  score[i][j-1] - p)
 * The cell function f of Fig. 2 is never written out in the paper (it only shows the
 * dependence A[i,j] = f(A[i-1,j], A[i,j-1], A[i-1,j-1])); we take Rodinia's f as stated
 * in BASELINE.json north_star (reading R1 = SURVEY.md C1).  Row 0 and column 0
 * are inputs and are never written (the Fig. 2 loops start at 1).
 *
 * Pins (tests/test_oracle.py): hand example (tests/golden/appendix_b.txt), brute-force
 * enumeration of all alignments for n <= 8 (standard and arbitrary borders), the
 * constant-ref closed form, border-shift / transpose metamorphics, bounds, and an
 * independent max-plus prefix-scan formulation.  nw_traceback_ref is pinned separately
 * (tests/test_traceback_oracle.py): hand example, brute force over every alignment for n <= 6
 * with the tie rule, and the path's independently summed score.  Every function here is pinned.
 */
#ifndef NW_REF_H
#define NW_REF_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

/* Full-matrix oracle.  score, ref: (n+1) x (n+1) row-major, leading dims lds/ldr.
 * Reads row 0 / col 0 of score (borders) and rows/cols 1..n of ref; writes the interior.
 * Returns 0, or -1 if some cell value does not fit in int32 (int64 intermediates). */
int nw_ref(int32_t* score, int64_t lds, const int32_t* ref, int64_t ldr, int64_t n, int32_t p);

/* Row-streaming oracle, O(n) memory: the same loop, one row at a time.
 *   h = nw_ref_stream_new(n, p, row0)     row0[0..n] = score row 0 (copied)
 *   nw_ref_stream_rows(h, ref_rows, ldr, col0, nrows, out, ldo)
 *        consumes the next `nrows` rows: ref_rows + k*ldr is ref row (i0+k) (cols 0..n,
 *        col 0 unused), col0[k] = score[i0+k][0]; writes score row i0+k (cols 0..n) to
 *        out + k*ldo (out may be NULL).  Returns 0 or -1 on int32 overflow.
 *   nw_ref_stream_last(h) -> pointer to the last computed row (n+1 values).
 *   nw_ref_stream_free(h) */
void* nw_ref_stream_new(int64_t n, int32_t p, const int32_t* row0);
int nw_ref_stream_rows(void* h, const int32_t* ref_rows, int64_t ldr, const int32_t* col0,
                       int64_t nrows, int32_t* out, int64_t ldo);
const int32_t* nw_ref_stream_last(void* h);
void nw_ref_stream_free(void* h);

/* Traceback of a filled matrix (NEXT-3): ops[0..L) in forward order, 0 = diagonal, 1 = up
 * (a_i vs gap), 2 = left (gap vs b_j); tie order diagonal > up > left; border cells follow the
 * border to the origin.  ops needs 2n bytes.  Returns L or -1 (a cell matches no move). */
int64_t nw_traceback_ref(const int32_t* score, int64_t lds, const int32_t* ref, int64_t ldr, int64_t n,
                         int32_t p, uint8_t* ops);

#ifdef __cplusplus
}
#endif
#endif
