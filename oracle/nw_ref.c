/*
 * nw_ref.c — CPU ORACLE (test infrastructure only; see nw_ref.h for who may use it).
 *
 * Plain C11, single-threaded, no SIMD intrinsics, no OpenMP.  It is the paper's
 * "Golden Sequential" loop (Fig. 2) with Rodinia's cell function
 * (BASELINE.json north_star; reading R1), written out literally:
 *
 *     for (i = 1; i <= n; i++)
 *       for (j = 1; j <= n; j++)
 *         A[i][j] = max(A[i-1][j-1] + ref[i][j], A[i-1][j] - p, A[i][j-1] - p);
 *
 * Intermediates are int64; a stored value outside int32 makes the call return -1
 * (reading R14: integers, no rounding; overflow is rejected, not wrapped).
 * Build: cc -O2 -std=c11 -shared -fPIC oracle/nw_ref.c -o oracle/liboracle.so
 */
#include "nw_ref.h"

#include <stdlib.h>
#include <string.h>

static int64_t max3(int64_t a, int64_t b, int64_t c) {
  int64_t m = a > b ? a : b;
  return m > c ? m : c;
}

static int fits_i32(int64_t v) { return v >= INT32_MIN && v <= INT32_MAX; }

int nw_ref(int32_t* score, int64_t lds, const int32_t* ref, int64_t ldr, int64_t n, int32_t p) {
  int bad = 0;
  for (int64_t i = 1; i <= n; ++i) {
    for (int64_t j = 1; j <= n; ++j) {
      int64_t diag = (int64_t)score[(i - 1) * lds + (j - 1)] + ref[i * ldr + j];
      int64_t up = (int64_t)score[(i - 1) * lds + j] - p;
      int64_t left = (int64_t)score[i * lds + (j - 1)] - p;
      int64_t v = max3(diag, up, left);
      if (!fits_i32(v)) bad = 1;
      score[i * lds + j] = (int32_t)v;
    }
  }
  return bad ? -1 : 0;
}

typedef struct {
  int64_t n;
  int32_t p;
  int32_t* prev; /* score row i-1, cols 0..n */
  int32_t* cur;  /* score row i,   cols 0..n */
} nw_stream;

void* nw_ref_stream_new(int64_t n, int32_t p, const int32_t* row0) {
  nw_stream* s = (nw_stream*)calloc(1, sizeof(nw_stream));
  if (!s) return NULL;
  s->n = n;
  s->p = p;
  s->prev = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n + 1));
  s->cur = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n + 1));
  if (!s->prev || !s->cur) {
    free(s->prev);
    free(s->cur);
    free(s);
    return NULL;
  }
  memcpy(s->prev, row0, sizeof(int32_t) * (size_t)(n + 1));
  return s;
}

int nw_ref_stream_rows(void* h, const int32_t* ref_rows, int64_t ldr, const int32_t* col0,
                       int64_t nrows, int32_t* out, int64_t ldo) {
  nw_stream* s = (nw_stream*)h;
  int bad = 0;
  const int64_t n = s->n;
  const int32_t p = s->p;
  for (int64_t k = 0; k < nrows; ++k) {
    const int32_t* r = ref_rows + k * ldr;
    s->cur[0] = col0[k];
    for (int64_t j = 1; j <= n; ++j) {
      int64_t diag = (int64_t)s->prev[j - 1] + r[j];
      int64_t up = (int64_t)s->prev[j] - p;
      int64_t left = (int64_t)s->cur[j - 1] - p;
      int64_t v = max3(diag, up, left);
      if (!fits_i32(v)) bad = 1;
      s->cur[j] = (int32_t)v;
    }
    if (out) memcpy(out + k * ldo, s->cur, sizeof(int32_t) * (size_t)(n + 1));
    int32_t* t = s->prev;
    s->prev = s->cur;
    s->cur = t;
  }
  return bad ? -1 : 0;
}

const int32_t* nw_ref_stream_last(void* h) { return ((nw_stream*)h)->prev; }

void nw_ref_stream_free(void* h) {
  nw_stream* s = (nw_stream*)h;
  if (!s) return;
  free(s->prev);
  free(s->cur);
  free(s);
}

/* Traceback (not in the paper — Rodinia's NW stops at the matrix, the
 * alignment is recovered by walking it back).  Plain definition: from (n,n), at an interior
 * cell take the first move, in the order diagonal > up > left (reading R12 = SURVEY
 * C12), whose predecessor reproduces the cell value under the Fig. 2 cell function:
 *     diagonal  S[i][j] == S[i-1][j-1] + ref[i][j]   op 0 (a_i aligned to b_j)
 *     up        S[i][j] == S[i-1][j]   - p           op 1 (a_i against a gap)
 *     left      S[i][j] == S[i][j-1]   - p           op 2 (gap against b_j)
 * On row 0 / column 0 the path follows the border to the origin (global alignment, C5):
 * ups while i > 0, lefts while j > 0.  ops[0..L) is written in forward order (origin first).
 * Returns L, or -1 if some interior cell matches none of its three moves (not a filled
 * matrix).  int64 arithmetic. */
int64_t nw_traceback_ref(const int32_t* score, int64_t lds, const int32_t* ref, int64_t ldr, int64_t n,
                         int32_t p, uint8_t* ops) {
  uint8_t* back = (uint8_t*)malloc((size_t)(2 * n + 1));
  if (!back) return -1;
  int64_t i = n, j = n, L = 0;
  while (i > 0 && j > 0) {
    int64_t v = score[i * lds + j];
    if (v == (int64_t)score[(i - 1) * lds + (j - 1)] + ref[i * ldr + j]) {
      back[L++] = 0; --i; --j;
    } else if (v == (int64_t)score[(i - 1) * lds + j] - p) {
      back[L++] = 1; --i;
    } else if (v == (int64_t)score[i * lds + (j - 1)] - p) {
      back[L++] = 2; --j;
    } else {
      free(back);
      return -1;
    }
  }
  while (i > 0) { back[L++] = 1; --i; }
  while (j > 0) { back[L++] = 2; --j; }
  for (int64_t k = 0; k < L; ++k) ops[k] = back[L - 1 - k];
  free(back);
  return L;
}
