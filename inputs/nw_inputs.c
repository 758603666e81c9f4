/*
 * nw_inputs.c — seeded synthetic input generator (see include/nw_inputs.h).
 *
 * Shared by the oracle side and the CUDA side; contains no NW recurrence arithmetic.
 * Build: cc -O2 -std=c11 -shared -fPIC -Iinclude inputs/nw_inputs.c -o inputs/libnwinputs.so
 */
#include "nw_inputs.h"

#include <string.h>

uint64_t nw_splitmix64_next(uint64_t* state) {
  uint64_t z = (*state += 0x9E3779B97F4A7C15ULL);
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

uint64_t nw_pair_seed(uint64_t base, int64_t k) {
  return base ^ ((uint64_t)k * 0xD1B54A32D192ED03ULL);
}

void nw_gen_pair(uint64_t seed, int64_t n, uint8_t* a, uint8_t* b) {
  uint64_t s = seed;
  for (int64_t i = 0; i < n; ++i) a[i] = (uint8_t)(1 + nw_splitmix64_next(&s) % 10);
  for (int64_t j = 0; j < n; ++j) b[j] = (uint8_t)(1 + nw_splitmix64_next(&s) % 10);
}

void nw_gen_homologous(uint64_t seed, int64_t n, int32_t sub_per_mille, uint8_t* a, uint8_t* b) {
  uint64_t s = seed;
  for (int64_t i = 0; i < n; ++i) a[i] = (uint8_t)(1 + nw_splitmix64_next(&s) % 10);
  for (int64_t j = 0; j < n; ++j) {
    uint64_t z = nw_splitmix64_next(&s);
    if ((int64_t)(z % 1000) < (int64_t)sub_per_mille)
      b[j] = (uint8_t)(1 + nw_splitmix64_next(&s) % 10);
    else
      b[j] = a[j];
  }
}

/* BLOSUM62, NCBI order A R N D C Q E G H I L K M F P S T W Y V B Z X * (SURVEY.md App. A). */
static const int8_t B62[24 * 24] = {
     4,-1,-2,-2, 0,-1,-1, 0,-2,-1,-1,-1,-1,-2,-1, 1, 0,-3,-2, 0,-2,-1, 0,-4,
    -1, 5, 0,-2,-3, 1, 0,-2, 0,-3,-2, 2,-1,-3,-2,-1,-1,-3,-2,-3,-1, 0,-1,-4,
    -2, 0, 6, 1,-3, 0, 0, 0, 1,-3,-3, 0,-2,-3,-2, 1, 0,-4,-2,-3, 3, 0,-1,-4,
    -2,-2, 1, 6,-3, 0, 2,-1,-1,-3,-4,-1,-3,-3,-1, 0,-1,-4,-3,-3, 4, 1,-1,-4,
     0,-3,-3,-3, 9,-3,-4,-3,-3,-1,-1,-3,-1,-2,-3,-1,-1,-2,-2,-1,-3,-3,-2,-4,
    -1, 1, 0, 0,-3, 5, 2,-2, 0,-3,-2, 1, 0,-3,-1, 0,-1,-2,-1,-2, 0, 3,-1,-4,
    -1, 0, 0, 2,-4, 2, 5,-2, 0,-3,-3, 1,-2,-3,-1, 0,-1,-3,-2,-2, 1, 4,-1,-4,
     0,-2, 0,-1,-3,-2,-2, 6,-2,-4,-4,-2,-3,-3,-2, 0,-2,-2,-3,-3,-1,-2,-1,-4,
    -2, 0, 1,-1,-3, 0, 0,-2, 8,-3,-3,-1,-2,-1,-2,-1,-2,-2, 2,-3, 0, 0,-1,-4,
    -1,-3,-3,-3,-1,-3,-3,-4,-3, 4, 2,-3, 1, 0,-3,-2,-1,-3,-1, 3,-3,-3,-1,-4,
    -1,-2,-3,-4,-1,-2,-3,-4,-3, 2, 4,-2, 2, 0,-3,-2,-1,-2,-1, 1,-4,-3,-1,-4,
    -1, 2, 0,-1,-3, 1, 1,-2,-1,-3,-2, 5,-1,-3,-1, 0,-1,-3,-2,-2, 0, 1,-1,-4,
    -1,-1,-2,-3,-1, 0,-2,-3,-2, 1, 2,-1, 5, 0,-2,-1,-1,-1,-1, 1,-3,-1,-1,-4,
    -2,-3,-3,-3,-2,-3,-3,-3,-1, 0, 0,-3, 0, 6,-4,-2,-2, 1, 3,-1,-3,-3,-1,-4,
    -1,-2,-2,-1,-3,-1,-1,-2,-2,-3,-3,-1,-2,-4, 7,-1,-1,-4,-3,-2,-2,-1,-2,-4,
     1,-1, 1, 0,-1, 0, 0, 0,-1,-2,-2, 0,-1,-2,-1, 4, 1,-3,-2,-2, 0, 0, 0,-4,
     0,-1, 0,-1,-1,-1,-1,-2,-2,-1,-1,-1,-1,-2,-1, 1, 5,-2,-2, 0,-1,-1, 0,-4,
    -3,-3,-4,-4,-2,-2,-3,-2,-2,-3,-2,-3,-1, 1,-4,-3,-2,11, 2,-3,-4,-3,-2,-4,
    -2,-2,-2,-3,-2,-1,-2,-3, 2,-1,-1,-2,-1, 3,-3,-2,-2, 2, 7,-1,-3,-2,-1,-4,
     0,-3,-3,-3,-1,-2,-2,-3,-3, 3, 1,-2, 1,-1,-2,-2, 0,-3,-1, 4,-3,-2,-1,-4,
    -2,-1, 3, 4,-3, 0, 1,-1, 0,-3,-4, 0,-3,-3,-2, 0,-1,-4,-3,-3, 4, 1,-1,-4,
    -1, 0, 0, 1,-3, 3, 4,-2, 0,-3,-3, 1,-1,-3,-1, 0,-1,-3,-2,-2, 1, 4,-1,-4,
     0,-1,-1,-1,-2,-1,-1,-1,-1,-1,-1,-1,-1,-1,-2, 0, 0,-2,-1,-1,-1,-1,-1,-4,
    -4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4, 1,
};

const int8_t* nw_blosum62(void) { return B62; }
const char* nw_blosum62_alphabet(void) { return "ARNDCQEGHILKMFPSTWYVBZX*"; }

void nw_build_ref_block(int32_t* out, int64_t ld_out, const uint8_t* a, const uint8_t* b,
                        int64_t n, int64_t row_begin, int64_t row_end) {
  if (row_begin < 1) row_begin = 1;
  if (row_end > n + 1) row_end = n + 1;
  for (int64_t i = row_begin; i < row_end; ++i) {
    const int8_t* trow = B62 + 24 * (int)a[i - 1];
    int32_t* o = out + (i - row_begin) * ld_out;
    for (int64_t j = 1; j <= n; ++j) o[j] = trow[b[j - 1]];
  }
}

void nw_build_ref_rows(int32_t* ref, int64_t ld, const uint8_t* a, const uint8_t* b,
                       int64_t n, int64_t row_begin, int64_t row_end) {
  if (row_begin < 1) row_begin = 1;
  nw_build_ref_block(ref + row_begin * ld, ld, a, b, n, row_begin, row_end);
}

void nw_init_borders(int32_t* score, int64_t ld, int64_t n, int32_t p) {
  for (int64_t j = 0; j <= n; ++j) score[j] = (int32_t)(-j * (int64_t)p);
  for (int64_t i = 0; i <= n; ++i) score[i * ld] = (int32_t)(-i * (int64_t)p);
}

void nw_fill_interior(int32_t* score, int64_t ld, int64_t n, int32_t value) {
  for (int64_t i = 1; i <= n; ++i)
    for (int64_t j = 1; j <= n; ++j) score[i * ld + j] = value;
}
