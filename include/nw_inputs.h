/*
 * nw_inputs.h — seeded synthetic INPUT generator for Needleman–Wunsch (host, plain C).
 *
 * This module is shared by the oracle side (tests, bench cpu_baseline) and the CUDA side
 * (tests, bench, smoke).  It holds NONE of the method's arithmetic: it only draws random
 * sequences, looks up the substitution table and writes the border convention the
 * method's input contract asks for.  The NW recurrence itself lives
 * in oracle/ (CPU) and in the product library (CUDA) — never here.
 *
 * Paper context (PAPER.md = /root/reference/PAPER.md, cited as P:<line>):
 *   - the NW running example is Rodinia's NW; the paper never states the
 *     substitution table, alphabet, sequences or seeds (SURVEY.md §8c reading C2), so we
 *     follow Rodinia's convention: BLOSUM62, residues uniform on table indices 1..10.
 *   - row 0 and column 0 are inputs (Fig. 2 loops start at 1); global alignment
 *     borders score[0][j] = -j*p, score[i][0] = -i*p (reading C5).
 *
 * Sequence convention (reading C2): splitmix64 seeded with `seed`; draw a[0..n-1] then
 * b[0..n-1], residue = 1 + (z mod 10).  a[i-1] labels matrix row i, b[j-1] column j.
 * Batch pair k uses seed nw_pair_seed(7, k) = 7 ^ (k * 0xD1B54A32D192ED03).
 *
 * Layouts: matrices are row-major (n+1) x (n+1) int32 with leading dimension `ld`
 * (elements, ld >= n+1).  All pointers are HOST pointers owned by the caller.
 */
#ifndef NW_INPUTS_H
#define NW_INPUTS_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

/* splitmix64 step (Steele, Lea, Flood 2014): advances *state, returns the next 64-bit value. */
uint64_t nw_splitmix64_next(uint64_t* state);

/* Seed of batch pair k: base ^ (k * 0xD1B54A32D192ED03). */
uint64_t nw_pair_seed(uint64_t base, int64_t k);

/* Rodinia-style random pair: a[0..n-1], b[0..n-1] in 1..10 (BLOSUM62 indices R..L). */
void nw_gen_pair(uint64_t seed, int64_t n, uint8_t* a, uint8_t* b);

/* Homologous pair: a random as above; b = a with each position substituted (new uniform
 * residue in 1..10) with probability `sub_per_mille`/1000, from the same splitmix stream. */
void nw_gen_homologous(uint64_t seed, int64_t n, int32_t sub_per_mille, uint8_t* a, uint8_t* b);

/* The 24x24 BLOSUM62 table, NCBI order "ARNDCQEGHILKMFPSTWYVBZX*" (row-major int8). */
const int8_t* nw_blosum62(void);
const char* nw_blosum62_alphabet(void);

/* ref[i][j] = B62[a[i-1]][b[j-1]] for rows i in [row_begin, row_end) (1 <= i <= n), j in
 * 1..n.  Row/col 0 of ref are left untouched (unused by the method). `ref` points at
 * element (0,0) of the full matrix. */
void nw_build_ref_rows(int32_t* ref, int64_t ld, const uint8_t* a, const uint8_t* b,
                       int64_t n, int64_t row_begin, int64_t row_end);

/* Same, writing row i into out + (i - row_begin) * ld_out (a row block buffer). */
void nw_build_ref_block(int32_t* out, int64_t ld_out, const uint8_t* a, const uint8_t* b,
                        int64_t n, int64_t row_begin, int64_t row_end);

/* Global-alignment borders: score[0][j] = -j*p, score[i][0] = -i*p (reading C5). */
void nw_init_borders(int32_t* score, int64_t ld, int64_t n, int32_t p);

/* Fill the interior (rows/cols 1..n) with `value` (sentinel pre-fill for parity tests). */
void nw_fill_interior(int32_t* score, int64_t ld, int64_t n, int32_t value);

#ifdef __cplusplus
}
#endif
#endif
