/*
 * sw_oracle.h — ORACLE for the Smith-Waterman/Gotoh search hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load, call or link this library.  The
 * product path (libsw, include/sw.h) never touches it, and it shares no code,
 * headers, tables or helpers with the CUDA path.
 *
 * What it computes (the plain definition):
 *   For query q[1..m], database sequence d[1..n], substitution matrix S (24x24,
 *   NCBI order ARNDCQEGHILKMFPSTWYVBZX*, query residue = row), gap_open o >= 0,
 *   gap_extend e >= 0, alpha = o + e, beta = e:
 *     H(i,0) = H(0,j) = 0                                  PAPER.md P12 §II.A.1
 *       ("the first row and column are filled with zeroes")
 *     E(i,j) = max(E(i,j-1) - beta, H(i,j-1) - alpha)      P12 §II.A.3 (Gotoh,
 *     F(i,j) = max(F(i-1,j) - beta, H(i-1,j) - alpha)        "3 DP matrices: H, E and F")
 *     H(i,j) = max(0, H(i-1,j-1) + S[q_i][d_j], E(i,j), F(i,j))   Eq. 1 (P12)
 *     score  = max_{i,j} H(i,j)                            P12 §II.A.2
 *       ("the cell that has the highest value")
 *   A gap of length L costs o + L*e (reading R3).  E/F border values
 *   are -2^29 by default (reading R5; any value <= 0 gives the same score).
 *
 * Pins (tests/test_oracle.py): Fig. 2 score 3 (P12/P14), Fig. 1 alignment score 4
 * (P12), hand-worked affine pins, brute-force enumeration (sw_bruteforce_pair, a
 * separate file sharing no code with the DP), closed forms and invariants.
 */
#ifndef SW_ORACLE_H
#define SW_ORACLE_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

#define SW_ORACLE_ALPHABET "ARNDCQEGHILKMFPSTWYVBZX*"
#define SW_ORACLE_NCODES 24

/* ASCII letter -> index into SW_ORACLE_ALPHABET (case-insensitive); -1 if invalid. */
int sw_oracle_code(int c);

/* The BLOSUM62 table transcribed for the oracle (24x24 row-major, NCBI order). */
const int8_t *sw_oracle_blosum62(void);

/* Score of one pair.  q, d are ASCII (lengths m, n >= 0).  matrix NULL = BLOSUM62.
 * border_init = initial E(i,0) and F(0,j) value (reading R5; use -536870912 for -inf).
 * Returns the score (>= 0), or -1 on invalid residue / argument. */
int32_t sw_oracle_pair(const char *q, int64_t m, const char *d, int64_t n,
                       const int8_t *matrix, int32_t gap_open, int32_t gap_extend,
                       int32_t border_init);

/* Full-matrix dump for tiny inputs: H, E, F are caller-owned (m+1)*(n+1) int32,
 * row-major (row i = query prefix length).  Any of them may be NULL.
 * Returns the score, or -1 on error. */
int32_t sw_oracle_dump(const char *q, int64_t m, const char *d, int64_t n,
                       const int8_t *matrix, int32_t gap_open, int32_t gap_extend,
                       int32_t *H, int32_t *E, int32_t *F);

/* All pairs: scores[qi * nd + di].  Sequences in the paper's indexed format
 * (P20 §IV.B: count, offsets; residues ASCII).  OpenMP over database sequences,
 * longest first, dynamic schedule; n_threads <= 0 = all cores.
 * Returns 0, or -1 on invalid residue / argument. */
int sw_oracle_search(const char *q_res, const int64_t *q_off, int32_t nq,
                     const char *d_res, const int64_t *d_off, int32_t nd,
                     const int8_t *matrix, int32_t gap_open, int32_t gap_extend,
                     int32_t *scores, int n_threads);

/* Selected pairs only (sampled parity at full size): out[k] = score(q[qi[k]], d[di[k]]). */
int sw_oracle_pairs(const char *q_res, const int64_t *q_off, const char *d_res,
                    const int64_t *d_off, const int32_t *qi, const int32_t *di, int64_t npairs,
                    const int8_t *matrix, int32_t gap_open, int32_t gap_extend,
                    int32_t *out, int n_threads);

/* Brute force (tests only, oracle/bruteforce.c): maximum over every local alignment
 * of every pair of substrings, enumerated path by path (empty alignment = 0), each
 * maximal gap run of length L priced o + L*e.  Exponential: m, n <= 8. */
int32_t sw_bruteforce_pair(const char *q, int m, const char *d, int n,
                           const int8_t *matrix, int32_t gap_open, int32_t gap_extend);

/* Score of one given global alignment written as two equal-length gapped rows
 * ('-' = space), linear or affine: sum of S over aligned pairs minus (o + L*e) per
 * maximal gap run.  Used for the Fig. 1 pin (P12: "The score is the addition of
 * all these values").  Returns INT32_MIN on error. */
int32_t sw_alignment_score(const char *row_q, const char *row_d, int64_t len,
                           const int8_t *matrix, int32_t gap_open, int32_t gap_extend);

#ifdef __cplusplus
}
#endif
#endif
