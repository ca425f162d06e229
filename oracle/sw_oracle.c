/*
 * sw_oracle.c — ORACLE (test infrastructure only; see sw_oracle.h for who may use it).
 *
 * Plain, slow, obviously correct Smith-Waterman with Gotoh's affine gaps, written
 * as the definition in SURVEY §8(c) / PAPER.md P12 §II.A:
 *   - every cell computed, int32, two rolling rows, no banding/pruning/SIMD;
 *   - H floored at 0 with a zero first row and column (P12 §II.A.1, Eq. 1);
 *   - E, F gap matrices (P12 §II.A.3, "3 Dynamic Programming (DP) matrices: H, E and F");
 *   - the score is the highest cell of H (P12 §II.A.2).
 * Shares no code with the CUDA path.  Parity pins: tests/test_oracle.py.
 */
#include "sw_oracle.h"
#include <stdlib.h>
#include <string.h>
#include <limits.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define NEG_INF (-536870912) /* -2^29: reading R5 */

/* Reading R1: BLOSUM62, NCBI order ARNDCQEGHILKMFPSTWYVBZX*.
 * Transcribed for the oracle; checked by tests against the checksums in SURVEY §8(c)
 * item 1 (symmetry, diagonal, 20x20 sum -426, min -4, max 11, X/X -1, * / * 1). */
static const int8_t BLOSUM62[24 * 24] = {
/*        A  R  N  D  C  Q  E  G  H  I  L  K  M  F  P  S  T  W  Y  V  B  Z  X  * */
/* A */   4,-1,-2,-2, 0,-1,-1, 0,-2,-1,-1,-1,-1,-2,-1, 1, 0,-3,-2, 0,-2,-1, 0,-4,
/* R */  -1, 5, 0,-2,-3, 1, 0,-2, 0,-3,-2, 2,-1,-3,-2,-1,-1,-3,-2,-3,-1, 0,-1,-4,
/* N */  -2, 0, 6, 1,-3, 0, 0, 0, 1,-3,-3, 0,-2,-3,-2, 1, 0,-4,-2,-3, 3, 0,-1,-4,
/* D */  -2,-2, 1, 6,-3, 0, 2,-1,-1,-3,-4,-1,-3,-3,-1, 0,-1,-4,-3,-3, 4, 1,-1,-4,
/* C */   0,-3,-3,-3, 9,-3,-4,-3,-3,-1,-1,-3,-1,-2,-3,-1,-1,-2,-2,-1,-3,-3,-2,-4,
/* Q */  -1, 1, 0, 0,-3, 5, 2,-2, 0,-3,-2, 1, 0,-3,-1, 0,-1,-2,-1,-2, 0, 3,-1,-4,
/* E */  -1, 0, 0, 2,-4, 2, 5,-2, 0,-3,-3, 1,-2,-3,-1, 0,-1,-3,-2,-2, 1, 4,-1,-4,
/* G */   0,-2, 0,-1,-3,-2,-2, 6,-2,-4,-4,-2,-3,-3,-2, 0,-2,-2,-3,-3,-1,-2,-1,-4,
/* H */  -2, 0, 1,-1,-3, 0, 0,-2, 8,-3,-3,-1,-2,-1,-2,-1,-2,-2, 2,-3, 0, 0,-1,-4,
/* I */  -1,-3,-3,-3,-1,-3,-3,-4,-3, 4, 2,-3, 1, 0,-3,-2,-1,-3,-1, 3,-3,-3,-1,-4,
/* L */  -1,-2,-3,-4,-1,-2,-3,-4,-3, 2, 4,-2, 2, 0,-3,-2,-1,-2,-1, 1,-4,-3,-1,-4,
/* K */  -1, 2, 0,-1,-3, 1, 1,-2,-1,-3,-2, 5,-1,-3,-1, 0,-1,-3,-2,-2, 0, 1,-1,-4,
/* M */  -1,-1,-2,-3,-1, 0,-2,-3,-2, 1, 2,-1, 5, 0,-2,-1,-1,-1,-1, 1,-3,-1,-1,-4,
/* F */  -2,-3,-3,-3,-2,-3,-3,-3,-1, 0, 0,-3, 0, 6,-4,-2,-2, 1, 3,-1,-3,-3,-1,-4,
/* P */  -1,-2,-2,-1,-3,-1,-1,-2,-2,-3,-3,-1,-2,-4, 7,-1,-1,-4,-3,-2,-2,-1,-2,-4,
/* S */   1,-1, 1, 0,-1, 0, 0, 0,-1,-2,-2, 0,-1,-2,-1, 4, 1,-3,-2,-2, 0, 0, 0,-4,
/* T */   0,-1, 0,-1,-1,-1,-1,-2,-2,-1,-1,-1,-1,-2,-1, 1, 5,-2,-2, 0,-1,-1, 0,-4,
/* W */  -3,-3,-4,-4,-2,-2,-3,-2,-2,-3,-2,-3,-1, 1,-4,-3,-2,11, 2,-3,-4,-3,-2,-4,
/* Y */  -2,-2,-2,-3,-2,-1,-2,-3, 2,-1,-1,-2,-1, 3,-3,-2,-2, 2, 7,-1,-3,-2,-1,-4,
/* V */   0,-3,-3,-3,-1,-2,-2,-3,-3, 3, 1,-2, 1,-1,-2,-2, 0,-3,-1, 4,-3,-2,-1,-4,
/* B */  -2,-1, 3, 4,-3, 0, 1,-1, 0,-3,-4, 0,-3,-3,-2, 0,-1,-4,-3,-3, 4, 1,-1,-4,
/* Z */  -1, 0, 0, 1,-3, 3, 4,-2, 0,-3,-3, 1,-1,-3,-1, 0,-1,-3,-2,-2, 1, 4,-1,-4,
/* X */   0,-1,-1,-1,-2,-1,-1,-1,-1,-1,-1,-1,-1,-1,-2, 0, 0,-2,-1,-1,-1,-1,-1,-4,
/* * */  -4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4, 1,
};

const int8_t *sw_oracle_blosum62(void) { return BLOSUM62; }

int sw_oracle_code(int c) {
  static const char *alpha = SW_ORACLE_ALPHABET;
  if (c >= 'a' && c <= 'z') c = c - 'a' + 'A';
  for (int k = 0; k < SW_ORACLE_NCODES; k++)
    if (alpha[k] == c) return k;
  return -1;
}

static int32_t max2(int32_t a, int32_t b) { return a > b ? a : b; }

/* The recurrence of SURVEY §8(c), cell by cell, row by row (two rolling rows). */
static int32_t gotoh(const char *q, int64_t m, const char *d, int64_t n, const int8_t *S,
                     int32_t go, int32_t ge, int32_t border_init) {
  const int32_t alpha = go + ge, beta = ge;
  if (m <= 0 || n <= 0) return 0;
  int *dc = (int *)malloc(sizeof(int) * (size_t)n);
  int32_t *Hprev = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n + 1));
  int32_t *Fprev = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n + 1));
  int32_t *Hcur = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n + 1));
  int32_t *Fcur = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n + 1));
  int32_t best = 0;
  if (!dc || !Hprev || !Fprev || !Hcur || !Fcur) { best = -1; goto done; }
  for (int64_t j = 0; j < n; j++) {
    dc[j] = sw_oracle_code((unsigned char)d[j]);
    if (dc[j] < 0) { best = -1; goto done; }
  }
  for (int64_t j = 0; j <= n; j++) { Hprev[j] = 0; Fprev[j] = border_init; } /* row 0 */
  for (int64_t i = 1; i <= m; i++) {
    const int qc = sw_oracle_code((unsigned char)q[i - 1]);
    if (qc < 0) { best = -1; goto done; }
    int32_t E = border_init; /* E(i,0) */
    Hcur[0] = 0;             /* H(i,0) */
    Fcur[0] = border_init;
    for (int64_t j = 1; j <= n; j++) {
      E = max2(E - beta, Hcur[j - 1] - alpha);                      /* E(i,j) */
      Fcur[j] = max2(Fprev[j] - beta, Hprev[j] - alpha);           /* F(i,j) */
      int32_t h = Hprev[j - 1] + S[qc * SW_ORACLE_NCODES + dc[j - 1]]; /* diagonal */
      h = max2(h, E);
      h = max2(h, Fcur[j]);
      h = max2(h, 0);
      Hcur[j] = h;                                                  /* H(i,j) */
      best = max2(best, h);
    }
    int32_t *t = Hprev; Hprev = Hcur; Hcur = t;
    t = Fprev; Fprev = Fcur; Fcur = t;
  }
done:
  free(dc); free(Hprev); free(Fprev); free(Hcur); free(Fcur);
  return best;
}

static int valid_gaps(int32_t go, int32_t ge) {
  return go >= 0 && ge >= 0 && (int64_t)go + 2 * (int64_t)ge <= (1 << 20);
}

int32_t sw_oracle_pair(const char *q, int64_t m, const char *d, int64_t n,
                       const int8_t *matrix, int32_t go, int32_t ge, int32_t border_init) {
  if (!valid_gaps(go, ge) || m < 0 || n < 0 || border_init > 0 || border_init < NEG_INF) return -1;
  if ((m > 0 && !q) || (n > 0 && !d)) return -1;
  return gotoh(q, m, d, n, matrix ? matrix : BLOSUM62, go, ge, border_init);
}

int32_t sw_oracle_dump(const char *q, int64_t m, const char *d, int64_t n,
                       const int8_t *matrix, int32_t go, int32_t ge,
                       int32_t *H, int32_t *E, int32_t *F) {
  if (!valid_gaps(go, ge) || m < 0 || n < 0) return -1;
  const int8_t *S = matrix ? matrix : BLOSUM62;
  const int32_t alpha = go + ge, beta = ge;
  const int64_t W = n + 1;
  int32_t *h = (int32_t *)calloc((size_t)((m + 1) * W), sizeof(int32_t));
  int32_t *e = (int32_t *)calloc((size_t)((m + 1) * W), sizeof(int32_t));
  int32_t *f = (int32_t *)calloc((size_t)((m + 1) * W), sizeof(int32_t));
  int32_t best = 0;
  if (!h || !e || !f) { best = -1; goto done; }
  for (int64_t i = 0; i <= m; i++)
    for (int64_t j = 0; j <= n; j++) {
      h[i * W + j] = 0;
      e[i * W + j] = NEG_INF;
      f[i * W + j] = NEG_INF;
    }
  for (int64_t i = 1; i <= m; i++) {
    int qc = sw_oracle_code((unsigned char)q[i - 1]);
    if (qc < 0) { best = -1; goto done; }
    for (int64_t j = 1; j <= n; j++) {
      int dc = sw_oracle_code((unsigned char)d[j - 1]);
      if (dc < 0) { best = -1; goto done; }
      e[i * W + j] = max2(e[i * W + j - 1] - beta, h[i * W + j - 1] - alpha);
      f[i * W + j] = max2(f[(i - 1) * W + j] - beta, h[(i - 1) * W + j] - alpha);
      int32_t v = h[(i - 1) * W + j - 1] + S[qc * SW_ORACLE_NCODES + dc];
      v = max2(v, e[i * W + j]);
      v = max2(v, f[i * W + j]);
      v = max2(v, 0);
      h[i * W + j] = v;
      best = max2(best, v);
    }
  }
  if (H) memcpy(H, h, sizeof(int32_t) * (size_t)((m + 1) * W));
  if (E) memcpy(E, e, sizeof(int32_t) * (size_t)((m + 1) * W));
  if (F) memcpy(F, f, sizeof(int32_t) * (size_t)((m + 1) * W));
done:
  free(h); free(e); free(f);
  return best;
}

typedef struct { int64_t len; int32_t idx; } lenidx;
static int by_len_desc(const void *a, const void *b) {
  const lenidx *x = (const lenidx *)a, *y = (const lenidx *)b;
  if (x->len != y->len) return x->len < y->len ? 1 : -1;
  return x->idx - y->idx;
}

int sw_oracle_search(const char *q_res, const int64_t *q_off, int32_t nq,
                     const char *d_res, const int64_t *d_off, int32_t nd,
                     const int8_t *matrix, int32_t go, int32_t ge,
                     int32_t *scores, int n_threads) {
  if (!valid_gaps(go, ge) || nq < 0 || nd < 0) return -1;
  if (nq == 0 || nd == 0) return 0;
  if (!q_off || !d_off || !scores) return -1;
  const int8_t *S = matrix ? matrix : BLOSUM62;
  lenidx *order = (lenidx *)malloc(sizeof(lenidx) * (size_t)nd);
  if (!order) return -1;
  for (int32_t k = 0; k < nd; k++) { order[k].len = d_off[k + 1] - d_off[k]; order[k].idx = k; }
  qsort(order, (size_t)nd, sizeof(lenidx), by_len_desc); /* longest first */
  int err = 0;
#ifdef _OPENMP
  if (n_threads <= 0) n_threads = omp_get_num_procs();
#pragma omp parallel for schedule(dynamic, 1) num_threads(n_threads) reduction(| : err)
#endif
  for (int32_t k = 0; k < nd; k++) {
    const int32_t di = order[k].idx;
    for (int32_t qi = 0; qi < nq; qi++) {
      int32_t s = gotoh(q_res + q_off[qi], q_off[qi + 1] - q_off[qi], d_res + d_off[di],
                        d_off[di + 1] - d_off[di], S, go, ge, NEG_INF);
      if (s < 0) err = 1;
      scores[(int64_t)qi * nd + di] = s;
    }
  }
  free(order);
  return err ? -1 : 0;
}

int sw_oracle_pairs(const char *q_res, const int64_t *q_off, const char *d_res,
                    const int64_t *d_off, const int32_t *qi, const int32_t *di, int64_t npairs,
                    const int8_t *matrix, int32_t go, int32_t ge, int32_t *out, int n_threads) {
  if (!valid_gaps(go, ge) || npairs < 0) return -1;
  const int8_t *S = matrix ? matrix : BLOSUM62;
  int err = 0;
#ifdef _OPENMP
  if (n_threads <= 0) n_threads = omp_get_num_procs();
#pragma omp parallel for schedule(dynamic, 1) num_threads(n_threads) reduction(| : err)
#endif
  for (int64_t k = 0; k < npairs; k++) {
    int32_t s = gotoh(q_res + q_off[qi[k]], q_off[qi[k] + 1] - q_off[qi[k]], d_res + d_off[di[k]],
                      d_off[di[k] + 1] - d_off[di[k]], S, go, ge, NEG_INF);
    if (s < 0) err = 1;
    out[k] = s;
  }
  return err ? -1 : 0;
}

int32_t sw_alignment_score(const char *row_q, const char *row_d, int64_t len,
                           const int8_t *matrix, int32_t go, int32_t ge) {
  const int8_t *S = matrix ? matrix : BLOSUM62;
  int64_t total = 0;
  int run = 0; /* 0 none, 1 gap in d-row (query residue vs '-'), 2 gap in q-row */
  for (int64_t k = 0; k < len; k++) {
    const int a = row_q[k], b = row_d[k];
    if (a == '-' && b == '-') return INT32_MIN;
    if (a == '-') {
      total -= (run == 2) ? ge : go + ge;
      run = 2;
    } else if (b == '-') {
      total -= (run == 1) ? ge : go + ge;
      run = 1;
    } else {
      int x = sw_oracle_code(a), y = sw_oracle_code(b);
      if (x < 0 || y < 0) return INT32_MIN;
      total += S[x * SW_ORACLE_NCODES + y];
      run = 0;
    }
  }
  return (int32_t)total;
}
