/*
 * bruteforce.c — exhaustive local-alignment enumerator (TEST INFRASTRUCTURE ONLY).
 *
 * Pins the oracle's DP (sw_oracle.c) without sharing any of its code: it never
 * forms H, E or F.  It walks every alignment path explicitly.  A local alignment
 * (P12 §II.A: "optimal pairwise local alignment") of q and d is an alignment of a
 * substring of q with a substring of d: a start point (i0, j0) followed by a
 * sequence of columns, each one of
 *   'M'  q_i over d_j           scores S[q_i][d_j]       (P12: ma / mi)
 *   'I'  q_i over a space       (a gap in d)
 *   'D'  a space over d_j       (a gap in q)
 * where every maximal run of L columns of the same gap kind costs o + L*e
 * (reading R3; P12 §II.A.3 "a higher penalty ... to the first gap and a lower
 * penalty ... to the following ones").  The empty alignment scores 0.  The result
 * is the maximum over all of them.
 */
#include "sw_oracle.h"
#include <stdint.h>

typedef struct {
  const int *q, *d;
  int m, n;
  const int8_t *S;
  int32_t go, ge;
  int32_t best;
} bf_ctx;

/* last: 0 = start / after 'M', 1 = after 'I', 2 = after 'D' */
static void walk(bf_ctx *c, int i, int j, int last, int32_t score) {
  if (score > c->best) c->best = score;
  if (i < c->m && j < c->n)
    walk(c, i + 1, j + 1, 0, score + c->S[c->q[i] * SW_ORACLE_NCODES + c->d[j]]);
  if (i < c->m) walk(c, i + 1, j, 1, score - (last == 1 ? c->ge : c->go + c->ge));
  if (j < c->n) walk(c, i, j + 1, 2, score - (last == 2 ? c->ge : c->go + c->ge));
}

int32_t sw_bruteforce_pair(const char *q, int m, const char *d, int n,
                           const int8_t *matrix, int32_t go, int32_t ge) {
  if (m < 0 || n < 0 || m > 8 || n > 8 || go < 0 || ge < 0) return -1;
  int qc[8], dc[8];
  for (int i = 0; i < m; i++) if ((qc[i] = sw_oracle_code((unsigned char)q[i])) < 0) return -1;
  for (int j = 0; j < n; j++) if ((dc[j] = sw_oracle_code((unsigned char)d[j])) < 0) return -1;
  bf_ctx c = {qc, dc, m, n, matrix ? matrix : sw_oracle_blosum62(), go, ge, 0};
  for (int i0 = 0; i0 <= m; i0++)
    for (int j0 = 0; j0 <= n; j0++) walk(&c, i0, j0, 0, 0);
  return c.best;
}
