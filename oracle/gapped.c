/*
 * gapped.c -- CPU oracle for the gapped-extension consumer of the ungapped
 * HSP hand-off (PAPER.md 3.6: "only the
 * high-scoring seeds from ungapped extension can be passed to the gapped-
 * extension stage", then "alignment with traceback").
 *
 * TEST INFRASTRUCTURE ONLY (same rule as oracle.c): only tests/ and the CPU
 * legs of bench.py load it; the product never includes or calls it.
 *
 * The paper names the stage but prints no algorithm, so every step follows a
 * DESIGN.md reading (R18-R22), written out here as plainly as possible:
 *
 *   R18 scores: the substitution matrix of the search; a gap of k residues
 *       costs gap_open + gap_extend * k (BLASTP defaults 11 / 1).
 *   R19 one direction = Gotoh's affine recurrences anchored at the seed
 *       corner (H(0,0) = 0), cells visited in row-major order (row i = i
 *       query residues consumed, column j = j subject residues consumed);
 *       "best" = the largest H seen so far (starting at 0); a cell whose H is
 *       < best - xdrop is dead (H = E = F = -inf for its successors), a cell
 *       with H > best becomes the best (the first maximum in row-major order
 *       wins).  A row with no live cell ends the extension.
 *   R20 the seed of an ungapped HSP is its middle pair (q_start + length/2,
 *       s_start + length/2); the right extension reads the query and subject
 *       forward from that pair, the left one backward from the pair before.
 *   R21 per (query, subject) the HSPs are taken in descending score (ties:
 *       canonical order, R11); an HSP whose seed lies inside the box
 *       [q_start, q_end) x [s_start, s_end) of an alignment already computed
 *       for that pair is skipped; an alignment is reported iff its score is
 *       >= cutoff.
 *   R22 traceback from the best cell: in H prefer the diagonal, then E, then
 *       F; in E / F prefer the gap open over the gap extension.
 *
 * Parity status (pins in tests/test_oracle_gapped.py): oracle_gapped_dir is
 * pinned by brute-force enumeration of every alignment path on tiny inputs
 * (xdrop large), by closed forms (identical sequences, one deletion), by a
 * hand-worked X-drop cut, and by traceback invariants (the alignment's
 * recomputed score equals the reported one); oracle_gapped_hsps by the
 * containment and ordering rules on constructed HSP lists.
 */
#include <limits.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#include "oracle.h"

#define NEG (INT32_MIN / 4) /* -infinity that survives a few subtractions */

static int32_t max2(int32_t a, int32_t b) { return a > b ? a : b; }

/* one cell of the DP: scores of the three Gotoh states */
typedef struct {
  int32_t h, e, f;
} cell;

/* one row: live columns [lo, lo + n), cells[c] = column lo + c */
typedef struct {
  int32_t lo, n;
  cell *c;
} row;

static cell get(const row *r, int32_t j) {
  cell dead = {NEG, NEG, NEG};
  if (!r || j < r->lo || j >= r->lo + r->n) return dead;
  return r->c[j - r->lo];
}

/* R19: extend from the seed corner over a[0..la) x b[0..lb).  Returns the
 * best score; *bi / *bj = residues of a / b consumed at the best cell;
 * *ident / *gopen / *glen = identities, gaps opened and gap residues on the
 * R22 traceback path.  Returns -1 (and leaves outputs 0) on allocation
 * failure. */
int32_t oracle_gapped_dir(const uint8_t *a, int32_t la, const uint8_t *b, int32_t lb,
                          const int32_t *matrix, int32_t nalpha, int32_t gap_open,
                          int32_t gap_extend, int32_t xdrop, int32_t *bi, int32_t *bj,
                          int32_t *ident, int32_t *gopen, int32_t *glen) {
  *bi = *bj = *ident = *gopen = *glen = 0;
  row *rows = calloc((size_t)la + 1, sizeof(row));
  if (!rows) return -1;
  int32_t best = 0, besti = 0, bestj = 0, nrows = 0;
  cell *buf = malloc(sizeof(cell) * ((size_t)lb + 1));
  if (!buf) {
    free(rows);
    return -1;
  }
  for (int32_t i = 0; i <= la; ++i) {
    const row *up = i > 0 ? &rows[i - 1] : NULL;
    /* a cell beyond the previous row's last live column + 1 can only be
     * reached from its left neighbour (E); once that one is dead, every
     * later cell of the row is dead too */
    const int32_t up_end = up ? up->lo + up->n : 1; /* row -1: column 0 only */
    int32_t lo = -1, hi = -1;
    for (int32_t j = 0; j <= lb; ++j) {
      cell c;
      if (i == 0 && j == 0) {
        c.h = 0;
        c.e = NEG;
        c.f = NEG;
      } else {
        const cell left = j > 0 ? buf[j - 1] : (cell){NEG, NEG, NEG};
        const cell upc = get(up, j);
        const cell diag = get(up, j - 1);
        /* row 0 / column 0 follow from the same recurrences (a leading gap) */
        c.e = j > 0 ? max2(left.e - gap_extend, left.h - gap_open - gap_extend) : NEG;
        c.f = i > 0 ? max2(upc.f - gap_extend, upc.h - gap_open - gap_extend) : NEG;
        int32_t d = NEG;
        if (i > 0 && j > 0 && diag.h > NEG)
          d = diag.h + matrix[(int32_t)a[i - 1] * nalpha + b[j - 1]];
        c.h = max2(d, max2(c.e, c.f));
        if (c.h < best - xdrop) {
          c.h = c.e = c.f = NEG; /* dead */
        } else if (c.h > best) {
          best = c.h;
          besti = i;
          bestj = j;
        }
      }
      buf[j] = c;
      if (c.h > NEG) {
        if (lo < 0) lo = j;
        hi = j;
      } else if (j >= up_end && j > 0) {
        break; /* dead, and nothing to its right can be reached */
      }
    }
    if (lo < 0) break; /* a row without live cells ends the extension */
    rows[i].lo = lo;
    rows[i].n = hi - lo + 1;
    rows[i].c = malloc(sizeof(cell) * (size_t)rows[i].n);
    if (!rows[i].c) {
      best = -1;
      break;
    }
    memcpy(rows[i].c, buf + lo, sizeof(cell) * (size_t)rows[i].n);
    nrows = i + 1;
  }
  if (best >= 0) {
    /* R22 traceback */
    int32_t i = besti, j = bestj, state = 0; /* 0 = H, 1 = E, 2 = F */
    while (i > 0 || j > 0) {
      const cell c = get(&rows[i], j);
      if (state == 0) {
        const cell diag = (i > 0 && j > 0) ? get(&rows[i - 1], j - 1) : (cell){NEG, NEG, NEG};
        const int32_t s = (i > 0 && j > 0) ? matrix[(int32_t)a[i - 1] * nalpha + b[j - 1]] : 0;
        if (i > 0 && j > 0 && diag.h > NEG && c.h == diag.h + s) {
          if (a[i - 1] == b[j - 1]) ++*ident;
          --i;
          --j;
        } else if (c.h == c.e) {
          state = 1;
        } else {
          state = 2;
        }
      } else if (state == 1) { /* gap: b[j-1] against nothing */
        ++*glen;
        const cell left = get(&rows[i], j - 1);
        if (c.e == left.h - gap_open - gap_extend) { /* the gap opens here */
          ++*gopen;
          state = 0;
        }
        --j;
      } else { /* gap: a[i-1] against nothing */
        ++*glen;
        const cell upc = get(&rows[i - 1], j);
        if (c.f == upc.h - gap_open - gap_extend) {
          ++*gopen;
          state = 0;
        }
        --i;
      }
    }
    *bi = besti;
    *bj = bestj;
  }
  for (int32_t i = 0; i < nrows; ++i) free(rows[i].c);
  free(rows);
  free(buf);
  return best;
}

static int gapped_cmp(const void *pa, const void *pb) {
  const int32_t *x = (const int32_t *)pa, *y = (const int32_t *)pb;
  for (int k = 0; k < 10; ++k)
    if (x[k] != y[k]) return x[k] < y[k] ? -1 : 1;
  return 0;
}

/* order of HSPs inside one (query, subject) pair (R21) */
static int hsp_order_cmp(const void *pa, const void *pb) {
  const oracle_hsp *x = (const oracle_hsp *)pa, *y = (const oracle_hsp *)pb;
  if (x->score != y->score) return x->score > y->score ? -1 : 1;
  const int32_t *u = (const int32_t *)x, *v = (const int32_t *)y;
  for (int k = 0; k < 7; ++k)
    if (u[k] != v[k]) return u[k] < v[k] ? -1 : 1;
  return 0;
}

/* R20-R21 over a canonical HSP list.  queries[k] / qlens[k]: codes of batch
 * query k; db codes with offsets[nseq+1] (subject i's residues at
 * db[offsets[i] .. offsets[i+1])), subject ids of the HSPs are global ids
 * minus subject_base.  Writes up to cap records (10 int32 each, canonical
 * order) to out and returns the count, or -1 on a bad HSP / allocation
 * failure. */
int64_t oracle_gapped_hsps(const uint8_t *const *queries, const int32_t *qlens, int32_t nq,
                           const uint8_t *db, const int64_t *offsets, int64_t nseq,
                           int64_t subject_base, const oracle_hsp *hsps, int64_t n,
                           const int32_t *matrix, int32_t nalpha, int32_t gap_open,
                           int32_t gap_extend, int32_t xdrop, int32_t cutoff,
                           oracle_gapped *out, int64_t cap) {
  oracle_hsp *h = malloc(sizeof(oracle_hsp) * (size_t)(n > 0 ? n : 1));
  oracle_gapped *all = malloc(sizeof(oracle_gapped) * (size_t)(n > 0 ? n : 1));
  if (!h || !all) {
    free(h);
    free(all);
    return -1;
  }
  memcpy(h, hsps, sizeof(oracle_hsp) * (size_t)n);
  int64_t nout = 0;
  int64_t g0 = 0;
  while (g0 < n) {
    int64_t g1 = g0 + 1;
    while (g1 < n && h[g1].query_id == h[g0].query_id && h[g1].subject_id == h[g0].subject_id)
      ++g1;
    qsort(h + g0, (size_t)(g1 - g0), sizeof(oracle_hsp), hsp_order_cmp);
    const int32_t qid = h[g0].query_id;
    const int64_t sidx = (int64_t)h[g0].subject_id - subject_base;
    if (qid < 0 || qid >= nq || sidx < 0 || sidx >= nseq) {
      free(h);
      free(all);
      return -1;
    }
    const uint8_t *Q = queries[qid];
    const int32_t lq = qlens[qid];
    const uint8_t *S = db + offsets[sidx];
    const int32_t ls = (int32_t)(offsets[sidx + 1] - offsets[sidx]);
    const int64_t first = nout;
    for (int64_t k = g0; k < g1; ++k) {
      const int32_t qm = h[k].q_start + h[k].length / 2;
      const int32_t sm = h[k].s_start + h[k].length / 2;
      int inside = 0;
      for (int64_t t = first; t < nout; ++t)
        if (all[t].q_start <= qm && qm < all[t].q_end && all[t].s_start <= sm && sm < all[t].s_end)
          inside = 1;
      if (inside) continue;
      /* right: Q[qm..lq) x S[sm..ls) */
      int32_t ri, rj, rid, rgo, rgl;
      const int32_t R = oracle_gapped_dir(Q + qm, lq - qm, S + sm, ls - sm, matrix, nalpha,
                                          gap_open, gap_extend, xdrop, &ri, &rj, &rid, &rgo, &rgl);
      /* left: Q[qm-1], Q[qm-2], ... x S[sm-1], ... (reversed copies) */
      uint8_t *qa = malloc((size_t)qm + 1), *sb = malloc((size_t)sm + 1);
      if (!qa || !sb || R < 0) {
        free(qa);
        free(sb);
        free(h);
        free(all);
        return -1;
      }
      for (int32_t t = 0; t < qm; ++t) qa[t] = Q[qm - 1 - t];
      for (int32_t t = 0; t < sm; ++t) sb[t] = S[sm - 1 - t];
      int32_t li, lj, lid, lgo, lgl;
      const int32_t Lsc = oracle_gapped_dir(qa, qm, sb, sm, matrix, nalpha, gap_open, gap_extend,
                                            xdrop, &li, &lj, &lid, &lgo, &lgl);
      free(qa);
      free(sb);
      if (Lsc < 0) {
        free(h);
        free(all);
        return -1;
      }
      oracle_gapped *g = &all[nout++];
      g->query_id = qid;
      g->subject_id = h[k].subject_id;
      g->q_start = qm - li;
      g->q_end = qm + ri;
      g->s_start = sm - lj;
      g->s_end = sm + rj;
      g->score = Lsc + R;
      g->ident = lid + rid;
      g->gap_opens = lgo + rgo;
      g->gap_len = lgl + rgl;
    }
    g0 = g1;
  }
  /* R21: report those with score >= cutoff, canonical order */
  int64_t m = 0;
  for (int64_t t = 0; t < nout; ++t)
    if (all[t].score >= cutoff) all[m++] = all[t];
  qsort(all, (size_t)m, sizeof(oracle_gapped), gapped_cmp);
  for (int64_t t = 0; t < m && t < cap; ++t) out[t] = all[t];
  free(h);
  free(all);
  return m;
}
