/*
 * oracle.c -- CPU oracle for the cuBLASTP hot path.  TEST INFRASTRUCTURE
 * ONLY (see oracle.h).  Shares no code, header, table or constant generator
 * with the CUDA path; the two never include each other.
 *
 * Each step follows PAPER.md (P:L<n> = line of /root/reference/PAPER.md)
 * in the paper's order, with the readings R1..R13 of SURVEY.md section 8(c)
 * where the paper is silent or garbled (listed in DESIGN.md):
 *
 *   hit detection        Alg. 1 L1-4, Fig. 3
 *   diagonal             d = s - q            (R5)
 *   two-hit filter       P:L1344-1351         (R6)
 *   coverage / ext_reach Alg. 3 L12-23        (R10)
 *   hit-based extension  Alg. 4 L9-14          (ext_mode 1)
 *   X-drop extension     Fig. 8, P:L1579-1693 (R7-R9)
 *
 * Build: gcc -O2 -std=c99 -shared -fPIC -pthread oracle.c -o liboracle.so
 */
#define _POSIX_C_SOURCE 200809L
#include "oracle.h"

#include <pthread.h>
#include <stdlib.h>
#include <string.h>

/* ---------------------------------------------------------------- R1, R2 */

const char ORACLE_ALPHABET[ORACLE_NA + 1] = "ARNDCQEGHILKMFPSTWYVBZX*";

/* NCBI BLOSUM62 in the order above.  PAPER.md names
 * BLOSUM62 but does not print it. */
const int32_t ORACLE_BLOSUM62[ORACLE_NA * ORACLE_NA] = {
/*       A  R  N  D  C  Q  E  G  H  I  L  K  M  F  P  S  T  W  Y  V  B  Z  X  * */
/* A */  4,-1,-2,-2, 0,-1,-1, 0,-2,-1,-1,-1,-1,-2,-1, 1, 0,-3,-2, 0,-2,-1, 0,-4,
/* R */ -1, 5, 0,-2,-3, 1, 0,-2, 0,-3,-2, 2,-1,-3,-2,-1,-1,-3,-2,-3,-1, 0,-1,-4,
/* N */ -2, 0, 6, 1,-3, 0, 0, 0, 1,-3,-3, 0,-2,-3,-2, 1, 0,-4,-2,-3, 3, 0,-1,-4,
/* D */ -2,-2, 1, 6,-3, 0, 2,-1,-1,-3,-4,-1,-3,-3,-1, 0,-1,-4,-3,-3, 4, 1,-1,-4,
/* C */  0,-3,-3,-3, 9,-3,-4,-3,-3,-1,-1,-3,-1,-2,-3,-1,-1,-2,-2,-1,-3,-3,-2,-4,
/* Q */ -1, 1, 0, 0,-3, 5, 2,-2, 0,-3,-2, 1, 0,-3,-1, 0,-1,-2,-1,-2, 0, 3,-1,-4,
/* E */ -1, 0, 0, 2,-4, 2, 5,-2, 0,-3,-3, 1,-2,-3,-1, 0,-1,-3,-2,-2, 1, 4,-1,-4,
/* G */  0,-2, 0,-1,-3,-2,-2, 6,-2,-4,-4,-2,-3,-3,-2, 0,-2,-2,-3,-3,-1,-2,-1,-4,
/* H */ -2, 0, 1,-1,-3, 0, 0,-2, 8,-3,-3,-1,-2,-1,-2,-1,-2,-2, 2,-3, 0, 0,-1,-4,
/* I */ -1,-3,-3,-3,-1,-3,-3,-4,-3, 4, 2,-3, 1, 0,-3,-2,-1,-3,-1, 3,-3,-3,-1,-4,
/* L */ -1,-2,-3,-4,-1,-2,-3,-4,-3, 2, 4,-2, 2, 0,-3,-2,-1,-2,-1, 1,-4,-3,-1,-4,
/* K */ -1, 2, 0,-1,-3, 1, 1,-2,-1,-3,-2, 5,-1,-3,-1, 0,-1,-3,-2,-2, 0, 1,-1,-4,
/* M */ -1,-1,-2,-3,-1, 0,-2,-3,-2, 1, 2,-1, 5, 0,-2,-1,-1,-1,-1, 1,-3,-1,-1,-4,
/* F */ -2,-3,-3,-3,-2,-3,-3,-3,-1, 0, 0,-3, 0, 6,-4,-2,-2, 1, 3,-1,-3,-3,-1,-4,
/* P */ -1,-2,-2,-1,-3,-1,-1,-2,-2,-3,-3,-1,-2,-4, 7,-1,-1,-4,-3,-2,-2,-1,-2,-4,
/* S */  1,-1, 1, 0,-1, 0, 0, 0,-1,-2,-2, 0,-1,-2,-1, 4, 1,-3,-2,-2, 0, 0, 0,-4,
/* T */  0,-1, 0,-1,-1,-1,-1,-2,-2,-1,-1,-1,-1,-2,-1, 1, 5,-2,-2, 0,-1,-1, 0,-4,
/* W */ -3,-3,-4,-4,-2,-2,-3,-2,-2,-3,-2,-3,-1, 1,-4,-3,-2,11, 2,-3,-4,-3,-2,-4,
/* Y */ -2,-2,-2,-3,-2,-1,-2,-3, 2,-1,-1,-2,-1, 3,-3,-2,-2, 2, 7,-1,-3,-2,-1,-4,
/* V */  0,-3,-3,-3,-1,-2,-2,-3,-3, 3, 1,-2, 1,-1,-2,-2, 0,-3,-1, 4,-3,-2,-1,-4,
/* B */ -2,-1, 3, 4,-3, 0, 1,-1, 0,-3,-4, 0,-3,-3,-2, 0,-1,-4,-3,-3, 4, 1,-1,-4,
/* Z */ -1, 0, 0, 1,-3, 3, 4,-2, 0,-3,-3, 1,-1,-3,-1, 0,-1,-3,-2,-2, 1, 4,-1,-4,
/* X */  0,-1,-1,-1,-2,-1,-1,-1,-1,-1,-1,-1,-1,-1,-2, 0, 0,-2,-1,-1,-1,-1,-1,-4,
/* * */ -4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4,-4, 1,
};

int64_t oracle_encode(const char *ascii, int64_t n, uint8_t *codes) {
  for (int64_t i = 0; i < n; ++i) {
    char c = ascii[i];
    if (c >= 'a' && c <= 'z') c = (char)(c - 'a' + 'A');
    if (c == 'U' || c == 'O' || c == 'J') c = 'X';
    const char *hit = NULL;
    for (int k = 0; k < ORACLE_NA; ++k)
      if (ORACLE_ALPHABET[k] == c) { hit = &ORACLE_ALPHABET[k]; break; }
    if (!hit || c == '\0') return -(i + 1);
    codes[i] = (uint8_t)(hit - ORACLE_ALPHABET);
  }
  return 0;
}

/* -------------------------------------------------------------------- R3 */

static int64_t ipow(int64_t b, int32_t e) {
  int64_t r = 1;
  while (e-- > 0) r *= b;
  return r;
}

/* Score of query word at q against word v (letters of v most-significant
 * first, i.e. v = v_0*na^(w-1) + ... + v_(w-1)). */
static int32_t word_score(const uint8_t *query, int32_t q, int64_t v,
                          const int32_t *matrix, int32_t na, int32_t w) {
  int32_t sc = 0;
  for (int32_t i = w - 1; i >= 0; --i) {
    int32_t letter = (int32_t)(v % na);
    v /= na;
    sc += matrix[query[q + i] * na + letter];
  }
  return sc;
}

int64_t oracle_neighbourhood(const uint8_t *query, int32_t lq,
                             const int32_t *matrix, int32_t na,
                             int32_t word_len, int32_t T, int64_t *off,
                             int32_t *pos, int64_t cap) {
  const int64_t nwords = ipow(na, word_len);
  for (int64_t v = 0; v <= nwords; ++v) off[v] = 0;
  /* pass 1: count (DFA "query positions" per word) */
  for (int32_t q = 0; q + word_len <= lq; ++q)
    for (int64_t v = 0; v < nwords; ++v)
      if (word_score(query, q, v, matrix, na, word_len) >= T) off[v + 1]++;
  for (int64_t v = 0; v < nwords; ++v) off[v + 1] += off[v];
  const int64_t total = off[nwords];
  if (total > cap || pos == NULL) return total;
  /* pass 2: fill, q ascending within each word */
  int64_t *cursor = (int64_t *)malloc(sizeof(int64_t) * (size_t)nwords);
  if (!cursor) return -1;
  for (int64_t v = 0; v < nwords; ++v) cursor[v] = off[v];
  for (int32_t q = 0; q + word_len <= lq; ++q)
    for (int64_t v = 0; v < nwords; ++v)
      if (word_score(query, q, v, matrix, na, word_len) >= T)
        pos[cursor[v]++] = q;
  free(cursor);
  return total;
}

/* -------------------------------------------------------------------- R8 */

void oracle_xdrop_pairs(const uint8_t *a, const uint8_t *b, int32_t n,
                        int32_t step, const int32_t *matrix, int32_t na,
                        int32_t X, int32_t *best, int32_t *len,
                        int32_t *steps) {
  /* Fig. 8: running (prefix) score from the hit, the highest
   * score so far, and the drop since it; stop when the drop reaches X.  The
   * best is the shortest prefix attaining the maximum (strict >), and the
   * empty extension (score 0) is allowed. */
  int32_t run = 0, bst = 0, bl = 0, k = 0;
  for (k = 0; k < n; ++k) {
    run += matrix[a[(int64_t)k * step] * na + b[(int64_t)k * step]];
    if (run > bst) { bst = run; bl = k + 1; }
    if (bst - run >= X) { ++k; break; }
  }
  *best = bst;
  *len = bl;
  *steps = k;
}

/* -------------------------------------------------------------------- R6 */

void oracle_two_hit(const int32_t *s, int32_t n, int32_t min_gap,
                    int32_t window, int32_t mode, uint8_t *pass) {
  /* "A thread scheduled for one hit compares the distance to its neighbor
   * on left. If the distance to the neighbor is less than the threshold,
   * the hit is kept", with the non-overlap rule W <= h-p. */
  for (int32_t k = 0; k < n; ++k) {
    pass[k] = 0;
    for (int32_t m = 0; m < n; ++m) {
      int32_t dist = s[k] - s[m];
      if (mode == 1 && dist < 0) dist = -dist;
      if (dist >= min_gap && dist < window) { pass[k] = 1; break; }
    }
  }
}

/* Alg. 1 L8-19, filter_mode 2 (STATEFUL; reading R15): walk
 * the hits of one diagonal in ascending s with one `lasthit`.  distance =
 * h - lasthit; no lasthit (first hit of the diagonal in this subject) or
 * distance >= window: lasthit <- h (L17-19); min_gap <= distance < window:
 * extend from h (L12-14) and lasthit <- the end of the extension, ext.sub_pos
 * (L15-16; R10 reads it as the HSP's subject end, inclusive); distance <
 * min_gap (an overlapping word, or a hit inside the last extension): no
 * change (FSA-BLAST's rule, R15).  end_of(ctx, k) returns the subject end of
 * the extension from hit k, which does not depend on the walk (R7). */
typedef int32_t (*ext_end_fn)(void *ctx, int32_t k, int32_t *start);

/* filter_mode 3 adds Alg. 1 L13's second argument, ungapped_ext(hit_k,
 * lasthit) (reading R16): the extension from h is kept only if it
 * reaches back to the last hit -- its subject start is at or before
 * lasthit (the two-hit pair lies inside one ungapped alignment, as in
 * NCBI/FSA BLAST's two-hit method).  An extension that does not reach back
 * is dropped (no output) and h becomes the diagonal's last hit (L19).
 * end_of also returns the extension's subject start through *start. */
static void stateful_walk(const int32_t *s, int32_t n, int32_t min_gap,
                          int32_t window, int reach_back, ext_end_fn end_of,
                          void *ctx, uint8_t *trigger) {
  int32_t have = 0, lasthit = 0;
  for (int32_t k = 0; k < n; ++k) {
    trigger[k] = 0;
    const int32_t h = s[k];
    if (!have || h - lasthit >= window) { /* L17-19 */
      lasthit = h;
      have = 1;
      continue;
    }
    if (h - lasthit < min_gap) continue; /* R15 */
    int32_t start = 0;
    const int32_t end = end_of(ctx, k, &start); /* L13 */
    if (reach_back && start > lasthit) {        /* R16: not reaching back */
      lasthit = h;
      continue;
    }
    trigger[k] = 1;                      /* L11-14 */
    lasthit = end;                       /* L15-16 */
  }
}

typedef struct {
  const int32_t *start, *end;
} ext_arrays;

static int32_t end_from_array(void *ctx, int32_t k, int32_t *start) {
  const ext_arrays *a = (const ext_arrays *)ctx;
  *start = a->start ? a->start[k] : 0;
  return a->end[k];
}

void oracle_two_hit_stateful(const int32_t *s, int32_t n,
                             const int32_t *ext_end, int32_t min_gap,
                             int32_t window, uint8_t *trigger) {
  ext_arrays a = {0, ext_end};
  stateful_walk(s, n, min_gap, window, 0, end_from_array, &a, trigger);
}

void oracle_two_hit_stateful_rb(const int32_t *s, int32_t n,
                                const int32_t *ext_start,
                                const int32_t *ext_end, int32_t min_gap,
                                int32_t window, uint8_t *trigger) {
  ext_arrays a = {ext_start, ext_end};
  stateful_walk(s, n, min_gap, window, 1, end_from_array, &a, trigger);
}

/* ---------------------------------------------------------- search, R4-R11 */

typedef struct {
  oracle_hsp *v;
  int64_t n, cap;
} hsp_vec;

static int hsp_push(hsp_vec *vec, const oracle_hsp *h) {
  if (vec->n == vec->cap) {
    int64_t nc = vec->cap ? vec->cap * 2 : 256;
    oracle_hsp *nv = (oracle_hsp *)realloc(vec->v, sizeof(oracle_hsp) * (size_t)nc);
    if (!nv) return -1;
    vec->v = nv;
    vec->cap = nc;
  }
  vec->v[vec->n++] = *h;
  return 0;
}

static int hsp_cmp(const void *pa, const void *pb) {
  /* R11: lexicographic on (query_id, subject_id, diagonal, q_start,
   * s_start, length, score). */
  const int32_t *a = (const int32_t *)pa, *b = (const int32_t *)pb;
  for (int i = 0; i < 7; ++i)
    if (a[i] != b[i]) return a[i] < b[i] ? -1 : 1;
  return 0;
}

static void hitlist_push(oracle_hitlist *hl, int32_t subj, int32_t q,
                         int32_t s) {
  if (!hl) return;
  if (hl->count < hl->cap) {
    hl->subject[hl->count] = subj;
    hl->q[hl->count] = q;
    hl->s[hl->count] = s;
  }
  hl->count++;
}

typedef struct {
  /* inputs */
  const uint8_t *query;
  int32_t lq, query_id;
  const uint8_t *db;
  const int64_t *offsets;
  int64_t first, last; /* subject range [first, last) */
  int64_t subject_base;
  const int32_t *matrix;
  int32_t na;
  const oracle_params *p;
  const int64_t *off;
  const int32_t *pos;
  oracle_hitlist *hits, *passing;
  int collect_ext; /* keep every extension (else only count them) */
  int64_t cur_subject; /* subject being searched (index in offsets) */
  /* outputs */
  hsp_vec out, ext;
  int err;
} range_job;

/* R7-R9: the extension from the hit at subject position h of diagonal d:
 * seed word [q, q+w) x [h, h+w), then independent X-drop to the right (from
 * q+w, h+w) and to the left (from q-1, h-1).  Returns the HSP's subject end
 * (inclusive), the ext_reach / lasthit value of R10 / R15. */
static int32_t extend_hit(const range_job *J, const uint8_t *S, int32_t ls,
                          int32_t d, int32_t h, oracle_hsp *e) {
  const oracle_params *p = J->p;
  const int32_t w = p->word_len, lq = J->lq, na = J->na, q = h - d;
  int32_t s0 = 0;
  for (int32_t k2 = 0; k2 < w; ++k2)
    s0 += J->matrix[J->query[q + k2] * na + S[h + k2]];
  int32_t nr = lq - (q + w), nl = q;
  if (ls - (h + w) < nr) nr = ls - (h + w);
  if (h < nl) nl = h;
  int32_t bestR, rlen, stepsR, bestL, llen, stepsL;
  oracle_xdrop_pairs(J->query + q + w, S + h + w, nr, +1, J->matrix, na,
                     p->xdrop, &bestR, &rlen, &stepsR);
  oracle_xdrop_pairs(J->query + q - 1, S + h - 1, nl, -1, J->matrix, na,
                     p->xdrop, &bestL, &llen, &stepsL);
  e->query_id = J->query_id;
  e->subject_id = (int32_t)(J->subject_base + J->cur_subject);
  e->diagonal = d;
  e->q_start = q - llen;
  e->s_start = h - llen;
  e->length = llen + w + rlen;
  e->score = s0 + bestL + bestR;
  return h + w - 1 + rlen; /* HSP subject end, inclusive */
}

/* Keep an extension (every one, emitted or not) and emit it iff its score
 * reaches the cutoff (R10).  Nonzero on allocation failure. */
static int record_ext(range_job *J, const oracle_hsp *e) {
  if (J->collect_ext) {
    if (hsp_push(&J->ext, e)) return 1;
  } else {
    J->ext.n++;
  }
  if (e->score >= J->p->cutoff && hsp_push(&J->out, e)) return 1;
  return 0;
}

typedef struct {
  range_job *J;
  const uint8_t *S;
  int32_t ls, d;
  const int32_t *H;
  oracle_hsp scratch;
} ext_ctx;

static int32_t ext_end_of(void *ctx, int32_t k, int32_t *start) {
  ext_ctx *X = (ext_ctx *)ctx;
  const int32_t end = extend_hit(X->J, X->S, X->ls, X->d, X->H[k], &X->scratch);
  *start = X->scratch.s_start;
  return end;
}

static void search_range(range_job *J) {
  const oracle_params *p = J->p;
  const int32_t w = p->word_len, lq = J->lq, na = J->na;
  int32_t *dcount = NULL, *dstart = NULL, *dfill = NULL, *hs = NULL;
  uint8_t *pass = NULL;
  int64_t dcap = 0, hcap = 0;

  for (int64_t i = J->first; i < J->last && !J->err; ++i) {
    const uint8_t *S = J->db + J->offsets[i];
    const int32_t ls = (int32_t)(J->offsets[i + 1] - J->offsets[i]);
    const int32_t subj = (int32_t)(J->subject_base + i);
    J->cur_subject = i;
    if (ls < w || lq < w) continue;

    /* Hit detection (Alg. 1 L1-4; R4): scan the subject left to
     * right, look every word up in the query table.  Diagonal d = s - q
     * (R5) lies in [-(lq-w), ls-w]; index it as d + (lq-w). */
    const int32_t nd = lq + ls - 2 * w + 1;
    if (nd + 1 > dcap) {
      dcap = 2 * (int64_t)nd + 1;
      free(dcount); free(dstart); free(dfill);
      dcount = (int32_t *)malloc(sizeof(int32_t) * (size_t)dcap);
      dstart = (int32_t *)malloc(sizeof(int32_t) * (size_t)dcap);
      dfill = (int32_t *)malloc(sizeof(int32_t) * (size_t)dcap);
      if (!dcount || !dstart || !dfill) { J->err = 1; break; }
    }
    memset(dcount, 0, sizeof(int32_t) * (size_t)nd);
    int64_t nhits = 0;
    for (int32_t s = 0; s + w <= ls; ++s) {
      int64_t v = 0;
      for (int32_t k = 0; k < w; ++k) v = v * na + S[s + k];
      for (int64_t k = J->off[v]; k < J->off[v + 1]; ++k) {
        const int32_t q = J->pos[k];
        dcount[s - q + (lq - w)]++;
        nhits++;
        hitlist_push(J->hits, subj, q, s);
      }
    }
    if (nhits == 0) continue;
    /* Group the hits by diagonal, ascending s inside a diagonal ("hits in
     * a diagonal are checked from the top left to bottom right"). */
    dstart[0] = 0;
    for (int32_t d = 0; d < nd; ++d) dstart[d + 1] = dstart[d] + dcount[d];
    if (nhits > hcap) {
      hcap = 2 * nhits;
      free(hs); free(pass);
      hs = (int32_t *)malloc(sizeof(int32_t) * (size_t)hcap);
      pass = (uint8_t *)malloc((size_t)hcap);
      if (!hs || !pass) { J->err = 1; break; }
    }
    memcpy(dfill, dstart, sizeof(int32_t) * (size_t)nd);
    for (int32_t s = 0; s + w <= ls; ++s) {
      int64_t v = 0;
      for (int32_t k = 0; k < w; ++k) v = v * na + S[s + k];
      for (int64_t k = J->off[v]; k < J->off[v + 1]; ++k)
        hs[dfill[s - J->pos[k] + (lq - w)]++] = s;
    }

    for (int32_t di = 0; di < nd; ++di) {
      const int32_t n = dcount[di];
      if (n == 0) continue;
      const int32_t d = di - (lq - w);
      const int32_t *H = hs + dstart[di];
      if (p->filter_mode == 2 || p->filter_mode == 3) {
        /* Alg. 1 L8-19 (STATEFUL, R15; mode 3 with L13's reach-back, R16):
         * the walk decides which hits are extended; each extension is the
         * same R7-R9 extension as below. */
        ext_ctx X = {J, S, ls, d, H, {0, 0, 0, 0, 0, 0, 0}};
        stateful_walk(H, n, p->min_gap, p->window, p->filter_mode == 3, ext_end_of, &X, pass);
        for (int32_t k = 0; k < n; ++k) {
          if (!pass[k]) continue;
          hitlist_push(J->passing, subj, H[k] - d, H[k]);
        }
        /* record the extensions (recomputed: the walk only kept the ends) */
        for (int32_t k = 0; k < n && !J->err; ++k) {
          if (!pass[k]) continue;
          oracle_hsp e;
          extend_hit(J, S, ls, d, H[k], &e);
          if (record_ext(J, &e)) J->err = 1;
        }
        continue;
      }
      /* Two-hit filter (R6). */
      oracle_two_hit(H, n, p->min_gap, p->window, p->filter_mode, pass);
      /* Diagonal-based ungapped extension (Alg. 3): walk the
       * kept hits in ascending order; extend iff sub_pos > ext_reach, then
       * ext_reach <- end of the extension (R10). */
      int32_t ext_reach = -1;
      for (int32_t k = 0; k < n; ++k) {
        if (!pass[k]) continue;
        const int32_t h = H[k];
        hitlist_push(J->passing, subj, h - d, h);
        /* Alg. 3 L19: skip a hit covered by the previous extension of the
         * diagonal (DIAGONAL); Alg. 4 L9-14 extends every hit (HIT). */
        if (p->ext_mode == 0 && h <= ext_reach) continue;
        oracle_hsp e;
        ext_reach = extend_hit(J, S, ls, d, h, &e);
        if (record_ext(J, &e)) { J->err = 1; break; }
      }
    }
  }
  free(dcount); free(dstart); free(dfill); free(hs); free(pass);
}

static void *search_thread(void *arg) {
  search_range((range_job *)arg);
  return NULL;
}

int64_t oracle_search(const uint8_t *query, int32_t lq, int32_t query_id,
                      const uint8_t *db, const int64_t *offsets, int64_t nseq,
                      int64_t subject_base, const int32_t *matrix, int32_t na,
                      const oracle_params *p, const int64_t *table_off,
                      const int32_t *table_pos, int32_t nthreads,
                      oracle_hsp *out, int64_t cap, oracle_hsp *ext_out,
                      int64_t ext_cap, int64_t *ext_count,
                      oracle_hitlist *hits, oracle_hitlist *passing) {
  if (!query || !p || !matrix || na <= 0 || p->word_len <= 0 || nseq < 0)
    return -2;
  if (nthreads < 1) nthreads = 1;
  if ((hits || passing) && nthreads != 1) return -2;
  if (hits) hits->count = 0;
  if (passing) passing->count = 0;

  int64_t *off = (int64_t *)table_off;
  int32_t *pos = (int32_t *)table_pos;
  int own_table = 0;
  if (!off) {
    const int64_t nwords = ipow(na, p->word_len);
    off = (int64_t *)malloc(sizeof(int64_t) * (size_t)(nwords + 1));
    if (!off) return -1;
    int64_t total = oracle_neighbourhood(query, lq, matrix, na, p->word_len,
                                         p->threshold, off, NULL, 0);
    pos = (int32_t *)malloc(sizeof(int32_t) * (size_t)(total + 1));
    if (!pos) { free(off); return -1; }
    oracle_neighbourhood(query, lq, matrix, na, p->word_len, p->threshold, off,
                         pos, total);
    own_table = 1;
  }

  range_job *jobs = (range_job *)calloc((size_t)nthreads, sizeof(range_job));
  pthread_t *tids = (pthread_t *)calloc((size_t)nthreads, sizeof(pthread_t));
  int64_t result = 0;
  if (!jobs || !tids) { result = -1; goto done; }
  /* contiguous subject ranges balanced by residues */
  {
    const int64_t total = offsets[nseq] - offsets[0];
    int64_t cur = 0;
    for (int32_t t = 0; t < nthreads; ++t) {
      range_job *J = &jobs[t];
      J->query = query; J->lq = lq; J->query_id = query_id;
      J->db = db; J->offsets = offsets; J->subject_base = subject_base;
      J->matrix = matrix; J->na = na; J->p = p; J->off = off; J->pos = pos;
      J->hits = hits; J->passing = passing;
      J->collect_ext = ext_out != NULL;
      J->first = cur;
      int64_t target = offsets[0] + total * (t + 1) / nthreads;
      while (cur < nseq && offsets[cur] < target) ++cur;
      if (t == nthreads - 1) cur = nseq;
      J->last = cur;
    }
  }
  if (nthreads == 1) {
    search_range(&jobs[0]);
  } else {
    for (int32_t t = 0; t < nthreads; ++t)
      if (pthread_create(&tids[t], NULL, search_thread, &jobs[t])) {
        search_range(&jobs[t]); /* run inline if a thread cannot start */
        tids[t] = 0;
      }
    for (int32_t t = 0; t < nthreads; ++t)
      if (tids[t]) pthread_join(tids[t], NULL);
  }
  {
    hsp_vec all = {0, 0, 0}, allx = {0, 0, 0};
    for (int32_t t = 0; t < nthreads && result >= 0; ++t) {
      if (jobs[t].err) { result = -1; break; }
      for (int64_t k = 0; k < jobs[t].out.n; ++k)
        if (hsp_push(&all, &jobs[t].out.v[k])) { result = -1; break; }
      for (int64_t k = 0; k < jobs[t].ext.n && ext_out; ++k)
        if (hsp_push(&allx, &jobs[t].ext.v[k])) { result = -1; break; }
      if (!ext_out) allx.n += jobs[t].ext.n;
    }
    if (result >= 0) {
      if (all.n) qsort(all.v, (size_t)all.n, sizeof(oracle_hsp), hsp_cmp);
      if (allx.v && allx.n) qsort(allx.v, (size_t)allx.n, sizeof(oracle_hsp), hsp_cmp);
      if (out)
        for (int64_t k = 0; k < all.n && k < cap; ++k) out[k] = all.v[k];
      if (ext_out)
        for (int64_t k = 0; k < allx.n && k < ext_cap; ++k) ext_out[k] = allx.v[k];
      if (ext_count) *ext_count = allx.n;
      result = all.n;
    }
    free(all.v);
    free(allx.v);
  }
done:
  if (jobs)
    for (int32_t t = 0; t < nthreads; ++t) {
      free(jobs[t].out.v);
      free(jobs[t].ext.v);
    }
  free(jobs);
  free(tids);
  if (own_table) { free(off); free(pos); }
  return result;
}
