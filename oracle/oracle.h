/*
 * oracle.h -- CPU oracle for the cuBLASTP hot path (hit detection, two-hit
 * filter, X-drop ungapped extension).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * The product path (paper_conf_ipps_zhangwlf14_b200/, libblastp.so) never
 * includes, links or calls anything in oracle/, and this file includes
 * nothing from the product tree.
 *
 * Plain, slow, obviously-correct C99 that follows PAPER.md step by step
 * (citations "P:L<n>" are lines of /root/reference/PAPER.md) and the
 * binding readings R1..R13 of SURVEY.md section 8(c), which DESIGN.md lists.
 *
 * Everything is generic over an alphabet of `na` letters with an na x na
 * integer scoring matrix, so that the paper's toy examples (3-letter
 * alphabet of Fig. 2(a), Fig. 8 score strings) can be run through exactly
 * the same code as BLOSUM62 searches.
 *
 * Parity status of each function (pins live in tests/test_oracle_*.py):
 *   oracle_encode            pinned: R1 alphabet round-trip, U/O/J->X, errors
 *   ORACLE_BLOSUM62          pinned: symmetry, lambda_u = 0.3176 with RR freqs
 *   oracle_neighbourhood     pinned: Fig. 2(a) example, exhaustive word pairs,
 *                                    neighbourhood-size statistics
 *   oracle_xdrop_pairs       pinned: Fig. 8 worked example, X=inf closed form
 *   oracle_two_hit           pinned: Fig. 7 example (both modes), O(n^2) brute force
 *   oracle_two_hit_stateful  pinned: hand-walked Alg. 1 examples (tests/golden/
 *                                    alg1_stateful.json), = LEFT on diagonals of
 *                                    <= 2 hits, covering-extension special case,
 *                                    trigger spacing invariant
 *   oracle_two_hit_stateful_rb  pinned: hand-walked reach-back examples
 *                                    (tests/golden/alg1_reachback.json), = STATEFUL
 *                                    when every extension reaches back, oracle-B
 *   oracle_search            pinned: P5-P9 invariants, independent oracle-B
 *                                    (oracle/oracle_b.py) on random tiny cases,
 *                                    planted exact copies, E[hits] closed form;
 *                                    HIT mode: oracle-B, one extension per
 *                                    passing hit, Alg. 3 chain of HIT = DIAGONAL.
 *   oracle_gapped_dir / oracle_gapped_hsps (gapped.c): see gapped.c's header
 *   Whole HSP list vs FSA-BLAST: parity unpinned (FSA-BLAST's rules are not
 *   in the paper); see DESIGN.md.
 */
#ifndef BLASTP_ORACLE_H
#define BLASTP_ORACLE_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define ORACLE_NA 24 /* letters of the BLOSUM62 alphabet, R1 */

/* R1: NCBI letter order; code = index in this string. */
extern const char ORACLE_ALPHABET[ORACLE_NA + 1];
/* R2: NCBI BLOSUM62, row-major [a][b]. */
extern const int32_t ORACLE_BLOSUM62[ORACLE_NA * ORACLE_NA];

typedef struct {
  int32_t word_len;    /* W-length of words, 3                  */
  int32_t threshold;   /* T: neighbour iff word score >= T (R3)              */
  int32_t window;      /* A: two-hit window, hit passes iff min_gap<=h-p<A   */
  int32_t min_gap;     /* non-overlap distance, = word_len (R6)              */
  int32_t xdrop;       /* X: stop when best - run >= X (R8)                  */
  int32_t cutoff;      /* emit iff score >= cutoff (R10)                     */
  int32_t filter_mode; /* 0 = LEFT (R6 default), 1 = EITHER (Fig. 7 reading),
                          2 = STATEFUL: Alg. 1 L8-19's lasthit walk (R15),
                          which also decides coverage (ext_mode ignored),
                          3 = STATEFUL with L13's reach-back: an extension is
                          kept only if it reaches back to lasthit (R16) */
  int32_t ext_mode;    /* 0 = DIAGONAL: Alg. 3 coverage chain (R10, default);
                          1 = HIT: Alg. 4, every
                          passing hit extended independently, duplicates kept */
} oracle_params;

/* One ungapped extension (R10/R11).  diagonal = s_start - q_start. */
typedef struct {
  int32_t query_id, subject_id, diagonal, q_start, s_start, length, score;
} oracle_hsp;

/* Optional per-hit debug lists (single-threaded search only). */
typedef struct {
  int64_t cap;   /* capacity of the arrays                      */
  int64_t count; /* number of entries produced (may exceed cap) */
  int32_t *subject, *q, *s;
} oracle_hitlist;

/* R1: ASCII -> codes.  Lowercase is upper-cased, U/O/J -> X.
 * Returns 0, or -(i+1) where i is the index of the first invalid byte. */
int64_t oracle_encode(const char *ascii, int64_t n, uint8_t *codes);

/* R3: brute-force neighbourhood table.  For every query position
 * q in [0, lq-word_len] and every word v in [0, na^word_len), v is a
 * neighbour of q iff sum_i matrix[query[q+i]][v_i] >= T.  Output is CSR:
 * the query positions of word v are pos[off[v] .. off[v+1]), ascending.
 * off has na^word_len + 1 entries.  Returns the total number of entries
 * (the pos array is only written while it fits in cap). */
int64_t oracle_neighbourhood(const uint8_t *query, int32_t lq,
                             const int32_t *matrix, int32_t na,
                             int32_t word_len, int32_t T, int64_t *off,
                             int32_t *pos, int64_t cap);

/* R8: X-drop over the pair scores matrix[a[k*step]][b[k*step]],
 * k = 0 .. n-1 (n = pairs available before either sequence ends).
 * best = max(0, max prefix sum), len = shortest prefix reaching best
 * (0 if best == 0), steps = pairs consumed (index of the stopping pair
 * + 1, or n if the sequence ended first). */
void oracle_xdrop_pairs(const uint8_t *a, const uint8_t *b, int32_t n,
                        int32_t step, const int32_t *matrix, int32_t na,
                        int32_t X, int32_t *best, int32_t *len,
                        int32_t *steps);

/* R6: two-hit test on the ascending subject positions s[0..n) of the hits
 * of ONE diagonal of ONE subject.  mode 0 (LEFT): pass[k] iff some m with
 * min_gap <= s[k]-s[m] < window.  mode 1 (EITHER): |s[k]-s[m]| in that
 * range for some m. */
void oracle_two_hit(const int32_t *s, int32_t n, int32_t min_gap,
                    int32_t window, int32_t mode, uint8_t *pass);

/* Alg. 1 L8-19 (R15): the STATEFUL walk over the ascending
 * subject positions s[0..n) of the hits of ONE diagonal of ONE subject.
 * ext_end[k] = subject end (inclusive) of the extension from hit k (R7-R10;
 * it does not depend on the walk).  trigger[k] = 1 iff hit k is extended:
 * lasthit <- h when there is none or h - lasthit >= window; extend when
 * min_gap <= h - lasthit < window, then lasthit <- ext_end[k]; otherwise
 * (h - lasthit < min_gap) nothing changes. */
void oracle_two_hit_stateful(const int32_t *s, int32_t n,
                             const int32_t *ext_end, int32_t min_gap,
                             int32_t window, uint8_t *trigger);

/* The same walk with Alg. 1 L13's reach-back (ungapped_ext(hit_k,
 * lasthit); R16): ext_start[k] = subject start of the extension from hit k;
 * an extension with ext_start[k] > lasthit is dropped (trigger[k] = 0) and
 * lasthit <- s[k] instead. */
void oracle_two_hit_stateful_rb(const int32_t *s, int32_t n,
                                const int32_t *ext_start,
                                const int32_t *ext_end, int32_t min_gap,
                                int32_t window, uint8_t *trigger);

/* Full search of one query against the subjects of `db` (codes,
 * concatenated; subject i is db[offsets[i] .. offsets[i+1]) ).
 * subject_id written = subject_base + i.  Emits HSPs with score >= cutoff
 * into out (canonical order, R11) and every extension performed (emitted
 * or not) into ext_out (also canonical), either may be NULL.  When
 * table_off/table_pos are NULL the table is built with
 * oracle_neighbourhood; otherwise the given table is used (Fig. 3/5
 * table-injection tests).  nthreads > 1 splits subjects into contiguous
 * ranges over pthreads.  hits / passing (optional) collect every hit and
 * every hit passing the two-hit test; they require nthreads == 1.
 * Returns the number of HSPs (entries beyond cap are counted, not written),
 * or a negative value on allocation failure / bad arguments. */
int64_t oracle_search(const uint8_t *query, int32_t lq, int32_t query_id,
                      const uint8_t *db, const int64_t *offsets, int64_t nseq,
                      int64_t subject_base, const int32_t *matrix, int32_t na,
                      const oracle_params *p, const int64_t *table_off,
                      const int32_t *table_pos, int32_t nthreads,
                      oracle_hsp *out, int64_t cap, oracle_hsp *ext_out,
                      int64_t ext_cap, int64_t *ext_count,
                      oracle_hitlist *hits, oracle_hitlist *passing);

/* ---- gapped extension of the HSP hand-off (gapped.c; R18-R22) ---- */

/* One gapped alignment: query [q_start, q_end) x subject [s_start, s_end),
 * score, and its traceback path's identities, gaps opened and gap residues. */
typedef struct {
  int32_t query_id, subject_id, q_start, q_end, s_start, s_end, score, ident, gap_opens, gap_len;
} oracle_gapped;

/* R19/R22: one direction from the seed corner over a[0..la) x b[0..lb). */
int32_t oracle_gapped_dir(const uint8_t *a, int32_t la, const uint8_t *b, int32_t lb,
                          const int32_t *matrix, int32_t nalpha, int32_t gap_open,
                          int32_t gap_extend, int32_t xdrop, int32_t *bi, int32_t *bj,
                          int32_t *ident, int32_t *gopen, int32_t *glen);

/* R20/R21 over a canonical HSP list (query k's codes queries[k]/qlens[k];
 * subject i - subject_base at db[offsets[i] .. offsets[i+1])).  Returns the
 * number of reported alignments (canonical order, first `cap` written). */
int64_t oracle_gapped_hsps(const uint8_t *const *queries, const int32_t *qlens, int32_t nq,
                           const uint8_t *db, const int64_t *offsets, int64_t nseq,
                           int64_t subject_base, const oracle_hsp *hsps, int64_t n,
                           const int32_t *matrix, int32_t nalpha, int32_t gap_open,
                           int32_t gap_extend, int32_t xdrop, int32_t cutoff,
                           oracle_gapped *out, int64_t cap);

#ifdef __cplusplus
}
#endif
#endif
