/*
 * blastp.h -- C-ABI of libblastp.so, the B200-native (sm_100a) hot path of
 * cuBLASTP (Zhang, Wang, Feng; IPDPS'14 / TCBB'15): BLASTP hit detection,
 * two-hit filtering on diagonals and X-drop ungapped extension.
 *
 * Citations "P:L<n>" are lines of the paper text;
 * "R<k>" are the readings of SURVEY.md section 8(c), restated in DESIGN.md.
 *
 * Conventions (all entry points):
 *  - Every function returns an int status: BLASTP_OK (0) or a negative
 *    BLASTP_E_* code.  Nothing throws or aborts.  blastp_last_error() gives a
 *    thread-local, human-readable detail of the last failure.
 *  - Plain pointers and sizes only.  "host" pointers are ordinary (ideally
 *    pinned) CPU memory; "device" pointers are CUDA global memory on the
 *    device the handle was created on (e.g. a torch.cuda tensor's data_ptr()).
 *  - `cuda_stream` is a cudaStream_t passed as void* (NULL = legacy default
 *    stream).  All device work of a call is enqueued on it.
 *  - Inputs are copied; the caller keeps ownership.  Handles and library-
 *    allocated host arrays are owned by the library until the matching
 *    *_free call.
 *  - A database handle owns scratch counters: do not run two searches on
 *    the same blastp_db concurrently on different streams.
 *
 * Residue encoding (R1): 24 letters in NCBI order "ARNDCQEGHILKMFPSTWYVBZX*"
 * -> codes 0..23; lowercase is upper-cased; U, O and J map to X; any other
 * byte is BLASTP_E_BAD_RESIDUE.  Scoring is BLOSUM62 (R2).
 */
#ifndef BLASTP_H
#define BLASTP_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define BLASTP_OK 0
#define BLASTP_E_INVALID_ARG (-1) /* NULL pointer, bad size or parameter   */
#define BLASTP_E_BAD_RESIDUE (-2) /* character outside R1's alphabet       */
#define BLASTP_E_TOO_LONG (-3)    /* query > BLASTP_MAX_QUERY_LEN, subject > BLASTP_MAX_SUBJECT_LEN */
#define BLASTP_E_NOMEM (-4)       /* host or device allocation failed      */
#define BLASTP_E_CUDA (-5)        /* CUDA runtime error (detail in last_error) */
#define BLASTP_E_CAPACITY (-6)    /* caller buffer too small (see below)   */

#define BLASTP_MAX_QUERY_LEN 16000
#define BLASTP_MAX_SUBJECT_LEN (1 << 30)
#define BLASTP_FILTER_LEFT 0   /* R6 default: W <= h - p < A              */
#define BLASTP_FILTER_EITHER 1 /* Fig. 7 reading: W <= |h - p| < A        */
#define BLASTP_FILTER_STATEFUL 2 /* Alg. 1 L8-19, reading R15: one lasthit per
                                    diagonal; h - lasthit >= A (or none): lasthit <- h;
                                    W <= h - lasthit < A: extend, lasthit <- HSP subject
                                    end; else no change.  Decides coverage itself, so it
                                    requires ext_mode BLASTP_EXT_DIAGONAL.  Warp kernel
                                    only; long subjects are split by diagonal range. */
#define BLASTP_FILTER_STATEFUL_RB 3 /* STATEFUL plus Alg. 1 L13's second argument,
                                    ungapped_ext(hit, lasthit), reading R16: an
                                    extension is kept only if its subject start is at or
                                    before the lasthit it pairs with (the two hits lie in
                                    one ungapped alignment, NCBI/FSA BLAST's two-hit
                                    method); otherwise it is dropped (no output) and
                                    lasthit <- the hit (L19).  Same constraints as
                                    STATEFUL. */
#define BLASTP_EXT_DIAGONAL 0  /* Alg. 3: a passing hit covered by the
                                  previous extension of its diagonal is skipped (R10) */
#define BLASTP_EXT_HIT 1       /* Alg. 4: every passing
                                  hit is extended independently; duplicates kept      */
#define BLASTP_EXT_WINDOW 2    /* Alg. 5 + Fig. 8: Alg. 3's coverage rule,
                                  each extension a warp-wide window scan (prefix sum,
                                  running max, drop flag over 32 positions at a time);
                                  results identical to DIAGONAL                       */
#define BLASTP_EXT_HIT_DEDUP 3 /* Alg. 4 followed by the de-duplication step the paper
                                  puts after it (reading R17): every
                                  passing hit is extended independently (Alg. 4), then
                                  each diagonal's extensions, in seed order, are reduced
                                  by Alg. 3's coverage rule (a seed covered by the last
                                  kept extension's subject end is dropped) -- exactly
                                  DIAGONAL's list.  blastp_search_ungapped applies the
                                  step itself; blastp_search_ungapped_device returns the
                                  SEED RECORDS of every extension (q_start = the seed's
                                  query position, s_start = llen; see
                                  blastp_dedup_covered_device) for the caller to reduce */

/* Search parameters.  Defaults (blastp_params_default) are the BASELINE.json
 * configuration: w = 3, T = 11, A = 40, X = 7 bits -> 16 raw, cutoff 41. */
typedef struct {
  int32_t word_len;    /* word length W; only 3 is supported     */
  int32_t threshold;   /* T: word v neighbours query word iff score >= T (R3) */
  int32_t window;      /* A: two-hit window (R6), 1..256        */
  int32_t min_gap;     /* non-overlap distance (R6), 1..8; default = word_len */
  int32_t xdrop;       /* X: stop when best - run >= X (Fig. 8, R8), 1..127   */
  int32_t cutoff;      /* emit an extension iff score >= cutoff (R10)         */
  int32_t filter_mode; /* BLASTP_FILTER_LEFT, _EITHER, _STATEFUL, _STATEFUL_RB */
  int32_t ext_mode;    /* BLASTP_EXT_DIAGONAL (default), _HIT or _WINDOW       */
} blastp_params;

/* One ungapped extension ("start and end position of this extension with
 * the highest score").  28 bytes; it is also the hand-off
 * record to a gapped-extension stage (out of scope here).
 * diagonal = s_start - q_start; the segment is
 * [q_start, q_start+length) x [s_start, s_start+length), score = sum of
 * BLOSUM62 over it.  subject_id is GLOBAL (shard base + local index). */
typedef struct {
  int32_t query_id, subject_id, diagonal, q_start, s_start, length, score;
} blastp_hsp;

/* Debug record of a hit / passing hit (subject-local coordinates). */
typedef struct {
  int32_t query_id, subject_id, q, s;
} blastp_hit;

typedef struct blastp_query_table blastp_query_table; /* opaque */
typedef struct blastp_db blastp_db;                   /* opaque: one shard */

void blastp_params_default(blastp_params *p);
const char *blastp_strerror(int status);
const char *blastp_last_error(void);
const char *blastp_version(void);

/* Query lookup table (R3): for every query position
 * q in [0, len-3] the list of all 24^3 words v with
 * sum_i BLOSUM62[query[q+i]][v_i] >= p->threshold, stored as a CSR table
 * word -> ascending query positions (the function of the paper's DFA),
 * plus the query codes.  The codes are validated and encoded on the host,
 * the table is built on `device` (one thread per word: count, scan, fill;
 * BLASTP_TABLE_BUILD=host enumerates on the host instead) on `cuda_stream`;
 * the call returns when the table is complete.
 * query_ascii: host, `len` bytes (3 <= len <= BLASTP_MAX_QUERY_LEN).
 * Errors: INVALID_ARG (NULL, len < 3, word_len != 3), BAD_RESIDUE,
 * TOO_LONG, NOMEM, CUDA. */
int blastp_build_query_table(const char *query_ascii, int32_t len,
                             const blastp_params *p, int device,
                             void *cuda_stream, blastp_query_table **out);

/* Same for `nq` queries; query_id of results = index in `queries`.
 * Queries of a batch are also packed into query groups (SURVEY 8(f) rank 1:
 * one database scan for several queries): first-fit decreasing into groups
 * of combined length <= 1280 with p->window + 8 sentinel codes between
 * members (BLASTP_GROUP=0 disables).  A search uses the groups when its
 * window A satisfies A + 8 <= that gap (else, and for the debug entry
 * points, it searches query by query); results are identical either way. */
int blastp_build_query_batch(const char *const *queries, const int32_t *lens,
                             int32_t nq, const blastp_params *p, int device,
                             void *cuda_stream, blastp_query_table **out);

/* Database pack + shard (coalesced residue access).
 * residues_ascii: host, all subjects concatenated; subject i is
 * residues_ascii[offsets[i] .. offsets[i+1]) (offsets: host, nseq+1 entries,
 * non-decreasing, offsets[0] may be non-zero).  The subjects are split into
 * num_shards contiguous ranges balanced by residues (blastp_shard_range) and
 * only range `shard_index` is packed: its bytes are copied host->device on
 * `cuda_stream` and encoded on the GPU into a sentinel-separated code stream
 * (1 byte per residue).  Returns after the device work completes.
 * Errors: INVALID_ARG, BAD_RESIDUE, TOO_LONG (a subject > MAX_SUBJECT_LEN),
 * NOMEM, CUDA. */
int blastp_pack_db(const char *residues_ascii, const int64_t *offsets,
                   int64_t nseq, int32_t shard_index, int32_t num_shards,
                   int device, void *cuda_stream, blastp_db **out);

/* Subject range [*lo, *hi) of shard `shard_index` (host-only helper, no GPU):
 * the first subject of shard k is the first i with
 * offsets[i] - offsets[0] >= total * k / num_shards. */
int blastp_shard_range(const int64_t *offsets, int64_t nseq,
                       int32_t shard_index, int32_t num_shards, int64_t *lo,
                       int64_t *hi);

/* Shard description: number of subjects, residues, global id of its first
 * subject (shard base), packed stream bytes.  Any pointer may be NULL. */
int blastp_db_info(const blastp_db *db, int64_t *nseq, int64_t *residues,
                   int64_t *subject_base, int64_t *stream_bytes,
                   int64_t *num_chunks);
/* End-to-end search of a HOST-resident database shard (no blastp_db kept):
 * the shard's subjects (blastp_shard_range) are cut into parts of whole
 * subjects (num_parts > 0: that many residue-balanced parts; 0: automatic,
 * growing 1.25x from ~1/64 of the shard) and each part is packed (H2D copy
 * + encode, as blastp_pack_db, on an internal stream) while the previous
 * part is searched on `cuda_stream` -- the copy overlaps the search (not in
 * the paper, whose database is resident; DESIGN.md "Host-resident
 * databases").  Every HSP of every query is appended to d_out (device,
 * capacity records, unsorted; subject_id global) and the total count,
 * possibly > capacity, is written to *d_count (device int64).  Same results
 * as blastp_pack_db + blastp_search_ungapped_device on the whole shard.
 * Returns when the last part's search is enqueued; part buffers are
 * released in stream order.  Errors: as blastp_pack_db and
 * blastp_search_ungapped_device. */
int blastp_search_host_db(const blastp_query_table *q, const char *residues_ascii,
                          const int64_t *offsets, int64_t nseq, int32_t shard_index,
                          int32_t num_shards, const blastp_params *p, int32_t num_parts,
                          void *cuda_stream, blastp_hsp *d_out, int64_t capacity,
                          int64_t *d_count);

/* Formatted host database (the makeblastdb step): the shard `shard_index`
 * of `num_shards` (as blastp_pack_db) is packed on `device` in parts
 * (num_parts > 0: that many residue-balanced parts; 0: parts growing 1.25x
 * from a small first one, as blastp_search_host_db) and each part's device
 * image -- code stream, subject starts, chunk plan, long-item plan -- is
 * copied back into one pinned host buffer owned by the handle.  Synchronous.
 * blastp_search_formatted_db then streams the parts: one host->device copy
 * per part on a copy stream (no kernel, no host synchronisation between
 * parts) and the part's search on one of two alternating search streams
 * once its copy has landed; HSPs are appended to d_out / *d_count exactly as
 * blastp_search_ungapped_device does for the whole shard (same results as
 * blastp_pack_db + blastp_search_ungapped_device).  Asynchronous on
 * cuda_stream; device memory is released in stream order.  The streaming
 * overlaps each part's host->device copy with the previous part's search and
 * bounds device memory: a ring of min(num_parts, BLASTP_PIPE_SLOTS = 3) part
 * slots, each the largest part's image plus its scratch, is allocated; part
 * k is copied into slot k mod slots once the search of the slot's previous
 * part has completed (stream-ordered events, no host synchronisation) -- a
 * shard larger than HBM is searched by formatting it into enough parts.
 * Errors: as blastp_pack_db (format) and blastp_search_ungapped_device
 * (search), E_NOMEM if the pinned image or the slots cannot be allocated. */
typedef struct blastp_host_db blastp_host_db;
int blastp_format_host_db(const char *residues_ascii, const int64_t *offsets, int64_t nseq,
                          int32_t shard_index, int32_t num_shards, int32_t num_parts,
                          int device, void *cuda_stream, blastp_host_db **out);
int blastp_search_formatted_db(const blastp_query_table *q, const blastp_host_db *h,
                               const blastp_params *p, void *cuda_stream, blastp_hsp *d_out,
                               int64_t capacity, int64_t *d_count);
int blastp_host_db_info(const blastp_host_db *h, int64_t *nseq, int64_t *residues,
                        int64_t *subject_base, int32_t *num_parts, int64_t *host_bytes);
void blastp_host_db_free(blastp_host_db *h);

/* Long-subject plan of the shard (implementation detail, exposed for tests
 * and tuning): chunks longer than 2C residues that are scheduled first
 * (*long_items), the segments they are split into for parallel two-hit
 * filtering (*segments; 0 = every long chunk is walked whole) and the
 * segment length in positions.  Results never depend on the plan.  Any
 * pointer may be NULL.  Errors: INVALID_ARG (db NULL). */
int blastp_db_long_info(const blastp_db *db, int64_t *long_items,
                        int64_t *segments, int64_t *segment_len);
int blastp_query_table_info(const blastp_query_table *q, int32_t *num_queries,
                            int64_t *table_entries);
/* Query groups of a batch table: *groups (searched as one scan each),
 * *alone (queries searched by themselves) and the sentinel *gap between
 * members; a search with window A launches groups + alone kernels per
 * shard when A + 8 <= gap, else num_queries.  Any pointer may be NULL. */
int blastp_query_table_groups(const blastp_query_table *q, int32_t *groups, int32_t *alone,
                              int32_t *gap);

/* Ungapped search (Alg. 1-5; R4-R10): every hit of every query against
 * every subject of the shard, the two-hit filter per (subject, diagonal),
 * X-drop extension of passing hits not covered by a previous extension of
 * the same diagonal (ext_mode DIAGONAL; ext_mode HIT extends every passing
 * hit, so one HSP may be returned once per seed inside it), and every
 * extension with score >= cutoff returned.
 * HOST variant: *out_host (library-malloc'd, free with blastp_hsp_free) gets
 * *out_count HSPs in canonical order (R11: lexicographic on all 7 fields).
 * Synchronous on cuda_stream.  `p` must equal the params of the table for
 * word_len/threshold (they shaped the table); the others may differ. */
int blastp_search_ungapped(const blastp_query_table *q, const blastp_db *db,
                           const blastp_params *p, void *cuda_stream,
                           blastp_hsp **out_host, int64_t *out_count);

/* DEVICE variant, asynchronous: HSPs are appended (unordered) to d_out
 * (device, `capacity` records); d_count (device, one int64) receives the
 * number of HSPs found, which may exceed capacity -- then only `capacity`
 * records were written and the caller should retry with a larger buffer.
 * Nothing is read back; no host synchronisation. */
int blastp_search_ungapped_device(const blastp_query_table *q,
                                  const blastp_db *db, const blastp_params *p,
                                  void *cuda_stream, blastp_hsp *d_out,
                                  int64_t capacity, int64_t *d_count);

/* APPEND variant for multi-GPU result collection, asynchronous:
 * as blastp_search_ungapped_device, except that *d_count is NOT reset -- each
 * HSP takes the next index of the shared counter (device atomics) -- and
 * d_out / d_count may be another GPU's memory mapped with blastp_ipc_open:
 * the search kernel then stores its HSPs straight into that GPU's buffer over
 * NVLink / NVSwitch (no separate gather), each record performed at system
 * scope (__threadfence_system) before the kernel completes.  Several ranks
 * append to one buffer; the order is unspecified (sort with
 * blastp_sort_hsps_device) and a count above capacity means records were
 * dropped (retry larger).  The caller orders the counter reset before every
 * rank's append and every rank's completion before reading (stream order
 * plus a collective, see dist.py PeerHspBuffer).  Errors: as
 * blastp_search_ungapped_device. */
int blastp_search_ungapped_append(const blastp_query_table *q, const blastp_db *db,
                                  const blastp_params *p, void *cuda_stream, blastp_hsp *d_out,
                                  int64_t capacity, int64_t *d_count);

/* Exported device buffers (CUDA IPC) for blastp_search_ungapped_append.
 * blastp_ipc_alloc: `bytes` of device memory on `device` (cudaMalloc) and
 * its IPC handle (BLASTP_IPC_HANDLE_BYTES bytes written to handle_out, to be
 * sent to the other processes); free with blastp_ipc_free in the allocating
 * process after every opener closed it.  blastp_ipc_open: maps a handle from
 * another process into this one's address space for `device` (peer access
 * enabled on demand); unmap with blastp_ipc_close.  A handle cannot be
 * opened by the process that allocated it.  Errors: INVALID_ARG, NOMEM,
 * CUDA. */
#define BLASTP_IPC_HANDLE_BYTES 64
int blastp_ipc_alloc(int device, int64_t bytes, void **d_ptr, void *handle_out);
int blastp_ipc_open(int device, const void *handle, void **d_ptr);
int blastp_ipc_close(void *d_ptr);
int blastp_ipc_free(void *d_ptr);

/* The coverage-aware de-duplication of ext_mode HIT_DEDUP (R17), on the
 * device, in place: d_rec[0..n) are seed records {query_id, subject_id,
 * diagonal, q_seed, llen, length, score} of every extension (one per passing
 * hit; the HSP starts at q_seed - llen); they are sorted, each diagonal's
 * records are walked in seed order keeping a record iff its seed's subject
 * position exceeds the subject end of the last kept one (Alg. 3 L19-23), and
 * the kept ones with score >= cutoff are written back as canonical HSPs
 * (R11).  *d_n_out (device int64) receives their count; runs on cuda_stream
 * and synchronises it (the kept count sizes the final sort).  Errors:
 * INVALID_ARG, NOMEM, CUDA. */
int blastp_dedup_covered_device(blastp_hsp *d_rec, int64_t n, int32_t cutoff, int64_t *d_n_out,
                                void *cuda_stream);

/* Canonical order (R11) of n device HSPs, in place, on the GPU. */
int blastp_sort_hsps_device(blastp_hsp *d_hsps, int64_t n, void *cuda_stream);

/* De-duplication of a canonically ordered (blastp_sort_hsps_device) device
 * HSP list, in place: runs of identical records collapse to one.  This is the
 * step Alg. 4 (ext_mode HIT) leaves before gapped extension ("requires a
 * de-duplication step"); a DIAGONAL-mode list has no
 * duplicates.  *d_n_out (device int64) receives the new count; asynchronous
 * on cuda_stream.  Errors: INVALID_ARG (n < 0, NULL buffers), NOMEM, CUDA. */
int blastp_unique_hsps_device(blastp_hsp *d_hsps, int64_t n, int64_t *d_n_out,
                              void *cuda_stream);

/* ---- Gapped-extension consumer of the HSP hand-off ----
 * PAPER.md 3.6: "only the high-scoring seeds from ungapped
 * extension can be passed to the gapped-extension stage", which the paper
 * runs on the CPU, overlapped with the GPU search (Fig. 12).
 * The paper prints no algorithm; R18-R22 fix it:
 *  R18 a gap of k residues costs gap_open + gap_extend * k;
 *  R19 per direction one Gotoh DP anchored at the seed corner, cells in
 *      row-major order, a cell dead iff H < best - xdrop (best = the largest
 *      H so far, from 0), the first maximum wins, a row without live cells
 *      ends the direction;
 *  R20 the seed of an HSP is its middle pair (q_start + length/2,
 *      s_start + length/2): right = forward from it, left = backward from
 *      the pair before;
 *  R21 per (query, subject) the HSPs in descending score (ties: canonical
 *      order); an HSP whose seed lies in the box [q_start, q_end) x
 *      [s_start, s_end) of an alignment already made for the pair is
 *      skipped; an alignment is reported iff score >= cutoff; the list is in
 *      canonical order (lexicographic on all 10 fields);
 *  R22 traceback from the best cell preferring the diagonal, then a gap in
 *      the query, then a gap in the subject; a gap opening over its
 *      extension.  ident / gap_opens / gap_len count the path's identical
 *      pairs, gaps and gap residues. */
typedef struct {
  int32_t gap_open;   /* default 11 */
  int32_t gap_extend; /* default 1, >= 1 */
  int32_t xdrop;      /* raw score, default 38 (15 bits at the gapped lambda 0.267) */
  int32_t cutoff;     /* report iff score >= cutoff, default 41 */
} blastp_gapped_params;

/* One gapped alignment: query [q_start, q_end) against subject
 * [s_start, s_end) (subject_id global, as in blastp_hsp).  40 bytes. */
typedef struct {
  int32_t query_id, subject_id, q_start, q_end, s_start, s_end, score, ident, gap_opens,
      gap_len;
} blastp_gapped;

void blastp_gapped_params_default(blastp_gapped_params *gp);

/* Gapped extension of n ungapped HSPs on the GPU.  d_hsps: DEVICE records of
 * THIS shard (subject ids global = the shard base + local index) for the
 * queries of `q` (query_id = batch index), in canonical order (R11, e.g.
 * from blastp_sort_hsps_device; any order with each (query, subject) pair's
 * records contiguous and pairs ascending works).  The reported alignments
 * (R21) are written to d_out (device, `capacity` records) in canonical
 * order; *out_count (HOST) receives their number.  Synchronous on
 * cuda_stream (it reads the traceback store size back).  Errors: INVALID_ARG
 * (NULL pointers, bad params, an id outside the table / shard, pairs not
 * contiguous, a seed outside its sequences), CAPACITY (count > capacity:
 * the first `capacity` records are written, *out_count is the full count),
 * NOMEM, CUDA.  At most 2^30 - 1 HSPs per call; device scratch ~300 bytes
 * per HSP from the library's pool (returned to it after the call; plus ~2 GB
 * of per-thread rings and code logs with BLASTP_GAPPED_KERNEL=thread). */
int blastp_gapped_extend_device(const blastp_query_table *q, const blastp_db *db,
                                const blastp_hsp *d_hsps, int64_t n,
                                const blastp_gapped_params *gp, void *cuda_stream,
                                blastp_gapped *d_out, int64_t capacity, int64_t *out_count);

/* The two stages in one call: the ungapped search (as blastp_search_ungapped)
 * and the gapped extension of its HSP list on the GPU; *out_host
 * (library-malloc'd, free with blastp_gapped_free) receives *out_count
 * alignments in canonical order.  If ungapped_host / ungapped_count are not
 * NULL the canonical ungapped list is returned too (free with
 * blastp_hsp_free).  Synchronous.  Errors: as the two stages. */
int blastp_search_gapped(const blastp_query_table *q, const blastp_db *db,
                         const blastp_params *p, const blastp_gapped_params *gp,
                         void *cuda_stream, blastp_gapped **out_host, int64_t *out_count,
                         blastp_hsp **ungapped_host, int64_t *ungapped_count);
void blastp_gapped_free(blastp_gapped *g);

/* Debug / parity entry points (synchronous, host buffers).  They run the
 * same kernel as the search with tracing enabled and return:
 *  hits:    every hit (R4) as (query_id, subject_id, q, s), unordered;
 *  passing: every hit passing the two-hit filter (R6), unordered;
 *  exts:    every extension performed (R10), emitted or not, unordered.
 * Counts are written even when they exceed the capacities (then only the
 * first `cap` records are filled and BLASTP_E_CAPACITY is returned).
 * Any buffer may be NULL (with cap 0) to skip that list. */
int blastp_debug_trace(const blastp_query_table *q, const blastp_db *db,
                       const blastp_params *p, void *cuda_stream,
                       blastp_hit *hits, int64_t hits_cap, int64_t *n_hits,
                       blastp_hit *passing, int64_t passing_cap,
                       int64_t *n_passing, blastp_hsp *exts, int64_t exts_cap,
                       int64_t *n_exts);
int blastp_debug_hits(const blastp_query_table *q, const blastp_db *db,
                      const blastp_params *p, void *cuda_stream,
                      blastp_hit *hits, int64_t cap, int64_t *n);
int blastp_debug_passing(const blastp_query_table *q, const blastp_db *db,
                         const blastp_params *p, void *cuda_stream,
                         blastp_hit *passing, int64_t cap, int64_t *n);

/* Event counters of a traced search (synchronous): stats[i] for i < nstats,
 * in this order: 32-position windows, 32-hit rounds, rounds with two hits
 * on one diagonal, hits, passing hits, enqueued hits, extension batches,
 * extensions computed, extensions accepted (R10), HSPs emitted, X-drop
 * residues scored, X-drop lane slots (32 x longest lane per batch). */
int blastp_debug_stats(const blastp_query_table *q, const blastp_db *db,
                       const blastp_params *p, void *cuda_stream, int64_t *stats,
                       int32_t nstats);

/* The measured integer-ALU roof of `device` (synchronous, ~0.1 s): lane
 * operations per second of independent integer add / logic / multiply-add
 * chains on every SM at the search kernel's residency (32 warps per SM).
 * bench.py divides the method's work (ops per residue scanned,
 * per hit, per X-drop step, counted by blastp_debug_stats) by the search
 * time and by this roof: the on-chip roofline beside the HBM one. */
int blastp_debug_alu_peak(int device, double *lane_ops_per_s);

/* The library's stream-ordered device allocations come from its own memory
 * pool per device, which keeps freed memory for reuse (repeated pack /
 * search calls do not pay cudaMalloc again); this returns the pool's unused
 * memory to the device (synchronises the device).  Errors: CUDA. */
int blastp_trim_memory(int device);

void blastp_hsp_free(blastp_hsp *h);
void blastp_query_table_free(blastp_query_table *q);
void blastp_db_free(blastp_db *db);

#ifdef __cplusplus
}
#endif
#endif /* BLASTP_H */
