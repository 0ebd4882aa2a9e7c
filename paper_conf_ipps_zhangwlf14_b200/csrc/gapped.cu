// gapped.cu -- gapped-extension consumer of the ungapped HSP hand-off
// (PAPER.md 3.6: "only the high-scoring
// seeds from ungapped extension can be passed to the gapped-extension stage").
//
// The paper names the stage (run on the CPU with pthreads, overlapped with the
// GPU search, Fig. 12) but prints no algorithm; R18-R22
// fix it: affine gaps (open + extend * k), one Gotoh DP per direction from the
// HSP's middle pair (R20), anchored at the seed corner, row-major cell order
// with the X-drop rule "dead iff H < best - X" against the running best (R19),
// per (query, subject) pair the HSPs in descending score, skipping a seed that
// lies in the box of an alignment already made (R21), traceback preferring the
// diagonal, then E, then F, a gap opening over its extension (R22).
//
// B200 form.  An alignment depends only on its own HSP --
// R21 only decides whether it is used -- so every HSP's two directions are
// independent work items and R21 runs afterwards, per pair.  Along a row R19
// is sequential only through E and the running best, both prefix maxima once
// the kills are taken out (a killed cell cannot make a later one live), so a
// warp computes a row 32 columns at a time.
//   order    : pairs = runs of equal (query, subject) in the canonical list; a
//              stable radix sort by (pair, descending score) gives R21's order
//              inside each pair; pass 1a takes HSPs by descending score;
//   pass 1a  : gapped_warp_kernel<false> (default): a warp per direction, the
//              previous row in a shared-memory ring, codes (H from diagonal /
//              E / F, E opened, F opened) as ballot bit-planes in shared
//              memory, traced back at once by lane 0;  gapped_first_kernel
//              (BLASTP_GAPPED_KERNEL=thread): a thread per direction, one DP
//              cell per loop turn, codes to per-thread nibble logs;
//   pass 1b  : gapped_resolve_kernel: R21 per pair over the boxes; the
//              directions not traced yet go to a work list;
//   big ring : gapped_score_kernel: pairs with a row wider than the ring,
//              redone by a thread per pair with subject-sized rings;
//   leftover : gapped_warp_kernel<true>: the work list's directions whose codes
//              did not fit, a warp per block with a 194 KB shared-memory log;
//   pass 2   : gapped_trace_kernel: whatever is still left -- the thread
//              form's logs, or a re-run up to the best row into an exactly
//              sized store -- traced back;
//   emit     : gapped_emit_kernel: per pair, its reported alignments in
//              canonical order at the pair's offset of an exclusive scan.
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_reduce.cuh>
#include <cub/device/device_scan.cuh>
#include <cuda_runtime.h>

#include <algorithm>
#include <cassert>
#include <cstdio>
#include <cstdlib>
#include <cstring>

#include "common.cuh"

namespace blastp {

namespace {

constexpr int32_t kNeg = INT32_MIN / 4;  // -infinity that survives a few subtractions

// -DGAPPED_CHECK: device asserts on every sequence read and store index (the
// bounds-checked build the tests run besides the product build)
#ifdef GAPPED_CHECK
#define GCHECK(c) assert(c)
#else
#define GCHECK(c) ((void)0)
#endif

// counters[]
enum {
  kCurPass1 = 0, kCurBig, kNumOver, kErr, kNumGroups, kTotal, kCurTrace, kCurFirst, kCells, kNumWork,
  kNumCounters = 11
};

// a reported direction for pass 2: its best cell, widest span, and whether
// pass 1 logged its codes (then at nib_off / hdr_off of the logs)
struct DirInfo {
  int32_t bi, bj, maxspan, logged;
  int64_t nib_off, hdr_off;
};


__device__ __forceinline__ int32_t imax(int32_t a, int32_t b) { return a > b ? a : b; }

__host__ __device__ inline int64_t align16(int64_t x) { return (x + 15) & ~int64_t(15); }
__host__ __device__ inline int32_t pow2_at_least(int32_t x) {
  int32_t c = 1;
  while (c < x) c <<= 1;
  return c;
}
// Traceback store of one direction (pass 2): row headers {start column, first
// cell} (int2 per row), the cells' nibbles, then the DP ring (pow2 >= the
// widest span, int2 per column).
__host__ __device__ inline int64_t slab_hdr_bytes(int32_t rows) { return align16(int64_t(rows) * 8); }
__host__ __device__ inline int64_t slab_nib_bytes(int64_t cells) { return align16((cells + 7) / 8 * 4); }
__host__ __device__ inline int32_t slab_ring_cols(int32_t maxspan) {
  return pow2_at_least(maxspan < 2 ? 2 : maxspan);
}
__host__ __device__ inline int64_t slab_bytes(int32_t rows, int64_t cells, int32_t maxspan) {
  return slab_hdr_bytes(rows) + slab_nib_bytes(cells) + int64_t(slab_ring_cols(maxspan)) * 8;
}


// One direction of the DP (R19) as a state machine advanced one cell per
// dir_step(): a thread's cells run in lock-step with its warp's other lanes
// whatever row, direction or pair each lane is in (the nested row / direction
// / pair loops written directly leave ~3 of 32 lanes active: every lane sits
// at another loop level).  a[i] = A[i * step] (i < la), b[j] = B[j * step]
// (j < lb); ring: mask + 1 int2 cells {H, F} indexed by column.  With
// nibw set, every computed cell's 4-bit code goes to the nibble stream (8 per
// 32-bit word, cells numbered row after row) and each row's {start column,
// first cell} to hdr[i]: bits 0-1 where H came from (0 diagonal, 1 E,
// 2 F: R22's order of preference), bit 2 E opened here, bit 3 F opened here.
// cap_cells / cap_rows bound the stream (a row that might not fit stops it:
// nibw = nullptr).  Row 0 is the generic row under a dead row -1 (its F
// values are -inf minus a gap cost instead of -inf: a live cell's H never
// comes from such an F, so nothing observable differs).
struct Dir {
  const uint8_t *A, *B;
  const int8_t *mrow;
  uint32_t *nibw;
  int2 *hdr;
  int64_t cum, r_cells, nc, cap_cells;  // cells of the rows done / of rows 0..best; next nibble
  uint32_t nword;
  int32_t cap_rows;
  int32_t step, la, lb, stop_row;
  int32_t i, j, start, phi, lo, hi;  // phi: last live cell of the previous row
  int32_t lh, le, dh;                // left H / E, previous row's H at j - 1
  int32_t best, best_row, bi, bj, maxspan_all, r_maxspan;
  bool done, overflow;
};

__device__ __forceinline__ void dir_finish(Dir &d) {
  if (d.nibw && (d.nc & 7)) {
    GCHECK(d.nc - 1 < d.cap_cells);
    d.nibw[d.nc >> 3] = d.nword;
  }
  d.done = true;
}

__device__ __forceinline__ void dir_end_row(Dir &d, const int8_t (*M)[32], const int2 *ring,
                                            int32_t mask) {
  if (d.lo < 0) {  // a row without live cells ends the extension
    dir_finish(d);
    return;
  }
  const int32_t span = d.j - d.start + 1;
  d.cum += span;
  d.maxspan_all = imax(d.maxspan_all, span);
  if (d.best_row == d.i) {
    d.r_cells = d.cum;
    d.r_maxspan = d.maxspan_all;
  }
  d.phi = d.hi;
  d.start = d.j = d.lo;  // cells left of the previous row's first live one are dead
  d.i += 1;
  if (d.i > d.la || d.i > d.stop_row) {
    dir_finish(d);
    return;
  }
  d.lo = d.hi = -1;
  d.lh = d.le = d.dh = kNeg;
  GCHECK(d.i - 1 < d.la);
  d.mrow = M[d.A[int64_t(d.i - 1) * d.step]];
  if (d.nibw) {
    if (d.cum + mask + 1 > d.cap_cells || d.i >= d.cap_rows) {
      d.nibw = nullptr;  // this row might not fit: no traceback store for this direction
    } else {
      GCHECK(d.i < d.cap_rows);
      d.hdr[d.i] = make_int2(d.start, int32_t(d.cum));
    }
  }
}

__device__ __forceinline__ void dir_begin(Dir &d, const uint8_t *A, const uint8_t *B, int step,
                                          int32_t la, int32_t lb, int32_t stop_row,
                                          const int8_t (*M)[32], int2 *ring, int32_t mask,
                                          uint32_t *nibw, int2 *hdr, int64_t cap_cells,
                                          int32_t cap_rows) {
  d.A = A;
  d.B = B;
  d.step = step;
  d.la = la;
  d.lb = lb;
  d.stop_row = stop_row;
  d.mrow = M[0];
  d.cum = d.r_cells = 0;
  d.i = d.j = d.start = 0;
  d.phi = -1;
  d.lo = d.hi = 0;  // the origin H(0,0) = 0 is live
  d.lh = 0;
  d.le = d.dh = kNeg;
  d.best = d.best_row = d.bi = d.bj = 0;
  d.maxspan_all = d.r_maxspan = 0;
  d.done = d.overflow = false;
  d.hdr = hdr;
  d.cap_cells = cap_cells;
  d.cap_rows = cap_rows;
  d.nibw = (nibw && mask + 1 <= cap_cells && cap_rows >= 1) ? nibw : nullptr;
  d.nc = 0;
  d.nword = 0;
  ring[0] = make_int2(0, kNeg);
  if (d.nibw) {
    hdr[0] = make_int2(0, 0);
    d.nword = 1;  // the origin's code (never read)
    d.nc = 1;
  }
  if (lb == 0) {
    dir_end_row(d, M, ring, mask);
  } else {
    d.j = 1;
  }
}

__device__ __forceinline__ void dir_step(Dir &d, const int8_t (*M)[32], int2 *ring, int32_t mask,
                                         int32_t ge, int32_t goe, int32_t X) {
  const int32_t j = d.j;
  // (loading the next cell's ring entry and residue one step ahead, carried
  // in registers, measured 5x slower: 300 vs 62 ms at config 3)
  const int2 up = (j <= d.phi) ? ring[j & mask] : make_int2(kNeg, kNeg);
  GCHECK(j <= d.lb && j >= d.start && (j <= d.phi || j > 0 || d.i == 0));
  const int32_t bres = j > 0 ? d.B[int64_t(j - 1) * d.step] : 0;
  const int32_t e = j > 0 ? imax(d.le - ge, d.lh - goe) : kNeg;
  const int32_t f = imax(up.y - ge, up.x - goe);
  const int32_t dg = (j > 0 && d.dh > kNeg) ? d.dh + d.mrow[bres] : kNeg;
  const int32_t hraw = imax(dg, imax(e, f));
  int32_t h = hraw, ee = e, ff = f;
  if (h < d.best - X) {
    h = ee = ff = kNeg;  // dead
  } else if (h > d.best) {
    d.best = h;
    d.best_row = d.i;
    d.bi = d.i;
    d.bj = j;
  }
  if (j - d.start > mask) {
    d.overflow = true;
    d.nibw = nullptr;
    d.done = true;
    return;
  }
  d.dh = up.x;
  ring[j & mask] = make_int2(h, ff);
  if (d.nibw) {
    const uint32_t code = uint32_t((hraw == dg ? 0 : (hraw == e ? 1 : 2)) |
                                   (e == d.lh - goe ? 4 : 0) | (f == up.x - goe ? 8 : 0));
    d.nword |= code << ((d.nc & 7) * 4);
    if ((d.nc & 7) == 7) {
      GCHECK(d.nc < d.cap_cells);
      d.nibw[d.nc >> 3] = d.nword;
      d.nword = 0;
    }
    ++d.nc;
  }
  d.lh = h;
  d.le = ee;
  bool row_end = (j == d.lb);
  if (h > kNeg) {
    if (d.lo < 0) d.lo = j;
    d.hi = j;
  } else if (j > d.phi && j > 0) {
    row_end = true;  // dead and beyond the previous row's live cells: the row ends
  }
  // (the row end as selects for every lane plus a small branch for its loads
  // and stores measured the same: 51.6 vs 51.2 ms)
  if (row_end) dir_end_row(d, M, ring, mask);
  else d.j = j + 1;
}

// R22 traceback from (bi, bj) over a direction's stored codes, one move per
// step.
struct Trace {
  int32_t i, j, state, ident, gopen, glen;
};
__device__ __forceinline__ bool trace_step(Trace &t, const uint8_t *A, const uint8_t *B, int step,
                                           const uint32_t *nibw, const int2 *hdr) {
  if (t.i == 0 && t.j == 0) return true;
  const int2 h = hdr[t.i];
  const int64_t c = int64_t(h.y) + (t.j - h.x);
  const int code = (nibw[c >> 3] >> ((c & 7) * 4)) & 15;
  if (t.state == 0) {
    const int src = code & 3;
    if (src == 0) {
      t.ident += A[int64_t(t.i - 1) * step] == B[int64_t(t.j - 1) * step];
      --t.i;
      --t.j;
    } else {
      t.state = src;  // 1: in E (gap in a), 2: in F (gap in b)
    }
  } else if (t.state == 1) {
    ++t.glen;
    if (code & 4) {
      ++t.gopen;
      t.state = 0;
    }
    --t.j;
  } else {
    ++t.glen;
    if (code & 8) {
      ++t.gopen;
      t.state = 0;
    }
    --t.i;
  }
  return false;
}

// BLOSUM62 (R18: the search's matrix), passed by value to the kernels
struct Matrix32 {
  int8_t m[32][32];
};
Matrix32 host_matrix() {
  Matrix32 h;
  for (int x = 0; x < 32; ++x)
    for (int y = 0; y < 32; ++y)
      h.m[x][y] = (x < kNumLetters && y < kNumLetters) ? kBlosum62[x][y] : int8_t(kSentinelScore);
  return h;
}
__device__ __forceinline__ void load_matrix(int8_t (*M)[32], const Matrix32 &src) {
  for (int t = threadIdx.x; t < 32 * 32; t += blockDim.x) M[t >> 5][t & 31] = src.m[t >> 5][t & 31];
  __syncthreads();
}

struct Subject {
  const uint8_t *S;
  int32_t ls;
};
__device__ __forceinline__ Subject subject_of(const GappedArgs &a, int64_t sidx) {
  const int64_t st = a.sstart[sidx];
  const int64_t en = sidx + 1 < a.nseq ? a.sstart[sidx + 1] - 1 : a.stream_end;
  return Subject{a.stream + st, int32_t(en - st)};
}

// pair starts, validation (ids in range, pairs contiguous = the list is in
// canonical order)
__global__ void gapped_flags_kernel(GappedArgs a, int32_t *flag, unsigned long long *counters) {
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < a.n;
       i += int64_t(gridDim.x) * blockDim.x) {
    const blastp_hsp h = a.hsps[i];
    const int64_t sidx = int64_t(h.subject_id) - a.subject_base;
    bool bad = h.query_id < 0 || h.query_id >= a.nq || sidx < 0 || sidx >= a.nseq ||
               h.length < 0 || h.q_start < 0 || h.s_start < 0;
    int32_t start = 1;
    if (i > 0) {
      const blastp_hsp p = a.hsps[i - 1];
      start = (p.query_id != h.query_id || p.subject_id != h.subject_id) ? 1 : 0;
      if (p.query_id > h.query_id || (p.query_id == h.query_id && p.subject_id > h.subject_id))
        bad = true;  // not in canonical order
    }
    flag[i] = start;
    if (bad) atomicOr(&counters[kErr], 1ull);
  }
}

__global__ void gapped_keys_kernel(GappedArgs a, const int32_t *flag, const int32_t *gid,
                                   unsigned long long *key, uint32_t *val, int32_t *gstart,
                                   unsigned long long *counters) {
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < a.n;
       i += int64_t(gridDim.x) * blockDim.x) {
    const int32_t g = gid[i] - 1;
    // descending score inside the pair; the stable sort keeps canonical
    // order among equal scores (R21)
    const uint32_t sk = ~(uint32_t(a.hsps[i].score) ^ 0x80000000u);
    key[i] = (static_cast<unsigned long long>(g) << 32) | sk;
    val[i] = uint32_t(i);
    if (flag[i]) gstart[g] = int32_t(i);
    if (i == a.n - 1) {
      gstart[g + 1] = int32_t(a.n);
      counters[kNumGroups] = static_cast<unsigned long long>(g + 1);
    }
  }
}

// pass 1a's work order: HSPs by descending ungapped score (high scores are
// the long homologous alignments; starting them first shortens the tail)
__global__ void gapped_order_keys_kernel(GappedArgs a, const uint32_t *perm, uint32_t *okey,
                                         uint32_t *oval) {
  for (int64_t k = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; k < a.n;
       k += int64_t(gridDim.x) * blockDim.x) {
    okey[k] = ~(uint32_t(a.hsps[perm[k]].score) ^ 0x80000000u);
    oval[k] = uint32_t(k);
  }
}

// Pass 1a's result for one direction of one HSP.
struct FirstDir {
  int32_t score, bi, bj, maxspan, logged, overflow;
  int64_t cells, nib_off, hdr_off;
  int32_t traced, ident, gopen, glen;  // traced: the traceback's counts are final
};

// pass 1a, thread form: every HSP's two directions as independent work items (item 2k:
// right, 2k + 1: left of the k-th HSP in R21 order), one DP cell per loop
// turn, codes appended to the thread's logs.  An alignment depends only on
// its own HSP; whether it is used (R21: its seed outside the boxes of the
// pair's earlier alignments) is decided afterwards by gapped_resolve_kernel,
// so a pair's HSPs run in parallel instead of as one thread's chain (the
// chain form left a 25 ms tail of pairs with many HSPs at config 3).  A
// direction outgrowing the ring sends its pair to the big-ring pass.
__global__ void __launch_bounds__(128) gapped_first_kernel(
    GappedArgs a, Matrix32 mat, const uint32_t *perm, const uint32_t *order, FirstDir *fd,
    int2 *scratch, int32_t ring_cols, uint32_t *nlog, int32_t nlog_words, int2 *hlog,
    int32_t hlog_rows, unsigned long long *counters) {
  __shared__ int8_t M[32][32];
  load_matrix(M, mat);
  const int64_t tid = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  int2 *ring = scratch + tid * ring_cols;
  const int64_t nbase = tid * nlog_words, hbase = tid * hlog_rows;
  int32_t ncur = 0, hcur = 0;
  const int32_t mask = ring_cols - 1, ge = a.gap_extend, goe = a.gap_open + a.gap_extend;
  const unsigned long long nitems = 2 * static_cast<unsigned long long>(a.n);
  Dir d;
  d.done = true;
  bool active = false;
  unsigned long long item = 0;
  for (;;) {
    if (active && !d.done) {  // the common turn: one cell, straight back to the top
      dir_step(d, M, ring, mask, ge, goe, a.xdrop);
      if (!d.done) continue;
    }
    if (active) {
      FirstDir f;
      f.score = d.best;
      f.bi = d.bi;
      f.bj = d.bj;
      f.maxspan = d.r_maxspan;
      f.cells = d.r_cells;
      f.overflow = d.overflow ? 1 : 0;
      f.logged = d.nibw != nullptr && !d.overflow ? 1 : 0;
      f.traced = f.ident = f.gopen = f.glen = 0;
      f.nib_off = nbase + ncur;
      f.hdr_off = hbase + hcur;
      if (f.logged) {
        ncur += int32_t((d.nc + 7) >> 3);
        hcur += d.i + 1;
      }
      fd[2 * int64_t(order[item >> 1]) + (item & 1)] = f;
      atomicAdd(&counters[kCells], static_cast<unsigned long long>(d.cum + (d.lo < 0 ? d.j - d.start + 1 : 0)));
      active = false;
    }
    item = atomicAdd(&counters[kCurFirst], 1ull);
    if (item >= nitems) break;
    const blastp_hsp h = a.hsps[perm[order[item >> 1]]];
    const uint8_t *Q = a.qcodes[h.query_id];
    const int32_t lq = a.qlens[h.query_id];
    const Subject sub = subject_of(a, int64_t(h.subject_id) - a.subject_base);
    const int32_t qm = h.q_start + h.length / 2, sm = h.s_start + h.length / 2;  // R20
    if (qm > lq || sm > sub.ls) {
      atomicOr(&counters[kErr], 2ull);
      continue;
    }
    if ((item & 1) == 0)
      dir_begin(d, Q + qm, sub.S + sm, 1, lq - qm, sub.ls - sm, INT32_MAX, M, ring, mask,
                nlog + nbase + ncur, hlog + hbase + hcur, int64_t(nlog_words - ncur) * 8,
                hlog_rows - hcur);
    else
      dir_begin(d, Q + qm - 1, sub.S + sm - 1, -1, qm, sm, INT32_MAX, M, ring, mask,
                nlog + nbase + ncur, hlog + hbase + hcur, int64_t(nlog_words - ncur) * 8,
                hlog_rows - hcur);
    active = true;
  }
}

// pass 1a, warp form (the default; BLASTP_GAPPED_KERNEL=thread selects the
// thread form above): one direction per warp,
// each row computed by the 32 lanes over 32 columns at a time.  R19 is
// sequential along a row only through E and the running best, and both are
// prefix maxima once the kills are taken out: with u_k = max(D_k, F_k) +
// ge * k, E_j = max_{k<j} u_k - go - ge * j (a gap never follows a gap), and
// the running best before cell j is the largest H of the row's earlier
// cells (a killed cell's H is below best - X, so neither it nor an E term
// from before it -- each below best - X for good -- can make a later cell
// live or move the best; the live cells' values, the best and the traceback
// codes are therefore R19's exactly).  The row ends at its first dead cell
// beyond the previous row's last live one (a ballot); the previous row is in
// a per-warp shared-memory ring; each 32-cell chunk's codes go to shared
// memory as 4 bit-planes (ballots), and lane 0 traces the direction back
// right away.  A direction whose rows outgrow the ring sends its pair to the
// big-ring pass; one whose codes outgrow the warp's log is traced by pass 2.
constexpr int kWRing = 256;       // ring columns (power of two)
constexpr int kWChunks = 256;     // 32-cell code chunks per warp (first launch)
constexpr int kWRows = 768;       // row headers per warp: start column | first chunk << 16
constexpr int kWWarps = 4;        // warps per block (first launch)
constexpr int kW2Chunks = 8192;   // second launch, one warp per block: 128 KB of chunks
constexpr int kW2Rows = 16384;    // + 64 KB of row headers
__host__ __device__ inline size_t warp_area_bytes(int chunks, int rows) {
  return size_t(kWRing) * 8 + size_t(chunks) * 16 + size_t(rows) * 4;
}

// kSecond: the directions pass 1b left over (work list, need > 0: a log that
// did not fit), one warp per block with a log as large as shared memory
// allows -- traced here, their counts added to the alignment, need cleared;
// any still too long stay for pass 2.
template <bool kSecond>
__global__ void __launch_bounds__(kWWarps * 32) gapped_warp_kernel(
    GappedArgs a, Matrix32 mat, const uint32_t *perm, const uint32_t *order, FirstDir *fd,
    const int32_t *work, int64_t *need, blastp_gapped *rec, int32_t cap_chunks, int32_t cap_rows,
    unsigned long long *counters) {
  __shared__ int8_t M[32][32];
  extern __shared__ __align__(16) uint8_t warp_smem[];
  load_matrix(M, mat);
  const int lane = threadIdx.x & 31;
  const size_t area = size_t(kWRing) * 8 + size_t(cap_chunks) * 16 + size_t(cap_rows) * 4;
  uint8_t *wbase = warp_smem + size_t(threadIdx.x >> 5) * area;
  int2 *ring = reinterpret_cast<int2 *>(wbase);
  uint4 *planes = reinterpret_cast<uint4 *>(wbase + size_t(kWRing) * 8);
  uint32_t *hdr = reinterpret_cast<uint32_t *>(wbase + size_t(kWRing) * 8 + size_t(cap_chunks) * 16);
  const int32_t ge = a.gap_extend, goe = a.gap_open + a.gap_extend, X = a.xdrop;
  const unsigned long long nitems =
      kSecond ? counters[kNumWork] : 2ull * static_cast<unsigned long long>(a.n);
  const unsigned FULL = 0xffffffffu;
  for (;;) {
    unsigned long long item = 0;
    if (lane == 0) item = atomicAdd(&counters[kSecond ? kCurBig : kCurFirst], 1ull);
    item = __shfl_sync(FULL, item, 0);
    if (item >= nitems) break;
    if (kSecond) {
      item = static_cast<unsigned long long>(work[item]);
      if (need[item] == 0) continue;  // a thread-form log: pass 2 traces it
    }
    const int64_t k = kSecond ? int64_t(item >> 1) : int64_t(order[item >> 1]);
    const bool right = (item & 1) == 0;
    const blastp_hsp h = a.hsps[perm[k]];
    const uint8_t *Q = a.qcodes[h.query_id];
    const int32_t lq = a.qlens[h.query_id];
    const Subject sub = subject_of(a, int64_t(h.subject_id) - a.subject_base);
    const int32_t qm = h.q_start + h.length / 2, sm = h.s_start + h.length / 2;  // R20
    if (qm > lq || sm > sub.ls) {
      if (lane == 0) atomicOr(&counters[kErr], 2ull);
      continue;
    }
    const uint8_t *A = right ? Q + qm : Q + qm - 1;
    const uint8_t *B = right ? sub.S + sm : sub.S + sm - 1;
    const int step = right ? 1 : -1;
    const int32_t la = right ? lq - qm : qm, lb = right ? sub.ls - sm : sm;
    int32_t best = 0, bi = 0, bj = 0, best_row = 0, i = 0, plo = 0, phi = -1;
    int64_t cum = 0, r_cells = 0;
    int32_t maxspan_all = 0, r_maxspan = 0, nch = 0;
    bool tb_ok = true, overflow = false, truncated = false;
    const int8_t *mrow = M[0];
    for (;;) {  // rows
      const int32_t start = plo;
      if (tb_ok) {
        // room for a full row of chunks; when the log is full, the rows after
        // the best row so far are dropped (the X-drop tail) -- a later move of
        // the best past them leaves the direction to pass 2
        if (nch + kWRing / 32 > cap_chunks) {
          if (best_row < i - 1) {
            nch = int32_t(hdr[best_row + 1] >> 16);
            truncated = true;
          } else {
            tb_ok = false;
          }
        }
        if (i >= cap_rows || start > 0xffff || nch + kWRing / 32 > 0xffff) tb_ok = false;
        if (tb_ok && lane == 0) hdr[i] = uint32_t(start) | (uint32_t(nch) << 16);
      }
      int32_t ucarry = kNeg, up_last = kNeg, h_last = kNeg;
      int32_t lo = -1, hi = -1, stop = -1;
      for (int32_t c0 = start;; c0 += 32) {
        const int32_t j = c0 + lane;
        const bool inr = j <= lb;
        int2 up = make_int2(kNeg, kNeg);
        if (inr && j <= phi) up = ring[j & (kWRing - 1)];
        int32_t dh = __shfl_up_sync(FULL, up.x, 1);
        if (lane == 0) dh = up_last;  // the previous chunk's last column (row start: dead)
        up_last = __shfl_sync(FULL, up.x, 31);
        int32_t d = kNeg;
        if (inr && j > 0 && dh > kNeg) d = dh + mrow[B[int64_t(j - 1) * step]];
        if (i == 0 && j == 0) d = 0;  // the origin
        const int32_t f = imax(up.y - ge, up.x - goe);
        const int32_t u = inr ? imax(d, f) + ge * j : kNeg;
        // (skipping this prefix maximum for chunks whose E bound is below best -
        // X measured 4% slower: the extra reduction costs more than it saves)
        // (a lane below the shuffle distance gets its own value back, which a
        // maximum ignores: no lane test)
        int32_t U = u;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) U = imax(U, __shfl_up_sync(FULL, U, o));
        int32_t Ux = __shfl_up_sync(FULL, U, 1);
        Ux = imax(lane == 0 ? kNeg : Ux, ucarry);
        const int32_t e = j > 0 ? Ux - goe - ge * (j - 1) : kNeg;
        const int32_t hraw = imax(d, imax(e, f));
        // running best before j: the carry, unless a cell of this chunk rises
        // above it (rare past the first rows) -- then a prefix maximum
        int32_t bprev = best;
        if (__reduce_max_sync(FULL, inr ? hraw : kNeg) > best) {
          int32_t Hm = inr ? hraw : kNeg;
#pragma unroll
          for (int o = 1; o < 32; o <<= 1) Hm = imax(Hm, __shfl_up_sync(FULL, Hm, o));
          const int32_t Hx = __shfl_up_sync(FULL, Hm, 1);
          bprev = imax(lane == 0 ? kNeg : Hx, best);
        }
        const bool live = inr && hraw >= bprev - X;
        const bool stopper = inr && ((!live && j > phi && j > 0) || j == lb);
        const unsigned sb = __ballot_sync(FULL, stopper);
        const int last = sb ? __ffs(sb) - 1 : 31;
        const bool valid = inr && lane <= last;
        // the best: the first live cell reaching the chunk's maximum, if above
        const int32_t cand = (valid && live) ? hraw : kNeg;
        const int32_t cm = __reduce_max_sync(FULL, cand);
        if (cm > best) {
          const unsigned at = __ballot_sync(FULL, cand == cm);
          if (truncated) tb_ok = false;  // rows between were dropped
          best = cm;
          bi = i;
          bj = c0 + __ffs(at) - 1;
          best_row = i;
        }
        const int32_t hs = live ? hraw : kNeg;
        if (valid) ring[j & (kWRing - 1)] = live ? make_int2(hraw, f) : make_int2(kNeg, kNeg);
        if (tb_ok) {
          int32_t lh = __shfl_up_sync(FULL, hs, 1);
          if (lane == 0) lh = h_last;
          const int src = hraw == d ? 0 : (hraw == e ? 1 : 2);
          const unsigned p0 = __ballot_sync(FULL, valid && (src & 1));
          const unsigned p1 = __ballot_sync(FULL, valid && (src & 2));
          const unsigned p2 = __ballot_sync(FULL, valid && e == lh - goe);
          const unsigned p3 = __ballot_sync(FULL, valid && f == up.x - goe);
          if (nch >= cap_chunks) {
            tb_ok = false;
          } else {
            if (lane == 0) planes[nch] = make_uint4(p0, p1, p2, p3);
            ++nch;
          }
        }
        h_last = __shfl_sync(FULL, hs, 31);
        const unsigned lv = __ballot_sync(FULL, valid && live);
        if (lv) {
          if (lo < 0) lo = c0 + __ffs(lv) - 1;
          hi = c0 + 31 - __clz(lv);
        }
        if (sb) {
          stop = c0 + last;
          break;
        }
        ucarry = imax(ucarry, __shfl_sync(FULL, U, 31));
        if (c0 + 64 - start > kWRing) {  // the next chunk would not fit the ring
          overflow = true;
          break;
        }
      }
      __syncwarp();  // the row's ring stores before the next row's loads
      if (overflow || lo < 0) break;  // a row without live cells ends the extension
      const int32_t span = stop - start + 1;
      cum += span;
      maxspan_all = imax(maxspan_all, span);
      if (best_row == i) {
        r_cells = cum;
        r_maxspan = maxspan_all;
      }
      plo = lo;
      phi = hi;
      ++i;
      if (i > la) break;
      mrow = M[A[int64_t(i - 1) * step]];
    }
    __syncwarp();
    FirstDir out;
    out.score = best;
    out.bi = bi;
    out.bj = bj;
    out.maxspan = r_maxspan;
    out.cells = r_cells;
    out.overflow = overflow ? 1 : 0;
    out.logged = 0;
    out.nib_off = out.hdr_off = 0;
    out.traced = 0;
    out.ident = out.gopen = out.glen = 0;
    if (!overflow && tb_ok && lane == 0) {  // R22 traceback over the bit-planes
      int32_t ti = bi, tj = bj, state = 0, idn = 0, gop = 0, gl = 0;
      while (ti > 0 || tj > 0) {
        const uint32_t hd = hdr[ti];
        const int32_t c = tj - int32_t(hd & 0xffffu);
        const uint4 pl = planes[(hd >> 16) + (c >> 5)];
        const int bit = c & 31;
        const int code = int((pl.x >> bit) & 1u) | (int((pl.y >> bit) & 1u) << 1) |
                         (int((pl.z >> bit) & 1u) << 2) | (int((pl.w >> bit) & 1u) << 3);
        if (state == 0) {
          const int src = code & 3;
          if (src == 0) {
            idn += A[int64_t(ti - 1) * step] == B[int64_t(tj - 1) * step];
            --ti;
            --tj;
          } else {
            state = src;
          }
        } else if (state == 1) {
          ++gl;
          if (code & 4) {
            ++gop;
            state = 0;
          }
          --tj;
        } else {
          ++gl;
          if (code & 8) {
            ++gop;
            state = 0;
          }
          --ti;
        }
      }
      out.traced = 1;
      out.ident = idn;
      out.gopen = gop;
      out.glen = gl;
    }
    if (kSecond) {
      if (out.traced && lane == 0) {
        atomicAdd(&rec[k].ident, out.ident);
        atomicAdd(&rec[k].gap_opens, out.gopen);
        atomicAdd(&rec[k].gap_len, out.glen);
        need[item] = 0;
      }
    } else if (lane == 0) {
      fd[2 * k + (right ? 0 : 1)] = out;
    }
    __syncwarp();
  }
}

// pass 1b: per pair, R21 over the alignments of pass 1a in the pair's order:
// an HSP whose seed lies in the box of an earlier kept alignment is skipped;
// pairs with an overflowing direction go to the big-ring pass.
__global__ void gapped_resolve_kernel(GappedArgs a, const uint32_t *perm, const int32_t *gstart,
                                      const FirstDir *fd, blastp_gapped *rec, uint8_t *status,
                                      DirInfo *dinfo, int64_t *need, int32_t *over_list,
                                      int32_t *work, unsigned long long *counters) {
  const int64_t ng = int64_t(counters[kNumGroups]);
  for (int64_t g = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; g < ng;
       g += int64_t(gridDim.x) * blockDim.x) {
    const int32_t g0 = gstart[g], g1 = gstart[g + 1];
    bool over = false;
    for (int32_t k = g0; k < g1 && !over; ++k) over = fd[2 * k].overflow || fd[2 * k + 1].overflow;
    if (over) {
      over_list[atomicAdd(&counters[kNumOver], 1ull)] = int32_t(g);
      continue;
    }
    for (int32_t k = g0; k < g1; ++k) {
      const blastp_hsp h = a.hsps[perm[k]];
      const int32_t qm = h.q_start + h.length / 2, sm = h.s_start + h.length / 2;  // R20
      bool inside = false;
      for (int32_t t = g0; t < k && !inside; ++t)
        if (status[t]) {
          const blastp_gapped &b = rec[t];
          inside = b.q_start <= qm && qm < b.q_end && b.s_start <= sm && sm < b.s_end;
        }
      status[k] = inside ? 0 : 1;
      if (inside) continue;
      const FirstDir R = fd[2 * k], L = fd[2 * k + 1];
      blastp_gapped o;
      o.query_id = h.query_id;
      o.subject_id = h.subject_id;
      o.q_start = qm - L.bi;
      o.q_end = qm + R.bi;
      o.s_start = sm - L.bj;
      o.s_end = sm + R.bj;
      o.score = L.score + R.score;
      // directions traced in pass 1a (warp kernel) count now; the others are
      // traced by pass 2 from the logs or re-run
      o.ident = (R.traced ? R.ident : 0) + (L.traced ? L.ident : 0);
      o.gap_opens = (R.traced ? R.gopen : 0) + (L.traced ? L.gopen : 0);
      o.gap_len = (R.traced ? R.glen : 0) + (L.traced ? L.glen : 0);
      rec[k] = o;
      if (o.score >= a.cutoff) {
        if (!R.traced) {
          dinfo[2 * k] = DirInfo{R.bi, R.bj, R.maxspan, R.logged, R.nib_off, R.hdr_off};
          if (!R.logged) need[2 * k] = slab_bytes(R.bi + 1, R.cells, R.maxspan);
          work[atomicAdd(&counters[kNumWork], 1ull)] = int32_t(2 * k);
        }
        if (!L.traced) {
          dinfo[2 * k + 1] = DirInfo{L.bi, L.bj, L.maxspan, L.logged, L.nib_off, L.hdr_off};
          if (!L.logged) need[2 * k + 1] = slab_bytes(L.bi + 1, L.cells, L.maxspan);
          work[atomicAdd(&counters[kNumWork], 1ull)] = int32_t(2 * k + 1);
        }
      }
    }
  }
}

// pass 1, general form (the big-ring pass): one thread per pair of a work
// list (work counter), the pair's HSPs in R21 order with the box test as it
// goes.  The thread's pairs, their HSPs (R21 order) and both
// directions of each run as one flat loop, one DP cell per turn.  The codes
// of each direction are appended to the thread's logs (nibbles: nlog_words
// 32-bit words; row headers: hlog_rows) and kept if the alignment is
// reported; pass 2 traces them back.  A direction that no longer fits is
// re-run by pass 2 into a store of its own (its need > 0).
// (minimum blocks 5 / 6 / 8 per SM: 96 / 80 / 64 registers with spills, 52-73 ms vs 49)
__global__ void __launch_bounds__(128) gapped_score_kernel(
    GappedArgs a, Matrix32 mat, const uint32_t *perm, const int32_t *gstart, blastp_gapped *rec,
    uint8_t *status, DirInfo *dinfo, int64_t *need, int2 *scratch, int32_t ring_cols,
    uint32_t *nlog, int32_t nlog_words, int2 *hlog, int32_t hlog_rows, int32_t *over_list,
    const int32_t *list, int list_count, int list_cursor, int32_t *work,
    unsigned long long *counters) {
  __shared__ int8_t M[32][32];
  load_matrix(M, mat);
  const int64_t tid = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  int2 *ring = scratch + tid * ring_cols;
  const int64_t nbase = tid * nlog_words, hbase = tid * hlog_rows;
  int32_t ncur = 0, hcur = 0;  // the logs' fill
  const int32_t mask = ring_cols - 1, ge = a.gap_extend, goe = a.gap_open + a.gap_extend;
  const unsigned long long ngroups = counters[list_count];
  Dir d;
  d.done = true;
  int phase = 0;  // 0 fetch, 1 DP
  int32_t g = 0, g0 = 0, g1 = 0, k = 0, cur = 0, side = 0;
  int32_t qm = 0, sm = 0, lq = 0, ls = 0;
  const uint8_t *Q = nullptr, *S = nullptr;
  int32_t r_score = 0, r_bi = 0, r_bj = 0, r_span = 0, n0 = 0, h0 = 0, r_n = 0, r_h = 0;
  int64_t r_cells = 0;
  bool r_logged = false;
  for (;;) {
    if (phase == 1 && !d.done) {  // the common turn: one cell, straight back to the top
      dir_step(d, M, ring, mask, ge, goe, a.xdrop);
      if (!d.done) continue;  // (this form: 49 ms; stepping and finishing in one turn: 61 ms)
    }
    if (phase == 1 && d.done) {
      if (d.overflow) {  // redo the whole pair with big rings
        for (int32_t t = g0; t < g1; ++t) {
          status[t] = 0;
          need[2 * t] = need[2 * t + 1] = 0;
          dinfo[2 * t].logged = dinfo[2 * t + 1].logged = 0;
        }
        over_list[atomicAdd(&counters[kNumOver], 1ull)] = g;
        k = g1;
        ncur = n0;
        hcur = h0;
        phase = 0;
      } else {
        const bool logged = d.nibw != nullptr;
        const int32_t used_n = logged ? int32_t((d.nc + 7) >> 3) : 0, used_h = logged ? d.i + 1 : 0;
        if (side == 0) {  // right done: the left direction from the pair before
          r_score = d.best;
          r_bi = d.bi;
          r_bj = d.bj;
          r_cells = d.r_cells;
          r_span = d.r_maxspan;
          r_logged = logged;
          r_n = ncur;
          r_h = hcur;
          ncur += used_n;
          hcur += used_h;
          side = 1;
          dir_begin(d, Q + qm - 1, S + sm - 1, -1, qm, sm, INT32_MAX, M, ring, mask,
                    nlog + nbase + ncur, hlog + hbase + hcur, int64_t(nlog_words - ncur) * 8,
                    hlog_rows - hcur);
          continue;
        }
        blastp_gapped o;
        o.query_id = rec[cur].query_id;
        o.subject_id = rec[cur].subject_id;
        o.q_start = qm - d.bi;
        o.q_end = qm + r_bi;
        o.s_start = sm - d.bj;
        o.s_end = sm + r_bj;
        o.score = d.best + r_score;
        o.ident = o.gap_opens = o.gap_len = 0;
        rec[cur] = o;
        status[cur] = 1;
        if (o.score >= a.cutoff) {  // reported: traced by pass 2 from the logs or re-run
          dinfo[2 * cur] = DirInfo{r_bi, r_bj, r_span, r_logged ? 1 : 0, nbase + r_n, hbase + r_h};
          dinfo[2 * cur + 1] = DirInfo{d.bi, d.bj, d.r_maxspan, logged ? 1 : 0, nbase + ncur,
                                       hbase + hcur};
          if (!r_logged) need[2 * cur] = slab_bytes(r_bi + 1, r_cells, r_span);
          if (!logged) need[2 * cur + 1] = slab_bytes(d.bi + 1, d.r_cells, d.r_maxspan);
          const unsigned long long wslot = atomicAdd(&counters[kNumWork], 2ull);
          work[wslot] = 2 * cur;
          work[wslot + 1] = 2 * cur + 1;
          ncur += used_n;
          hcur += used_h;
        } else {  // not reported: the logs forget both directions
          ncur = n0;
          hcur = h0;
        }
        phase = 0;
      }
    }
    if (phase != 0) continue;
    bool finished = false;
    while (phase == 0) {  // the next HSP to extend
      if (k >= g1) {
        const unsigned long long w = atomicAdd(&counters[list_cursor], 1ull);
        if (w >= ngroups) {
          finished = true;
          break;
        }
        g = list ? list[w] : int32_t(w);
        g0 = k = gstart[g];
        g1 = gstart[g + 1];
        n0 = ncur;  // the pair's first log position (a redo rewinds to it)
        h0 = hcur;
        continue;
      }
      cur = k++;
      status[cur] = 0;
      need[2 * cur] = need[2 * cur + 1] = 0;
      dinfo[2 * cur].logged = dinfo[2 * cur + 1].logged = 0;
      const blastp_hsp h = a.hsps[perm[cur]];
      Q = a.qcodes[h.query_id];
      lq = a.qlens[h.query_id];
      const Subject sub = subject_of(a, int64_t(h.subject_id) - a.subject_base);
      S = sub.S;
      ls = sub.ls;
      qm = h.q_start + h.length / 2;  // R20
      sm = h.s_start + h.length / 2;
      if (qm > lq || sm > ls) {
        atomicOr(&counters[kErr], 2ull);
        continue;
      }
      bool inside = false;  // R21: the seed inside an earlier alignment's box
      for (int32_t t = g0; t < cur && !inside; ++t)
        if (status[t]) {
          const blastp_gapped &b = rec[t];
          inside = b.q_start <= qm && qm < b.q_end && b.s_start <= sm && sm < b.s_end;
        }
      if (inside) continue;
      rec[cur].query_id = h.query_id;
      rec[cur].subject_id = h.subject_id;
      side = 0;
      n0 = ncur;  // this HSP's first log position (forgotten if not reported)
      h0 = hcur;
      dir_begin(d, Q + qm, S + sm, 1, lq - qm, ls - sm, INT32_MAX, M, ring, mask,
                nlog + nbase + ncur, hlog + hbase + hcur, int64_t(nlog_words - ncur) * 8,
                hlog_rows - hcur);
      phase = 1;
    }
    if (finished) break;
  }
}

// pass 2: per reported direction (work counter): a logged one is traced back
// from pass 1's logs; one that was not, if its store starts in [base, base +
// window), is re-run to its best row into that store and traced back.  One
// DP cell or one traceback move per loop turn.
__global__ void __launch_bounds__(128) gapped_trace_kernel(
    GappedArgs a, Matrix32 mat, const uint32_t *perm, blastp_gapped *rec, const DirInfo *dinfo,
    const int64_t *need, const int64_t *off, int64_t base, int64_t window, uint8_t *store,
    const uint32_t *nlog, const int2 *hlog, const int32_t *work, unsigned long long *counters) {
  __shared__ int8_t M[32][32];
  load_matrix(M, mat);
  const int32_t ge = a.gap_extend, goe = a.gap_open + a.gap_extend;
  Dir d;
  d.done = true;
  Trace tr{0, 0, 0, 0, 0, 0};
  int phase = 0;  // 0 fetch, 1 DP, 2 traceback
  int64_t item = 0;
  const unsigned long long nwork = counters[kNumWork];
  const uint32_t *nibw = nullptr;
  const int2 *hdr = nullptr;
  const uint8_t *A = nullptr, *B = nullptr;
  int step = 1;
  int2 *ring = nullptr;
  int32_t mask = 0;
  for (;;) {
    if (phase == 0) {
      bool got = false, logged = false;
      while (!got) {  // the directions resolve (or the big-ring pass) left to this pass
        const unsigned long long t = atomicAdd(&counters[kCurTrace], 1ull);
        if (t >= nwork) break;
        item = int64_t(work[t]);
        if (need[item] > 0) {
          got = off[item] >= base && off[item] < base + window;
        } else if (base == 0) {
          logged = got = dinfo[item].logged != 0;
        }
      }
      if (!got) break;
      const int64_t k = item >> 1;
      const bool right = (item & 1) == 0;
      const blastp_hsp h = a.hsps[perm[k]];
      const uint8_t *Q = a.qcodes[h.query_id];
      const int32_t lq = a.qlens[h.query_id];
      const Subject sub = subject_of(a, int64_t(h.subject_id) - a.subject_base);
      const int32_t qm = h.q_start + h.length / 2, sm = h.s_start + h.length / 2;
      const DirInfo di = dinfo[item];
      A = right ? Q + qm : Q + qm - 1;
      B = right ? sub.S + sm : sub.S + sm - 1;
      step = right ? 1 : -1;
      tr = Trace{di.bi, di.bj, 0, 0, 0, 0};
      if (logged) {
        nibw = nlog + di.nib_off;
        hdr = hlog + di.hdr_off;
        phase = 2;
        continue;
      }
      uint8_t *slab = store + (off[item] - base);
      const int32_t rows = di.bi + 1, rcols = slab_ring_cols(di.maxspan);
      int2 *shdr = reinterpret_cast<int2 *>(slab);
      uint32_t *snib = reinterpret_cast<uint32_t *>(slab + slab_hdr_bytes(rows));
      ring = reinterpret_cast<int2 *>(slab + need[item] - int64_t(rcols) * 8);
      mask = rcols - 1;
      // the store's capacities: rows 0..bi and their cells fit by construction
      // (+ one ring width: the per-row check is conservative by a row's span)
      const int64_t scells = (need[item] - slab_hdr_bytes(rows) - int64_t(rcols) * 8) * 2;
      dir_begin(d, A, B, step, right ? lq - qm : qm, right ? sub.ls - sm : sm, di.bi, M, ring,
                mask, snib, shdr, scells + mask + 1, rows);
      nibw = snib;
      hdr = shdr;
      phase = d.done ? 2 : 1;
      continue;
    }
    if (phase == 1) {
      dir_step(d, M, ring, mask, ge, goe, a.xdrop);
      if (d.done) phase = 2;
    } else if (trace_step(tr, A, B, step, nibw, hdr)) {
      blastp_gapped *r = rec + (item >> 1);
      atomicAdd(&r->ident, tr.ident);
      atomicAdd(&r->gap_opens, tr.gopen);
      atomicAdd(&r->gap_len, tr.glen);
      phase = 0;
    }
  }
}

__device__ __forceinline__ bool gapped_less(const blastp_gapped &x, const blastp_gapped &y) {
  const int32_t *u = reinterpret_cast<const int32_t *>(&x);
  const int32_t *v = reinterpret_cast<const int32_t *>(&y);
#pragma unroll
  for (int f = 0; f < 10; ++f)
    if (u[f] != v[f]) return u[f] < v[f];
  return false;
}

__global__ void gapped_count_kernel(const int32_t *gstart, const blastp_gapped *rec,
                                    const uint8_t *status, int32_t cutoff, int32_t *cnt,
                                    const unsigned long long *counters) {
  const int64_t ng = int64_t(counters[kNumGroups]);
  for (int64_t g = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; g < ng;
       g += int64_t(gridDim.x) * blockDim.x) {
    int32_t c = 0;
    for (int32_t k = gstart[g]; k < gstart[g + 1]; ++k) c += status[k] && rec[k].score >= cutoff;
    cnt[g] = c;
  }
}

// R21: the pair's reported alignments in canonical order (rank by counting;
// pairs hold few alignments), at the pair's offset
__global__ void gapped_emit_kernel(const int32_t *gstart, const blastp_gapped *rec,
                                   const uint8_t *status, int32_t cutoff, const int32_t *cnt,
                                   const int64_t *goff, blastp_gapped *out, int64_t cap,
                                   int64_t n, unsigned long long *counters) {
  const int64_t ng = int64_t(counters[kNumGroups]);
  for (int64_t g = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; g < ng;
       g += int64_t(gridDim.x) * blockDim.x) {
    const int32_t g0 = gstart[g], g1 = gstart[g + 1];
    for (int32_t k = g0; k < g1; ++k) {
      if (!status[k] || rec[k].score < cutoff) continue;
      int64_t rank = 0;
      for (int32_t u = g0; u < g1; ++u)
        if (u != k && status[u] && rec[u].score >= cutoff &&
            (gapped_less(rec[u], rec[k]) || (!gapped_less(rec[k], rec[u]) && u < k)))
          ++rank;
      const int64_t pos = goff[g] + rank;
      if (pos < cap) out[pos] = rec[k];
    }
    if (g == ng - 1) counters[kTotal] = static_cast<unsigned long long>(goff[g] + cnt[g]);
  }
  (void)n;
}

template <typename T>
cudaError_t alloc(T **p, size_t count, cudaStream_t s) {
  return pool_malloc_async(p, std::max<size_t>(count, 1) * sizeof(T), s);
}

}  // namespace

// Synchronous on s: reads the pair count, the traceback store size and the
// result count.  *h_count = the number of reported alignments (records beyond
// cap are not written).  *h_err: 0, or 1 = bad ids / not canonical, 2 = a
// seed outside its sequences.
cudaError_t launch_gapped(const GappedArgs &a, int num_sms, blastp_gapped *d_out, int64_t cap,
                          int64_t *h_count, int *h_err, cudaStream_t s) {
  *h_count = 0;
  *h_err = 0;
  if (a.n == 0) return cudaSuccess;
  if (a.n > (int64_t(1) << 30) - 1) return cudaErrorInvalidValue;  // 2n work items in an int
  const int64_t n = a.n;
  const Matrix32 mat = host_matrix();
  int32_t ring_small = 256;
  if (const char *v = std::getenv("BLASTP_GAPPED_RING"))  // tests: force the big-ring pass
    ring_small = pow2_at_least(std::max(2, std::min(1 << 16, std::atoi(v))));
  const int32_t ring_big = pow2_at_least(int32_t(std::min<int64_t>(a.max_subject_len + 2, 1 << 30)));
  const int threads = 128;
  // pass-1 blocks of 128 per SM: 4 (32.5 ms at config 3; 8: 31.0 ms but twice the logs'
  // memory, 3.6 GB, or half the log per thread and 38 MB of re-runs: 35.4 ms)
  int bps = 4;
  if (const char *v = std::getenv("BLASTP_GAPPED_BPS")) bps = std::max(1, std::min(16, std::atoi(v)));
  const int blocks1 = num_sms * bps;
  // per-thread logs of pass 1's codes: nibble words and row headers (the
  // nibble log in bytes; BLASTP_GAPPED_TBBUF=0: every direction re-run by pass 2)
  int32_t tb_bytes = 16384;  // + half as much for row headers: 24 KB per thread, 1.8 GB
  if (const char *v = std::getenv("BLASTP_GAPPED_TBBUF"))
    tb_bytes = std::max(0, std::min(1 << 20, std::atoi(v))) / 16 * 16;
  const int32_t nlog_words = tb_bytes / 4, hlog_rows = tb_bytes / 16;
  const bool verbose = std::getenv("BLASTP_GAPPED_VERBOSE") != nullptr;
  const int64_t t1 = int64_t(blocks1) * threads;
  const int64_t big_budget = int64_t(256) << 20;
  int64_t t2 = std::max<int64_t>(32, std::min<int64_t>(int64_t(num_sms) * 32,
                                                      big_budget / (int64_t(ring_big) * 8)));
  t2 = (t2 + 31) / 32 * 32;

  int32_t *flag = nullptr, *gid = nullptr, *gstart = nullptr, *over = nullptr, *cnt = nullptr,
          *work = nullptr;
  FirstDir *fd = nullptr;
  unsigned long long *key = nullptr, *key2 = nullptr, *counters = nullptr;
  uint32_t *val = nullptr, *perm = nullptr, *okey = nullptr, *okey2 = nullptr, *oval = nullptr,
           *order = nullptr;
  blastp_gapped *rec = nullptr;
  uint8_t *status = nullptr, *store = nullptr, *tbuf = nullptr;
  DirInfo *dinfo = nullptr;
  int64_t *need = nullptr, *off = nullptr, *goff = nullptr, *dmax = nullptr;
  int2 *scratch = nullptr, *scratch_big = nullptr;
  uint8_t *temp = nullptr;
  size_t temp_bytes = 0, tb = 0;
  cudaError_t e = cudaSuccess;
  auto cleanup = [&]() {
    void *ptrs[] = {flag, gid, gstart, over, cnt, key, key2, counters, val, perm, rec, status,
                    store, tbuf, dinfo, need, off, goff, dmax, scratch, scratch_big, temp, fd, okey, okey2, oval, order, work};
    for (void *p : ptrs)
      if (p) cudaFreeAsync(p, s);
  };
#define GTRY(expr)             \
  do {                         \
    if ((e = (expr)) != cudaSuccess) { \
      cleanup();               \
      return e;                \
    }                          \
  } while (0)
  int end_bit = 33;
  while ((int64_t(1) << (end_bit - 32)) <= n) ++end_bit;
  GTRY(cub::DeviceScan::InclusiveSum(nullptr, tb, flag, gid, int(n), s));
  temp_bytes = std::max(temp_bytes, tb);
  GTRY(cub::DeviceRadixSort::SortPairs(nullptr, tb, key, key2, val, perm, int(n), 0, end_bit, s));
  temp_bytes = std::max(temp_bytes, tb);
  GTRY(cub::DeviceScan::ExclusiveSum(nullptr, tb, need, off, int(2 * n), s));
  temp_bytes = std::max(temp_bytes, tb);
  GTRY(cub::DeviceReduce::Max(nullptr, tb, need, dmax, int(2 * n), s));
  temp_bytes = std::max(temp_bytes, tb);
  GTRY(cub::DeviceScan::ExclusiveSum(nullptr, tb, cnt, goff, int(n), s));
  temp_bytes = std::max(temp_bytes, tb);
  GTRY(cub::DeviceRadixSort::SortPairs(nullptr, tb, okey, okey2, oval, order, int(n), 0, 32, s));
  temp_bytes = std::max(temp_bytes, tb);

  GTRY(alloc(&flag, n, s));
  GTRY(alloc(&gid, n, s));
  GTRY(alloc(&gstart, n + 1, s));
  GTRY(alloc(&over, n, s));
  GTRY(alloc(&cnt, n, s));
  GTRY(alloc(&key, n, s));
  GTRY(alloc(&key2, n, s));
  GTRY(alloc(&counters, kNumCounters, s));
  GTRY(alloc(&val, n, s));
  GTRY(alloc(&perm, n, s));
  GTRY(alloc(&rec, n, s));
  GTRY(alloc(&status, n, s));
  GTRY(alloc(&dinfo, 2 * n, s));
  GTRY(alloc(&need, 2 * n, s));
  GTRY(alloc(&off, 2 * n, s));
  GTRY(alloc(&goff, n, s));
  GTRY(alloc(&dmax, 1, s));
  // pass 1a's form: the warp per direction (default) or BLASTP_GAPPED_KERNEL=thread,
  // whose per-thread rings and code logs (~1.8 GB) only it allocates
  const char *kv = std::getenv("BLASTP_GAPPED_KERNEL");
  const bool warp_form = !(kv && std::strcmp(kv, "thread") == 0);
  if (!warp_form) {
    GTRY(alloc(&scratch, size_t(t1) * ring_small, s));
    GTRY(alloc(&tbuf, size_t(t1) * (size_t(nlog_words) * 4 + size_t(hlog_rows) * 8), s));
  }
  uint32_t *nlog = reinterpret_cast<uint32_t *>(tbuf);
  int2 *hlog = reinterpret_cast<int2 *>(tbuf + size_t(t1) * size_t(nlog_words) * 4);
  GTRY(alloc(&fd, 2 * n, s));
  GTRY(alloc(&work, 2 * n, s));
  GTRY(alloc(&okey, n, s));
  GTRY(alloc(&okey2, n, s));
  GTRY(alloc(&oval, n, s));
  GTRY(alloc(&order, n, s));
  GTRY(alloc(&temp, temp_bytes, s));
  GTRY(cudaMemsetAsync(counters, 0, kNumCounters * sizeof(unsigned long long), s));
  GTRY(cudaMemsetAsync(cnt, 0, size_t(n) * sizeof(int32_t), s));
  GTRY(cudaMemsetAsync(dinfo, 0, size_t(2 * n) * sizeof(DirInfo), s));
  GTRY(cudaMemsetAsync(need, 0, size_t(2 * n) * sizeof(int64_t), s));

  const int gb = int(std::min<int64_t>((n + 255) / 256, int64_t(num_sms) * 16));
  gapped_flags_kernel<<<gb, 256, 0, s>>>(a, flag, counters);
  GTRY(cudaGetLastError());
  tb = temp_bytes;
  GTRY(cub::DeviceScan::InclusiveSum(temp, tb, flag, gid, int(n), s));
  gapped_keys_kernel<<<gb, 256, 0, s>>>(a, flag, gid, key, val, gstart, counters);
  GTRY(cudaGetLastError());
  tb = temp_bytes;
  GTRY(cub::DeviceRadixSort::SortPairs(temp, tb, key, key2, val, perm, int(n), 0, end_bit, s));
  unsigned long long hc[kNumCounters];
  GTRY(cudaMemcpyAsync(hc, counters, sizeof(hc), cudaMemcpyDeviceToHost, s));
  GTRY(cudaStreamSynchronize(s));
  if (hc[kErr]) {
    *h_err = int(hc[kErr]);
    cleanup();
    return cudaSuccess;
  }
  // pass 1: every HSP's two directions as independent items, R21 per pair,
  // then the pairs that overflowed the small rings (general kernel, big
  // rings, no logs)
  gapped_order_keys_kernel<<<gb, 256, 0, s>>>(a, perm, okey, oval);
  if (const char *v = std::getenv("BLASTP_GAPPED_ORDER"))  // A/B: 0 = the pairs' order
    if (std::atoi(v) == 0) GTRY(cudaMemsetAsync(okey, 0, size_t(n) * 4, s));
  GTRY(cudaGetLastError());
  tb = temp_bytes;
  GTRY(cub::DeviceRadixSort::SortPairs(temp, tb, okey, okey2, oval, order, int(n), 0, 32, s));
  // (warp form: 28 vs 31 ms for the thread form at config 3, same box)
  if (warp_form) {
    const size_t sm1 = size_t(kWWarps) * warp_area_bytes(kWChunks, kWRows);
    GTRY(cudaFuncSetAttribute(gapped_warp_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                              int(sm1)));
    gapped_warp_kernel<false><<<num_sms * 8, kWWarps * 32, sm1, s>>>(
        a, mat, perm, order, fd, nullptr, nullptr, nullptr, kWChunks, kWRows, counters);
  } else {
    gapped_first_kernel<<<blocks1, threads, 0, s>>>(a, mat, perm, order, fd, scratch, ring_small,
                                                    nlog, nlog_words, hlog, hlog_rows, counters);
  }
  GTRY(cudaGetLastError());
  gapped_resolve_kernel<<<gb, 128, 0, s>>>(a, perm, gstart, fd, rec, status, dinfo, need, over,
                                           work, counters);
  GTRY(cudaGetLastError());
  GTRY(cudaMemcpyAsync(hc, counters, sizeof(hc), cudaMemcpyDeviceToHost, s));
  GTRY(cudaStreamSynchronize(s));
  if (hc[kNumOver] > 0) {
    GTRY(alloc(&scratch_big, size_t(t2) * size_t(ring_big), s));
    gapped_score_kernel<<<int(t2 / 32), 32, 0, s>>>(a, mat, perm, gstart, rec, status, dinfo, need,
                                                    scratch_big, ring_big, nlog, 0, hlog, 0, over,
                                                    over, kNumOver, kCurBig, work, counters);
    GTRY(cudaGetLastError());
  }
  // the directions left over by the warp form, again by warps with large
  // shared-memory logs (a handful of long alignments: their thread-form re-runs
  // in pass 2 were a tail of single threads)
  if (warp_form && hc[kNumWork] > 0) {
    const size_t sm2 = warp_area_bytes(kW2Chunks, kW2Rows);
    GTRY(cudaFuncSetAttribute(gapped_warp_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                              int(sm2)));
    GTRY(cudaMemsetAsync(counters + kCurBig, 0, sizeof(unsigned long long), s));
    gapped_warp_kernel<true><<<num_sms, 32, sm2, s>>>(a, mat, perm, order, fd, work, need, rec,
                                                      kW2Chunks, kW2Rows, counters);
    GTRY(cudaGetLastError());
  }
  // traceback stores: exclusive scan of the needs, total and largest one
  tb = temp_bytes;
  GTRY(cub::DeviceScan::ExclusiveSum(temp, tb, need, off, int(2 * n), s));
  tb = temp_bytes;
  GTRY(cub::DeviceReduce::Max(temp, tb, need, dmax, int(2 * n), s));
  int64_t last[3] = {0, 0, 0};
  GTRY(cudaMemcpyAsync(&last[0], off + 2 * n - 1, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
  GTRY(cudaMemcpyAsync(&last[1], need + 2 * n - 1, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
  GTRY(cudaMemcpyAsync(&last[2], dmax, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
  GTRY(cudaMemcpyAsync(hc, counters, sizeof(hc), cudaMemcpyDeviceToHost, s));
  GTRY(cudaStreamSynchronize(s));
  if (hc[kErr]) {
    *h_err = int(hc[kErr]);
    cleanup();
    return cudaSuccess;
  }
  const int64_t total = last[0] + last[1], maxneed = last[2];
  if (verbose)
    fprintf(stderr, "gapped: %lld HSPs, %llu pairs, %llu pairs redone with %d-column rings "
            "(small %d), traceback store %.1f MB (largest %lld B), pass-1a cells %llu, "
            "directions left to pass 2 %llu\n",
            (long long)n, hc[kNumGroups], hc[kNumOver], ring_big, ring_small, total / 1e6,
            (long long)maxneed, hc[kCells], hc[kNumWork]);
  {  // pass 2: the logged directions (first window) and the re-runs, window by window
    int64_t window = std::max<int64_t>(std::min<int64_t>(total, int64_t(2) << 30), maxneed);
    if (const char *v = std::getenv("BLASTP_GAPPED_STORE"))  // tests: force several windows
      window = std::max<int64_t>(maxneed, std::atoll(v));
    window = std::max<int64_t>(window, 1);
    if (total > 0) GTRY(alloc(&store, size_t(window + maxneed), s));
    const int64_t items = int64_t(hc[kNumWork]);  // the directions left to this pass
    const int tblocks = int(std::min<int64_t>((items + threads - 1) / threads, int64_t(num_sms) * 8));
    for (int64_t base = 0; items > 0 && (base == 0 || base < total); base += window) {
      GTRY(cudaMemsetAsync(counters + kCurTrace, 0, sizeof(unsigned long long), s));
      gapped_trace_kernel<<<tblocks, threads, 0, s>>>(a, mat, perm, rec, dinfo, need, off, base,
                                                       window, store, nlog, hlog, work,
                                                       counters);
      GTRY(cudaGetLastError());
    }
  }
  // emit in canonical order
  const int eb = int(std::min<int64_t>((n + 127) / 128, int64_t(num_sms) * 16));
  gapped_count_kernel<<<eb, 128, 0, s>>>(gstart, rec, status, a.cutoff, cnt, counters);
  GTRY(cudaGetLastError());
  tb = temp_bytes;
  GTRY(cub::DeviceScan::ExclusiveSum(temp, tb, cnt, goff, int(n), s));
  gapped_emit_kernel<<<eb, 128, 0, s>>>(gstart, rec, status, a.cutoff, cnt, goff, d_out, cap, n,
                                        counters);
  GTRY(cudaGetLastError());
  GTRY(cudaMemcpyAsync(hc, counters, sizeof(hc), cudaMemcpyDeviceToHost, s));
  GTRY(cudaStreamSynchronize(s));
  *h_count = int64_t(hc[kTotal]);
  cleanup();
#undef GTRY
  return cudaStreamSynchronize(s);
}

}  // namespace blastp
