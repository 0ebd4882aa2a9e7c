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
// B200 form.  The recurrences are sequential inside a row (E and the running
// best), and R21 is sequential inside a (query, subject) pair, so a pair is
// one thread's work; pairs are independent (~286K at config 3), which fills
// the GPU several times over.  Per thread one DP row lives in a ring of
// (H, F) int32 pairs indexed by subject column (global scratch, L1/L2
// resident): the live band of a row only drifts right (a cell left of the
// previous row's first live cell is dead), so a ring of C columns suffices
// while no row's computed span exceeds C; a pair whose span does is re-run by
// a second launch with rings the size of the longest subject.
//   order   : pairs = runs of equal (query, subject) in the canonical list;
//             a stable radix sort by (pair, descending score) gives R21's
//             order inside each pair;
//   pass 1  : (gapped_score_kernel) per pair: scores, boxes, containment,
//             and per reported direction the traceback store it needs (rows
//             and cells up to the best cell);
//   pass 2  : (gapped_trace_kernel) per reported direction: the DP re-run up
//             to the best row into its store (4 bits per cell: H source,
//             E opened, F opened), then the traceback (identities, gap
//             opens, gap residues);
//   emit    : (gapped_emit_kernel) per pair: its reported alignments in
//             canonical order at the pair's offset of an exclusive scan.
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_reduce.cuh>
#include <cub/device/device_scan.cuh>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdlib>

#include "common.cuh"

namespace blastp {

namespace {

constexpr int32_t kNeg = INT32_MIN / 4;  // -infinity that survives a few subtractions

// counters[]
enum { kCurPass1 = 0, kCurBig, kNumOver, kErr, kNumGroups, kTotal, kNumCounters = 8 };

struct DirInfo {
  int32_t bi, bj, maxspan, pad;
};

struct DirResult {
  int32_t score, bi, bj;
  int32_t maxspan;  // widest computed span among rows 0..bi
  int64_t cells;    // cells of those rows' spans
  bool overflow;
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
__host__ __device__ inline int64_t slab_nib_bytes(int64_t cells) { return align16((cells + 1) / 2); }
__host__ __device__ inline int64_t slab_bytes(int32_t rows, int64_t cells, int32_t maxspan) {
  return slab_hdr_bytes(rows) + slab_nib_bytes(cells) + int64_t(pow2_at_least(maxspan)) * 8;
}

__device__ __forceinline__ void put_nib(uint8_t *nib, int64_t c, uint8_t code) {
  if (c & 1) nib[c >> 1] |= uint8_t(code << 4);
  else nib[c >> 1] = code;
}

// One direction (R19): a[i] = A[i * step] (i < la), b[j] = B[j * step]
// (j < lb).  ring: mask + 1 int2 cells {H, F}.  Pass 2 passes nib/hdr and
// stop_row (the best row found by pass 1): the rows 0..stop_row are stored.
// Cell codes (pass 2): bits 0-1 where H came from (0 diagonal, 1 E, 2 F, in
// R22's order of preference), bit 2 E opened here, bit 3 F opened here.
__device__ DirResult gapped_dir(const uint8_t *A, const uint8_t *B, int step, int32_t la,
                                int32_t lb, const int8_t (*M)[32], int32_t go, int32_t ge,
                                int32_t X, int2 *ring, int32_t mask, uint8_t *nib, int2 *hdr,
                                int32_t stop_row) {
  DirResult r{0, 0, 0, 0, 0, false};
  const int32_t goe = go + ge;
  int32_t best = 0, best_row = 0, maxspan_all = 0;
  int64_t cum = 0;  // cells of the rows computed so far
  int32_t plo = 0, phi = 0;  // live range of the previous row
  // row 0: the origin, then a leading gap in b (E only)
  {
    int32_t lh = 0, le = kNeg, j = 1;
    ring[0] = make_int2(0, kNeg);
    if (nib) {
      hdr[0] = make_int2(0, 0);
      put_nib(nib, 0, 1);
    }
    for (; j <= lb; ++j) {
      int32_t e = imax(le - ge, lh - goe);
      const uint8_t code = uint8_t(1 | (e == lh - goe ? 4 : 0));
      int32_t h = e;                      // no diagonal, no F in row 0
      if (h < best - X) h = e = kNeg;     // (h > best is impossible: best = 0)
      if (j > mask) {
        r.overflow = true;
        return r;
      }
      ring[j & mask] = make_int2(h, kNeg);
      if (nib) put_nib(nib, j, code);
      lh = h;
      le = e;
      if (h > kNeg) phi = j;
      else break;  // dead at j >= up_end (= 1): nothing to its right is reachable
    }
    const int32_t span = (j <= lb ? j : lb) + 1;
    cum = span;
    maxspan_all = span;
    r.maxspan = span;
    r.cells = span;
  }
  for (int32_t i = 1; i <= la && stop_row >= i; ++i) {
    const int8_t *mrow = M[A[int64_t(i - 1) * step]];
    int32_t lh = kNeg, le = kNeg, dh = kNeg;  // cell plo - 1 of both rows is dead
    int32_t lo = -1, hi = -1, j = plo;
    const int32_t start = plo;
    if (nib) hdr[i] = make_int2(start, int32_t(cum));
    for (;; ++j) {
      const int2 up = (j <= phi) ? ring[j & mask] : make_int2(kNeg, kNeg);
      const int32_t e = j > 0 ? imax(le - ge, lh - goe) : kNeg;
      const int32_t f = imax(up.y - ge, up.x - goe);
      const int32_t d = (j > 0 && dh > kNeg) ? dh + mrow[B[int64_t(j - 1) * step]] : kNeg;
      int32_t h = imax(d, imax(e, f)), ee = e, ff = f;
      const uint8_t code = uint8_t((h == d ? 0 : (h == e ? 1 : 2)) | (e == lh - goe ? 4 : 0) |
                                   (f == up.x - goe ? 8 : 0));
      if (h < best - X) {
        h = ee = ff = kNeg;  // dead
      } else if (h > best) {
        best = h;
        best_row = i;
        r.bi = i;
        r.bj = j;
      }
      if (j - start > mask) {
        r.overflow = true;
        return r;
      }
      dh = up.x;
      ring[j & mask] = make_int2(h, ff);
      if (nib) put_nib(nib, cum + (j - start), code);
      lh = h;
      le = ee;
      if (h > kNeg) {
        if (lo < 0) lo = j;
        hi = j;
      } else if (j > phi && j > 0) {
        break;  // dead and beyond the previous row's live cells: the row ends
      }
      if (j == lb) break;
    }
    if (lo < 0) break;  // a row without live cells ends the extension
    const int32_t span = j - start + 1;
    cum += span;
    maxspan_all = imax(maxspan_all, span);
    if (best_row == i) {
      r.cells = cum;
      r.maxspan = maxspan_all;
    }
    plo = lo;
    phi = hi;
  }
  r.score = best;
  return r;
}

// R22 traceback from (bi, bj) over the pass-2 store: identities, gap opens,
// gap residues.
__device__ void traceback(const uint8_t *A, const uint8_t *B, int step, int32_t bi, int32_t bj,
                          const uint8_t *nib, const int2 *hdr, int32_t *ident, int32_t *gopen,
                          int32_t *glen) {
  int32_t i = bi, j = bj, state = 0, idn = 0, go = 0, gl = 0;
  while (i > 0 || j > 0) {
    const int2 h = hdr[i];
    const int64_t c = int64_t(h.y) + (j - h.x);
    const int code = (nib[c >> 1] >> ((c & 1) * 4)) & 15;
    if (state == 0) {
      const int src = code & 3;
      if (src == 0) {
        idn += A[int64_t(i - 1) * step] == B[int64_t(j - 1) * step];
        --i;
        --j;
      } else {
        state = src;  // 1: in E (gap in a), 2: in F (gap in b)
      }
    } else if (state == 1) {
      ++gl;
      if (code & 4) {
        ++go;
        state = 0;
      }
      --j;
    } else {
      ++gl;
      if (code & 8) {
        ++go;
        state = 0;
      }
      --i;
    }
  }
  *ident = idn;
  *gopen = go;
  *glen = gl;
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

// pass 1: one thread per pair (work counter), or per pair of the overflow
// list (big rings).
__global__ void __launch_bounds__(128) gapped_score_kernel(
    GappedArgs a, Matrix32 mat, const uint32_t *perm, const int32_t *gstart, blastp_gapped *rec,
    uint8_t *status, DirInfo *dinfo, int64_t *need, int2 *scratch, int32_t ring_cols,
    int32_t *over_list, bool big, unsigned long long *counters) {
  __shared__ int8_t M[32][32];
  load_matrix(M, mat);
  const int64_t tid = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  int2 *ring = scratch + tid * ring_cols;
  const int32_t mask = ring_cols - 1;
  const unsigned long long ngroups = big ? counters[kNumOver] : counters[kNumGroups];
  for (;;) {
    const unsigned long long w = atomicAdd(&counters[big ? kCurBig : kCurPass1], 1ull);
    if (w >= ngroups) break;
    const int32_t g = big ? over_list[w] : int32_t(w);
    const int32_t g0 = gstart[g], g1 = gstart[g + 1];
    bool over = false;
    for (int32_t k = g0; k < g1 && !over; ++k) {
      status[k] = 0;
      need[2 * k] = need[2 * k + 1] = 0;
      const blastp_hsp h = a.hsps[perm[k]];
      const uint8_t *Q = a.qcodes[h.query_id];
      const int32_t lq = a.qlens[h.query_id];
      const Subject sub = subject_of(a, int64_t(h.subject_id) - a.subject_base);
      const int32_t qm = h.q_start + h.length / 2, sm = h.s_start + h.length / 2;  // R20
      if (qm > lq || sm > sub.ls) {
        atomicOr(&counters[kErr], 2ull);
        continue;
      }
      bool inside = false;  // R21: the seed inside an earlier alignment's box
      for (int32_t t = g0; t < k && !inside; ++t)
        if (status[t]) {
          const blastp_gapped &b = rec[t];
          inside = b.q_start <= qm && qm < b.q_end && b.s_start <= sm && sm < b.s_end;
        }
      if (inside) continue;
      const DirResult R = gapped_dir(Q + qm, sub.S + sm, 1, lq - qm, sub.ls - sm, M, a.gap_open,
                                     a.gap_extend, a.xdrop, ring, mask, nullptr, nullptr, INT32_MAX);
      if (R.overflow) {
        over = true;
        break;
      }
      const DirResult L = gapped_dir(Q + qm - 1, sub.S + sm - 1, -1, qm, sm, M, a.gap_open,
                                     a.gap_extend, a.xdrop, ring, mask, nullptr, nullptr,
                                     INT32_MAX);
      if (L.overflow) {
        over = true;
        break;
      }
      blastp_gapped o;
      o.query_id = h.query_id;
      o.subject_id = h.subject_id;
      o.q_start = qm - L.bi;
      o.q_end = qm + R.bi;
      o.s_start = sm - L.bj;
      o.s_end = sm + R.bj;
      o.score = L.score + R.score;
      o.ident = o.gap_opens = o.gap_len = 0;
      rec[k] = o;
      status[k] = 1;
      dinfo[2 * k] = DirInfo{R.bi, R.bj, R.maxspan, 0};
      dinfo[2 * k + 1] = DirInfo{L.bi, L.bj, L.maxspan, 0};
      if (o.score >= a.cutoff) {  // reported: its traceback is needed
        need[2 * k] = slab_bytes(R.bi + 1, R.cells, R.maxspan);
        need[2 * k + 1] = slab_bytes(L.bi + 1, L.cells, L.maxspan);
      }
    }
    if (over) {  // redo the whole pair with big rings
      for (int32_t k = g0; k < g1; ++k) {
        status[k] = 0;
        need[2 * k] = need[2 * k + 1] = 0;
      }
      const unsigned long long slot = atomicAdd(&counters[kNumOver], 1ull);
      over_list[slot] = g;
    }
  }
}

// pass 2: per reported direction whose store starts in [base, base + window)
__global__ void __launch_bounds__(128) gapped_trace_kernel(
    GappedArgs a, Matrix32 mat, const uint32_t *perm, blastp_gapped *rec, const DirInfo *dinfo,
    const int64_t *need, const int64_t *off, int64_t base, int64_t window, uint8_t *store) {
  __shared__ int8_t M[32][32];
  load_matrix(M, mat);
  for (int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < 2 * a.n;
       t += int64_t(gridDim.x) * blockDim.x) {
    if (need[t] == 0 || off[t] < base || off[t] >= base + window) continue;
    const int64_t k = t >> 1;
    const bool right = (t & 1) == 0;
    const blastp_hsp h = a.hsps[perm[k]];
    const uint8_t *Q = a.qcodes[h.query_id];
    const int32_t lq = a.qlens[h.query_id];
    const Subject sub = subject_of(a, int64_t(h.subject_id) - a.subject_base);
    const int32_t qm = h.q_start + h.length / 2, sm = h.s_start + h.length / 2;
    const DirInfo di = dinfo[t];
    uint8_t *slab = store + (off[t] - base);
    int2 *hdr = reinterpret_cast<int2 *>(slab);
    const int32_t rows = di.bi + 1;
    const int64_t nib_bytes = need[t] - slab_hdr_bytes(rows) - int64_t(pow2_at_least(di.maxspan)) * 8;
    uint8_t *nib = slab + slab_hdr_bytes(rows);
    int2 *ring = reinterpret_cast<int2 *>(nib + nib_bytes);
    const uint8_t *A = right ? Q + qm : Q + qm - 1;
    const uint8_t *B = right ? sub.S + sm : sub.S + sm - 1;
    const int step = right ? 1 : -1;
    const int32_t la = right ? lq - qm : qm, lb = right ? sub.ls - sm : sm;
    gapped_dir(A, B, step, la, lb, M, a.gap_open, a.gap_extend, a.xdrop, ring,
               pow2_at_least(di.maxspan) - 1, nib, hdr, di.bi);
    int32_t idn, gop, gl;
    traceback(A, B, step, di.bi, di.bj, nib, hdr, &idn, &gop, &gl);
    atomicAdd(&rec[k].ident, idn);
    atomicAdd(&rec[k].gap_opens, gop);
    atomicAdd(&rec[k].gap_len, gl);
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
  if (a.n > int64_t(0x7ffffff0)) return cudaErrorInvalidValue;
  const int64_t n = a.n;
  const Matrix32 mat = host_matrix();
  int32_t ring_small = 512;
  if (const char *v = std::getenv("BLASTP_GAPPED_RING"))  // tests: force the big-ring pass
    ring_small = pow2_at_least(std::max(2, std::min(1 << 16, std::atoi(v))));
  const int32_t ring_big = pow2_at_least(int32_t(std::min<int64_t>(a.max_subject_len + 2, 1 << 30)));
  const int threads = 128;
  const int blocks1 = num_sms * 4;
  const int64_t t1 = int64_t(blocks1) * threads;
  const int64_t big_budget = int64_t(256) << 20;
  int64_t t2 = std::max<int64_t>(32, std::min<int64_t>(int64_t(num_sms) * 32,
                                                      big_budget / (int64_t(ring_big) * 8)));
  t2 = (t2 + 31) / 32 * 32;

  int32_t *flag = nullptr, *gid = nullptr, *gstart = nullptr, *over = nullptr, *cnt = nullptr;
  unsigned long long *key = nullptr, *key2 = nullptr, *counters = nullptr;
  uint32_t *val = nullptr, *perm = nullptr;
  blastp_gapped *rec = nullptr;
  uint8_t *status = nullptr, *store = nullptr;
  DirInfo *dinfo = nullptr;
  int64_t *need = nullptr, *off = nullptr, *goff = nullptr, *dmax = nullptr;
  int2 *scratch = nullptr, *scratch_big = nullptr;
  uint8_t *temp = nullptr;
  size_t temp_bytes = 0, tb = 0;
  cudaError_t e = cudaSuccess;
  auto cleanup = [&]() {
    void *ptrs[] = {flag, gid, gstart, over, cnt, key, key2, counters, val, perm, rec, status,
                    store, dinfo, need, off, goff, dmax, scratch, scratch_big, temp};
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
  GTRY(alloc(&scratch, size_t(t1) * ring_small, s));
  GTRY(alloc(&temp, temp_bytes, s));
  GTRY(cudaMemsetAsync(counters, 0, kNumCounters * sizeof(unsigned long long), s));
  GTRY(cudaMemsetAsync(cnt, 0, size_t(n) * sizeof(int32_t), s));

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
  // pass 1, then the pairs that overflowed the small rings
  gapped_score_kernel<<<blocks1, threads, 0, s>>>(a, mat, perm, gstart, rec, status, dinfo, need,
                                                  scratch, ring_small, over, false, counters);
  GTRY(cudaGetLastError());
  GTRY(cudaMemcpyAsync(hc, counters, sizeof(hc), cudaMemcpyDeviceToHost, s));
  GTRY(cudaStreamSynchronize(s));
  if (hc[kNumOver] > 0) {
    GTRY(alloc(&scratch_big, size_t(t2) * size_t(ring_big), s));
    gapped_score_kernel<<<int(t2 / 32), 32, 0, s>>>(a, mat, perm, gstart, rec, status, dinfo, need,
                                                    scratch_big, ring_big, over, true, counters);
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
  if (total > 0) {
    int64_t window = std::max<int64_t>(std::min<int64_t>(total, int64_t(2) << 30), maxneed);
    if (const char *v = std::getenv("BLASTP_GAPPED_STORE"))  // tests: force several windows
      window = std::max<int64_t>(maxneed, std::atoll(v));
    GTRY(alloc(&store, size_t(window + maxneed), s));
    const int64_t items = 2 * n;
    const int tblocks = int(std::min<int64_t>((items + threads - 1) / threads, int64_t(num_sms) * 8));
    for (int64_t base = 0; base < total; base += window) {
      gapped_trace_kernel<<<tblocks, threads, 0, s>>>(a, mat, perm, rec, dinfo, need, off, base,
                                                       window, store);
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
