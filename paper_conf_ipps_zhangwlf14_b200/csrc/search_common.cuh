// search_common.cuh -- device helpers shared by the search kernels
// (search_block.cu: block two-hit state; search.cu: warp-private diagonal
// rings; search_cta.cu: CTA windows with per-diagonal buckets and
// warp-specialised extension).
#pragma once

#include <cuda_runtime.h>

#include "common.cuh"

namespace blastp {
namespace dev {

constexpr unsigned kFull = 0xffffffffu;
constexpr int kQPad = 4;  // sentinel codes before (and >= 4 after) the query codes

__host__ __device__ constexpr size_t align16(size_t x) { return (x + 15) & ~size_t(15); }

// BLOSUM62 extended to 32x32 codes, sentinel / unused codes score -128 (R2).
inline void fill_b62(int8_t *h) {
  for (int i = 0; i < 32; ++i)
    for (int j = 0; j < 32; ++j)
      h[i * 32 + j] = (i < kNumLetters && j < kNumLetters) ? kBlosum62[i][j]
                                                            : int8_t(kSentinelScore);
}

__device__ __forceinline__ unsigned lanemask_lt(int lane) { return (1u << lane) - 1u; }

__device__ __forceinline__ int score(const int8_t *b62, uint32_t qcode, uint32_t scode) {
  return b62[(qcode << 5) | scode];
}

__device__ __forceinline__ uint32_t ldg32(const uint8_t *p) {
  return __ldg(reinterpret_cast<const uint32_t *>(p));
}

// Work item ci of the chunk cursor without the segment pipeline: the long
// items whole (their single warp must not start last), then the regular
// plan.  False once all are taken.
__device__ __forceinline__ bool fetch_chunk(const SearchArgs &a, unsigned long long ci, Chunk &ch) {
  const unsigned long long nl = (unsigned long long)a.nlong;
  if (ci < nl) {
    ch = a.long_items[ci].c;
    return true;
  }
  ci -= nl;
  if (ci >= (unsigned long long)a.nchunks) return false;
  ch = a.chunks[ci];
  return true;
}

__device__ __forceinline__ unsigned ld_acquire(const unsigned *p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];\n" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release(unsigned *p, unsigned v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;\n" ::"l"(p), "r"(v) : "memory");
}

// Diagonal two-hit state, 16-bit positions, 0 = none:
//   last  most recent hit; far  largest hit <= last - W;
//   near  bit j set iff a hit at last - j (1 <= j < W).
// Append a hit at position p (> last).
__device__ __forceinline__ void st_append(uint32_t &last, uint32_t &far, uint32_t &near, int p,
                                          int W, uint32_t nearmask) {
  if (last != 0) {
    const int d = p - int(last);
    if (d >= W) {
      far = last;
      near = 0;
    } else {
      // near hits that fall out of (p-W, p): the largest becomes `far`
      const uint32_t gone = (near << d) & ~((1u << W) - 1u);
      if (gone) far = uint32_t(p - (__ffs(gone) - 1));
      near = ((near << d) | (1u << d)) & nearmask;
    }
  } else {
    near = 0;
  }
  last = uint32_t(p);
}

// Largest stored hit <= hi (hi > 0 frame position), or 0.
__device__ __forceinline__ int st_pred(uint32_t last, uint32_t far, uint32_t near, int hi) {
  if (last == 0) return 0;
  if (int(last) <= hi) return int(last);
  const int jmin = int(last) - hi;  // 1 .. W-1 when last < hi + W
  const uint32_t m = jmin < 32 ? near >> jmin : 0u;
  return m ? int(last) - (jmin + __ffs(m) - 1) : int(far);
}

// Four consecutive steps of the R8 scan (Fig. 8) on scores s0..s3 at offsets
// t..t+3, branch-free and exact: p_j = running sums, m_j = best after step j
// (max of the old best and p_0..p_j); the scan stops at the first j with
// m_j - p_j >= X, so the best is m_j* (= m_3 without a stop) and, if it rose,
// its length is the first step reaching it (strict >: shortest argmax).
// `run` is only meaningful while no stop has occurred.
__device__ __forceinline__ void xdrop_group4(int s0, int s1, int s2, int s3, int X, int t,
                                             int &run, int &best, int &bl, bool &stop) {
  const int p0 = run + s0, p1 = p0 + s1, p2 = p1 + s2, p3 = p2 + s3;
  const int m0 = max(best, p0), m1 = max(m0, p1), m2 = max(m1, p2), m3 = max(m2, p3);
  const bool st0 = m0 - p0 >= X, st1 = m1 - p1 >= X, st2 = m2 - p2 >= X, st3 = m3 - p3 >= X;
  const int mf = st0 ? m0 : st1 ? m1 : st2 ? m2 : m3;
  if (mf > best) bl = t + (p0 == mf ? 1 : p1 == mf ? 2 : p2 == mf ? 3 : 4);
  best = mf;
  run = p3;
  stop = st0 || st1 || st2 || st3;
}

// R7/R8: X-drop extension from the seed word at (q, sp).  qc is the query
// with kQPad sentinels before it and >= 4 after it; the stream has sentinels
// between subjects.  Sentinels score -128, which stops the walk at either
// sequence end.  Four residues per 32-bit load; the stop rule is applied
// position by position (predicated) so the result is exactly R8.
// `scanned` = residues examined (both sides, in groups of 4).
__device__ __forceinline__ void xdrop_extend(const uint8_t *__restrict__ stream, int64_t sp, int q,
                                             const uint8_t *qc, const int8_t *b62, int X,
                                             int &total, int &llen, int &rlen, int &scanned) {
  const uint8_t *qq = qc + kQPad;
  const int seed = score(b62, qq[q], __ldg(stream + sp)) +
                   score(b62, qq[q + 1], __ldg(stream + sp + 1)) +
                   score(b62, qq[q + 2], __ldg(stream + sp + 2));
  int run = 0, best = 0, bl = 0;
  {  // right, from (q+3, sp+3)
    const int64_t a = sp + 3;
    const uint8_t *base = stream + (a & ~int64_t(3));
    const uint32_t sh = uint32_t(a & 3) * 8;
    uint32_t lo = ldg32(base), hi = ldg32(base + 4);
    const uint8_t *qp = qq + q + 3;
    bool stop = false;
    int t = 0;
    for (; !stop; t += 4) {
      const uint32_t w = __funnelshift_r(lo, hi, sh);
      lo = hi;
      hi = ldg32(base + t + 8);
      xdrop_group4(score(b62, qp[t], w & 0xffu), score(b62, qp[t + 1], (w >> 8) & 0xffu),
                   score(b62, qp[t + 2], (w >> 16) & 0xffu), score(b62, qp[t + 3], w >> 24), X,
                   t, run, best, bl, stop);
    }
    scanned = t;
  }
  const int best_r = best;
  rlen = bl;
  run = 0;
  best = 0;
  bl = 0;
  {  // left, from (q-1, sp-1) downwards
    const int64_t a3 = sp - 4;  // bytes a3 .. a3+3 = positions sp-4 .. sp-1
    const uint8_t *base = stream + (a3 & ~int64_t(3));
    const uint32_t sh = uint32_t(a3 & 3) * 8;
    uint32_t lo = ldg32(base), hi = ldg32(base + 4);
    const uint8_t *qp = qq + q - 1;
    bool stop = false;
    int t = 0;
    for (; !stop; t += 4) {
      const uint32_t w = __funnelshift_r(lo, hi, sh);
      hi = lo;
      lo = ldg32(base - t - 4);
      xdrop_group4(score(b62, qp[-t], w >> 24), score(b62, qp[-(t + 1)], (w >> 16) & 0xffu),
                   score(b62, qp[-(t + 2)], (w >> 8) & 0xffu), score(b62, qp[-(t + 3)], w & 0xffu),
                   X, t, run, best, bl, stop);
    }
    scanned += t;
  }
  llen = bl;
  total = seed + best_r + best;
}

// EITHER mode (R6, Fig. 7 reading): a hit at (q+k, sp+k) for some k in
// [W, A-1], scored directly along the diagonal (the definition of a hit).
__device__ __forceinline__ bool has_successor(const uint8_t *__restrict__ stream, int64_t sp,
                                              int q, const uint8_t *qc, const int8_t *b62, int lq,
                                              int W, int A, int T) {
  // EITHER (R6): a later hit h' = h + k, W <= k < A, on h's diagonal and
  // subject -- the word pair at offset k scores >= T.  Residue scores r(j) =
  // B62[Q[q+j]][S[sp+j]], word(k) = r(k) + r(k+1) + r(k+2); the subject is
  // read four residues per 32-bit load (one sentinel test per load: a word
  // reaching the next subject is never a successor).
  const uint8_t *qq = qc + kQPad + q;
  const int kmax = min(A - 1, lq - 3 - q);
  if (kmax < W) return false;
  const uint32_t *__restrict__ sw = reinterpret_cast<const uint32_t *>(stream);
  const int64_t a0 = sp + 1;  // residues sp+1, sp+2, ... (r(1), r(2), ...)
  uint32_t wi = uint32_t(a0 >> 2);
  const uint32_t sh = uint32_t(a0 & 3) * 8;
  uint32_t lo = __ldg(sw + wi), hi = __ldg(sw + wi + 1);
  wi += 2;
  int s1 = 0, s2 = 0;  // r(j-2), r(j-1)
  const int jend = kmax + 2;  // last residue of the last word
  for (int j = 1; j <= jend; j += 4) {
    const uint32_t w = __funnelshift_r(lo, hi, sh);
    lo = hi;
    hi = __ldg(sw + wi);
    ++wi;
    // a sentinel byte (code 31) among the four: stop there (the words before
    // it were tested, the ones through it belong to no subject pair)
    const uint32_t x = w ^ 0x1f1f1f1fu;
    const uint32_t z = (x - 0x01010101u) & ~x & 0x80808080u;
#pragma unroll
    for (int b = 0; b < 4; ++b) {
      const int jj = j + b;
      if (jj > jend) return false;
      if ((z >> (8 * b + 7)) & 1u) return false;
      const int r = score(b62, qq[jj], (w >> (8 * b)) & 0xffu);
      const int k = jj - 2;
      if (k >= W && s1 + s2 + r >= T) return true;
      s1 = s2;
      s2 = r;
    }
  }
  return false;
}

__device__ __forceinline__ void trace_push(const SearchArgs &a, int which, int64_t sp, int q,
                                           int llen, int rlen, int sc) {
  unsigned long long i = atomicAdd(a.trace_count + which, 1ull);
  if ((long long)i < a.trace_cap[which]) {
    TraceRec r;
    r.sp = sp;
    r.q = q;
    r.llen = llen;
    r.rlen = rlen;
    r.score = sc;
    r.query_id = a.qv.query_id;
    r.pad = 0;
    a.trace[which][i] = r;
  }
}

// HSP record for an accepted extension of the seed at stream position sp;
// appended to the output if its score reaches the cutoff (R10).  The subject
// is found by binary search over [lo, hi) of the shard's subject starts.
__device__ __forceinline__ bool emit_hsp(const SearchArgs &a, int64_t sp, int q, int llen,
                                         int rlen, int total, int64_t lo, int64_t hi) {
  if (total < a.cutoff && !a.emit_seed) return false;
  hi -= 1;
  while (lo < hi) {
    const int64_t mid = (lo + hi + 1) >> 1;
    if (__ldg(a.sstart + mid) <= sp) lo = mid; else hi = mid - 1;
  }
  const int64_t s_local = sp - __ldg(a.sstart + lo);
  blastp_hsp h;
  h.query_id = a.qv.query_id;
  if (a.qv.nsub > 1) {
    // a query group: the member whose codes hold the seed (every extension
    // stops at the sentinels between members)
    int k = 0, hi_k = a.qv.nsub - 1;
    while (k < hi_k) {
      const int mid = (k + hi_k + 1) >> 1;
      if (__ldg(a.qv.sub + mid) <= q) k = mid; else hi_k = mid - 1;
    }
    q -= __ldg(a.qv.sub + k);
    h.query_id = __ldg(a.qv.sub + a.qv.nsub + k);
  }
  h.subject_id = int32_t(a.subject_base + lo);
  h.q_start = q - llen;
  h.s_start = int32_t(s_local) - llen;
  h.diagonal = h.s_start - h.q_start;
  h.length = llen + 3 + rlen;
  h.score = total;
  if (a.emit_seed) {  // ext_mode HIT_DEDUP: the seed record (blastp_dedup_covered_device)
    h.q_start = q;
    h.s_start = llen;
  }
  const unsigned long long idx = atomicAdd(a.hsp_count, 1ull);
  if ((long long)idx < a.out_cap) a.out[idx] = h;
  // a record stored into another GPU's memory over NVLink is performed at
  // system scope before the kernel can complete (blastp_search_ungapped_append)
#ifndef BLK_NOFENCE
  if (a.out_fence) __threadfence_system();
#endif
  return true;
}

}  // namespace dev
}  // namespace blastp
