// search_block.cu -- the default search kernel of filter_mode LEFT (sm_100a):
// hit detection, two-hit filter and X-drop ungapped extension fused per warp,
// with a per-diagonal "block" two-hit state that makes every 32-hit round
// conflict-free (no per-round loop over same-diagonal hits).
//
// Each warp owns a chunk of whole subjects at a time (work stealing) and
// walks it in ascending subject position, 32 positions per window, lane =
// position ("coalesced": one byte per lane, consecutive lanes,
// consecutive positions).
//
//   hit detection   Alg. 2: lane v looks up the word at its
//                   position in the query table (R3; radix-32 view, one
//                   8-byte L2 load: (first entry, count)), the window's hits
//                   are expanded in 32-hit rounds in s order.
//   bins / sort     P:L967-1343: replaced by a per-warp ring indexed by the
//                   diagonal (s - q) mod M, visited in ascending s -- the
//                   order the paper's segmented sort establishes.
//   two-hit filter  P:L1344-1351, reading R6 (LEFT): h passes iff a hit p on
//                   its diagonal and subject has W <= h - p < A.
//   extension       Alg. 3 + Fig. 8 (R7-R10): passing hits
//                   not covered by ext_reach are queued; 32 at a time are
//                   X-dropped lane-parallel and the ext_reach chain is
//                   resolved per diagonal in queue (= s) order.
//
// Block state.  Positions are cut into record blocks of 32:
// the window [b, b+32) of lanes is block k, split further at subject
// boundaries (a sentinel starts a new block: bid = max(b, last sentinel+1)).
// One 32-bit word per diagonal slot describes the hits recorded on it:
//   bid (14 bits, frame position of its block start; 0 = none),
//   min - bid, max - bid (5 bits each: the first and last hit of the block),
//   bid - prev (8 bits: prev = the last hit before the block; 0 = none).
// Test of a hit h at lane v, with L = W - 1:
//   * v >= L: valid predecessors are the block's hits <= h - W, and every
//     earlier hit (each is <= b - 1 <= h - W).  With A >= 32 + L every
//     block hit lies within A of h, so "a block hit <= h - W exists" is
//     "min <= h - W"; the earlier hits reduce to the largest (max of the
//     older state, or prev).  Hits of the same block in this round count
//     through the round's first member of the (slot, bid) group.
//   * v < L: h - W falls before the block, so h is tested against the
//     previous block's final state (the ring as the round starts): min of
//     that block <= h - W, else its prev.
// The state write is commutative per round: the group's first member gives
// min, its last member max, and the last member alone stores the word.
// Valid for filter LEFT when A >= 31 + W (block_kernel_eligible); other
// parameters run the warp kernel (search.cu), which keeps exact per-hit
// state (last / far / near) instead.
#include <cuda_runtime.h>

#include <algorithm>
#include <climits>
#include <cstdlib>
#include <cstring>

#include "search_common.cuh"

namespace blastp {

using namespace dev;

namespace {

// 2 CTAs of 18 warps per SM: 36 resident warps with <= 56 registers each
// (32 warps in one CTA: 2.4% slower on config 3, profiles/r02/ab_block_kernel.txt)
#ifndef BLK_WARPS
#define BLK_WARPS 18
#endif
#ifndef BLK_MINB
#define BLK_MINB 2
#endif
constexpr int kBlkWarps = BLK_WARPS;  // warps per CTA (independent walkers)
#ifdef BLK_PRMT  // A/B knob: X-drop scores from a [qcode][256] matrix indexed by one PRMT
constexpr int kBlkTab = 1024 + 8192;  // BLOSUM62 32x32 + the 32x256 X-drop matrix
#else
constexpr int kBlkTab = 1024;         // BLOSUM62 32x32
#endif
constexpr int kBlkMinCtas = BLK_MINB;  // CTAs per SM the register budget allows
constexpr int kBlkQcap = 64;         // extension queue slots per warp
constexpr int kBlkFrameMin = 512;    // first frame position (> A + 2 blocks)
constexpr int kBlkFrameSpan = 8192;  // rebase step: frame positions < 2^14
constexpr int kBlkFixed = 448;       // queue 256 B + flush / owner scratch 192 B

__constant__ int8_t c_b62_blk[32 * 32];

__device__ __forceinline__ int be_bid(uint32_t e) { return int(e & 0x3fffu); }
__device__ __forceinline__ int be_minoff(uint32_t e) { return int((e >> 14) & 31u); }
__device__ __forceinline__ int be_maxoff(uint32_t e) { return int((e >> 19) & 31u); }
__device__ __forceinline__ int be_prevoff(uint32_t e) { return int(e >> 24); }

// Per-warp shared memory: fixed parts first (every address is the warp's
// base plus a constant), then ring[M] (block state); reach[M] (ext_reach,
// read once per queued hit) in global memory, the warp's own region of
// a.reach_scratch (L1-resident; keeping it in shared memory costs 2 B per
// slot and 4 resident warps at q1054).
struct BlkArea {
  uint8_t *base;
  uint16_t *reach_g;
  __device__ __forceinline__ uint32_t *queue() const { return reinterpret_cast<uint32_t *>(base); }
  __device__ __forceinline__ uint32_t *scr() const { return reinterpret_cast<uint32_t *>(base + 256); }
  __device__ __forceinline__ uint16_t *fs_p() const { return reinterpret_cast<uint16_t *>(base + 256); }
  __device__ __forceinline__ uint16_t *fs_end() const { return fs_p() + 32; }
  __device__ __forceinline__ uint16_t *fs_acc() const { return fs_p() + 64; }
  __device__ __forceinline__ uint32_t *ring() const {
    return reinterpret_cast<uint32_t *>(base + kBlkFixed);
  }
  __device__ __forceinline__ uint16_t *reach() const { return reach_g; }
};

__host__ __device__ size_t blk_area_bytes(int ring) {
  return kBlkFixed + align16(size_t(ring) * 4);
}

struct BlkState {
  int64_t spbase;  // stream position of frame position 0
  int64_t first_subj, last_subj;
  int qhead, qcount;
  unsigned long long stat[kNumStats];  // tracing variant only
};

template <bool kStats>
__device__ __forceinline__ void bstat(BlkState &st, int i, unsigned long long v) {
  if (kStats) st.stat[i] += v;
}

// Query codes in shared memory with kBlkQPad sentinel codes on both sides
// (the X-drop's word loads stay inside the array).
constexpr int kBlkQPad = 16;

// PSSM: one row of 32 int8 scores per query
// position, row r = query position r - kBlkQPad (sentinel rows and codes
// score -128), PSSM[q][a] = BLOSUM62[query[q]][a] -- a perf-only switch
// (BLASTP_SCORE=pssm|pssm_global), the scores are identical.
__global__ void pssm_fill_kernel(const uint8_t *__restrict__ qcodes, int lq, int8_t *pssm) {
  const int rows = lq + 2 * kBlkQPad;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < rows * 32; i += gridDim.x * blockDim.x) {
    const int r = i >> 5, c = i & 31, k = r - kBlkQPad;
    const int qcode = (k >= 0 && k < lq) ? qcodes[k] : kSentinel;
    pssm[i] = c_b62_blk[qcode * 32 + c];
  }
}

// R7/R8 X-drop as xdrop_extend (search_common.cuh), the score of query
// position i against subject code c read as pssm[row(i)][c]: one load per
// residue instead of a query-code load and a matrix load.
__device__ __forceinline__ void xdrop_pssm(const uint8_t *__restrict__ stream, int64_t sp, int q,
                                           const int8_t *pssm, int X, int &total, int &llen,
                                           int &rlen, int &scanned) {
  const int8_t *pq = pssm + (q + kBlkQPad) * 32;
  const int seed = pq[int(__ldg(stream + sp))] + pq[32 + int(__ldg(stream + sp + 1))] +
                   pq[64 + int(__ldg(stream + sp + 2))];
  int run = 0, best = 0, bl = 0;
  {  // right, from (q+3, sp+3)
    const int64_t a = sp + 3;
    const uint8_t *base = stream + (a & ~int64_t(3));
    const uint32_t sh = uint32_t(a & 3) * 8;
    uint32_t lo = ldg32(base), hi = ldg32(base + 4);
    const int8_t *pr = pq + 96;
    bool stop = false;
    int t = 0;
    for (; !stop; t += 4) {
      const uint32_t w = __funnelshift_r(lo, hi, sh);
      lo = hi;
      hi = ldg32(base + t + 8);
      const int8_t *row = pr + t * 32;
      xdrop_group4(row[int(w & 0xffu)], row[32 + int((w >> 8) & 0xffu)],
                   row[64 + int((w >> 16) & 0xffu)], row[96 + int(w >> 24)], X, t, run, best, bl,
                   stop);
    }
    scanned = t;
  }
  const int best_r = best;
  rlen = bl;
  run = 0;
  best = 0;
  bl = 0;
  {  // left, from (q-1, sp-1) downwards
    const int64_t a3 = sp - 4;
    const uint8_t *base = stream + (a3 & ~int64_t(3));
    const uint32_t sh = uint32_t(a3 & 3) * 8;
    uint32_t lo = ldg32(base), hi = ldg32(base + 4);
    const int8_t *pl = pq - 32;
    bool stop = false;
    int t = 0;
    for (; !stop; t += 4) {
      const uint32_t w = __funnelshift_r(lo, hi, sh);
      hi = lo;
      lo = ldg32(base - t - 4);
      const int8_t *row = pl - t * 32;
      xdrop_group4(row[int(w >> 24)], row[-32 + int((w >> 16) & 0xffu)],
                   row[-64 + int((w >> 8) & 0xffu)], row[-96 + int(w & 0xffu)], X, t, run, best,
                   bl, stop);
    }
    scanned += t;
  }
  llen = bl;
  total = seed + best_r + best;
}

// R7/R8 X-drop, the same scan as search_common.cuh's xdrop_extend (Fig. 8's
// running sum / best / drop rule in branch-free groups of four), with the
// subject read as 32-bit words by a 32-bit word index from the stream base
// (one IMAD.WIDE per load): inside the round loop's register pressure the
// compiler otherwise rebuilds the 64-bit byte address every iteration.
__device__ __forceinline__ void blk_xdrop(const uint8_t *__restrict__ stream, int64_t sp, int q,
                                          const uint8_t *qc, const int8_t *b62, int X, int &total,
                                          int &llen, int &rlen, int &scanned) {
  const uint32_t *__restrict__ sw = reinterpret_cast<const uint32_t *>(stream);
  const uint8_t *qq = qc + kQPad;
  const int seed = score(b62, qq[q], __ldg(stream + sp)) +
                   score(b62, qq[q + 1], __ldg(stream + sp + 1)) +
                   score(b62, qq[q + 2], __ldg(stream + sp + 2));
  int run = 0, best = 0, bl = 0;
  {  // right, from (q+3, sp+3)
    const int64_t a = sp + 3;
    uint32_t wi = uint32_t(a >> 2);
    const uint32_t sh = uint32_t(a & 3) * 8;
    uint32_t lo = __ldg(sw + wi), hi = __ldg(sw + wi + 1);
    wi += 2;
    const uint8_t *qp = qq + q + 3;
    bool stop = false;
    int t = 0;
    for (; !stop; t += 4) {
      const uint32_t w = __funnelshift_r(lo, hi, sh);
      lo = hi;
      hi = __ldg(sw + wi);
      ++wi;
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
    uint32_t wi = uint32_t(a3 >> 2);
    const uint32_t sh = uint32_t(a3 & 3) * 8;
    uint32_t lo = __ldg(sw + wi), hi = __ldg(sw + wi + 1);
    --wi;
    const uint8_t *qp = qq + q - 1;
    bool stop = false;
    int t = 0;
    for (; !stop; t += 4) {
      const uint32_t w = __funnelshift_r(lo, hi, sh);
      hi = lo;
      lo = __ldg(sw + wi);
      --wi;
      xdrop_group4(score(b62, qp[-t], w >> 24), score(b62, qp[-(t + 1)], (w >> 16) & 0xffu),
                   score(b62, qp[-(t + 2)], (w >> 8) & 0xffu), score(b62, qp[-(t + 3)], w & 0xffu),
                   X, t, run, best, bl, stop);
    }
    scanned += t;
  }
  llen = bl;
  total = seed + best_r + best;
}

#ifdef BLK_PRMT
// prmt.b32 in its default mode: a selector nibble with bit 3 set replicates
// the sign of the selected byte (codes < 32: zero)
__device__ __forceinline__ uint32_t prmt(uint32_t a, uint32_t b, uint32_t sel) {
  uint32_t d;
  asm("prmt.b32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(sel));
  return d;
}
// byte k of the subject word | byte k of the query-code word << 8
template <int k>
__device__ __forceinline__ int xsc(const int8_t *bx, uint32_t w, uint32_t qw) {
  constexpr uint32_t sel = uint32_t(k) | (uint32_t(4 + k) << 4) | (uint32_t(8 | k) << 8) |
                           (uint32_t(8 | k) << 12);
  return bx[prmt(w, qw, sel)];
}

// blk_xdrop with the query codes read four per shared load (funnel-shifted
// like the subject) and each score one PRMT + one shared load from the
// [qcode][256] matrix bx (bx[(qcode << 8) | scode] = BLOSUM62[qcode][scode]).
__device__ __forceinline__ void blk_xdrop_prmt(const uint8_t *__restrict__ stream, int64_t sp,
                                               int q, const uint8_t *qcb, const int8_t *b62,
                                               const int8_t *bx, int X, int &total, int &llen,
                                               int &rlen, int &scanned) {
  const uint32_t *__restrict__ sw = reinterpret_cast<const uint32_t *>(stream);
  const uint32_t *qw = reinterpret_cast<const uint32_t *>(qcb);  // 16-byte aligned
  const uint8_t *qq = qcb + kBlkQPad;
  const int seed = score(b62, qq[q], __ldg(stream + sp)) +
                   score(b62, qq[q + 1], __ldg(stream + sp + 1)) +
                   score(b62, qq[q + 2], __ldg(stream + sp + 2));
  int run = 0, best = 0, bl = 0;
  {  // right, from (q+3, sp+3)
    const int64_t a = sp + 3;
    uint32_t wi = uint32_t(a >> 2);
    const uint32_t sh = uint32_t(a & 3) * 8;
    uint32_t lo = __ldg(sw + wi), hi = __ldg(sw + wi + 1);
    wi += 2;
    const uint32_t qa = uint32_t(kBlkQPad + q + 3);
    uint32_t qi = qa >> 2;
    const uint32_t qsh = (qa & 3u) * 8;
    uint32_t qlo = qw[qi], qhi = qw[qi + 1];
    qi += 2;
    bool stop = false;
    int t = 0;
    for (; !stop; t += 4) {
      const uint32_t w = __funnelshift_r(lo, hi, sh);
      const uint32_t qv = __funnelshift_r(qlo, qhi, qsh);
      lo = hi;
      hi = __ldg(sw + wi);
      ++wi;
      qlo = qhi;
      qhi = qw[qi];
      ++qi;
      xdrop_group4(xsc<0>(bx, w, qv), xsc<1>(bx, w, qv), xsc<2>(bx, w, qv), xsc<3>(bx, w, qv), X,
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
    uint32_t wi = uint32_t(a3 >> 2);
    const uint32_t sh = uint32_t(a3 & 3) * 8;
    uint32_t lo = __ldg(sw + wi), hi = __ldg(sw + wi + 1);
    --wi;
    const uint32_t qa = uint32_t(kBlkQPad + q - 4);  // query positions q-4 .. q-1
    uint32_t qi = qa >> 2;
    const uint32_t qsh = (qa & 3u) * 8;
    uint32_t qlo = qw[qi], qhi = qw[qi + 1];
    --qi;
    bool stop = false;
    int t = 0;
    for (; !stop; t += 4) {
      const uint32_t w = __funnelshift_r(lo, hi, sh);
      const uint32_t qv = __funnelshift_r(qlo, qhi, qsh);
      hi = lo;
      lo = __ldg(sw + wi);
      --wi;
      qhi = qlo;
      qlo = qw[qi];
      --qi;
      xdrop_group4(xsc<3>(bx, w, qv), xsc<2>(bx, w, qv), xsc<1>(bx, w, qv), xsc<0>(bx, w, qv), X,
                   t, run, best, bl, stop);
    }
    scanned += t;
  }
  llen = bl;
  total = seed + best_r + best;
}
#endif

// REGION: flush
// Extend up to 32 queued passing hits lane-parallel (R7-R9), then resolve the
// ext_reach chain (Alg. 3 L19-23, R10) per diagonal in queue (= s) order;
// kHit: Alg. 4, every passing hit extended and kept (reading R14).
template <bool kTrace, bool kHit, bool kPssm>
__device__ __forceinline__ void blk_flush(const SearchArgs &a, const BlkArea &w, BlkState &st,
                                          int n, const uint8_t *qc, const int8_t *b62, int lane,
                                          int slotc, int M, const int8_t *pssm) {
  const bool act = lane < n;
  uint32_t ent = 0;
  if (act) ent = w.queue()[(st.qhead + lane) & (kBlkQcap - 1)];
  const int P = int(ent & 0xffffu), q = int(ent >> 16);
  int slot = (P - q + slotc) % M;
  slot += slot < 0 ? M : 0;
  const int64_t sp = st.spbase + P;
  int total = 0, llen = 0, rlen = 0, scanned = 0;
  // (a variant reading the query codes four per shared load measured 3%
  // slower on config 3: DESIGN.md 5.9)
  if constexpr (kPssm) {
    if (act) xdrop_pssm(a.stream, sp, q, pssm, a.xdrop, total, llen, rlen, scanned);
  } else {
#ifdef BLK_OLD_XDROP  // A/B knob
    if (act) xdrop_extend(a.stream, sp, q, qc + (kBlkQPad - kQPad), b62, a.xdrop, total, llen,
                          rlen, scanned);
#elif defined(BLK_PRMT)
    if (act) blk_xdrop_prmt(a.stream, sp, q, qc, b62, b62 + 1024, a.xdrop, total, llen, rlen,
                            scanned);
#else
    if (act) blk_xdrop(a.stream, sp, q, qc + (kBlkQPad - kQPad), b62, a.xdrop, total, llen, rlen,
                       scanned);
#endif
  }
  if (kTrace) {
    bstat<kTrace>(st, kStatFlushes, 1);
    bstat<kTrace>(st, kStatExtended, n);
    bstat<kTrace>(st, kStatXdropSteps, __reduce_add_sync(kFull, unsigned(scanned)));
    bstat<kTrace>(st, kStatXdropLaneSlots, 32ull * __reduce_max_sync(kFull, unsigned(scanned)));
  }
  bool acc = false;
  if constexpr (kHit) {
    acc = act;
  } else {
    // HSP subject end (inclusive); < 2^16: P < 2^14 and an extension never
    // runs past the query (rlen < 16,000)
    const int endp = P + 2 + rlen;
    uint16_t *r16 = w.reach() + slot;
    const unsigned grp = __match_any_sync(kFull, act ? slot : -1);
    const bool uniq = grp == (1u << lane);
    if (__all_sync(kFull, uniq || !act)) {
      if (act) {
        acc = P > int(*r16);
        if (acc) *r16 = uint16_t(endp);
      }
    } else {
      w.fs_p()[lane] = uint16_t(P);
      w.fs_end()[lane] = uint16_t(endp);
      __syncwarp();
      if (act) {
        if (uniq) {
          acc = P > int(*r16);
          if (acc) *r16 = uint16_t(endp);
        } else if (lane == __ffs(grp) - 1) {
          int r = *r16;
          unsigned g = grp;
          while (g) {
            const int j = __ffs(g) - 1;
            g &= g - 1;
            const bool aj = int(w.fs_p()[j]) > r;
            if (aj) r = w.fs_end()[j];
            w.fs_acc()[j] = aj;
          }
          *r16 = uint16_t(r);
        }
      }
      __syncwarp();
      if (act && !uniq) acc = w.fs_acc()[lane] != 0;
    }
  }
  if (kTrace) {
    bstat<kTrace>(st, kStatAccepted, __popc(__ballot_sync(kFull, acc)));
    bstat<kTrace>(st, kStatEmitted, __popc(__ballot_sync(kFull, acc && total >= a.cutoff)));
  }
  if (acc) {
    if (kTrace) trace_push(a, 2, sp, q, llen, rlen, total);
    emit_hsp(a, sp, q, llen, rlen, total, st.first_subj, st.last_subj);
  }
  __syncwarp();
  st.qhead = (st.qhead + n) & (kBlkQcap - 1);
  st.qcount -= n;
}

// REGION: setup
// kDef: the default parameters (min_gap 3, window 40) as compile-time
// constants, else read from the arguments; kHit: ext_mode HIT (Alg. 4)
// instead of DIAGONAL (Alg. 3); kPssm: X-drop scores from a PSSM (in shared
// memory when a.pssm is null -- built here --, else a.pssm in global memory).
template <bool kTrace, bool kDef, bool kHit, bool kPssm>
__global__ void __launch_bounds__(kBlkWarps * 32, kBlkMinCtas) search_block_kernel(const SearchArgs a) {
  extern __shared__ __align__(16) uint8_t smem[];
  const int lq = a.qv.lq;
  int8_t *b62 = reinterpret_cast<int8_t *>(smem);
  uint8_t *qc = smem + kBlkTab;
  const size_t qc_bytes = align16(size_t(lq) + 2 * kBlkQPad);
  for (int i = threadIdx.x; i < 1024; i += blockDim.x) b62[i] = c_b62_blk[i];
#ifdef BLK_PRMT
  for (int i = threadIdx.x; i < 8192; i += blockDim.x)
    b62[1024 + i] = (i & 255) < 32 ? c_b62_blk[((i >> 8) << 5) | (i & 255)] : int8_t(0);
#endif
  for (int i = threadIdx.x; i < int(qc_bytes); i += blockDim.x) {
    const int k = i - kBlkQPad;
    qc[i] = (k >= 0 && k < lq) ? a.qv.qcodes[k] : uint8_t(kSentinel);
  }
  uint8_t *areas = smem + kBlkTab + qc_bytes;
  const int8_t *pssm = a.pssm;
  if constexpr (kPssm) {
    if (!pssm) {  // the PSSM in shared memory (hierarchical buffering)
      int8_t *ps = reinterpret_cast<int8_t *>(areas);
      const int rows = lq + 2 * kBlkQPad;
      for (int i = threadIdx.x; i < rows * 32; i += blockDim.x) {
        const int r = i >> 5, c = i & 31, k = r - kBlkQPad;
        const int qcode = (k >= 0 && k < lq) ? a.qv.qcodes[k] : kSentinel;
        ps[i] = c_b62_blk[qcode * 32 + c];
      }
      pssm = ps;
      areas += align16(size_t(rows) * 32);
    }
  }
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int M = a.ring;
  BlkArea w;
  w.base = areas + size_t(warp) * blk_area_bytes(M);
  w.reach_g = a.reach_scratch + size_t(blockIdx.x * (blockDim.x >> 5) + warp) * M;
  for (int i = lane; i < M; i += 32) {
    w.ring()[i] = 0;
    w.reach()[i] = 0;
  }
  __syncthreads();

  const uint8_t *__restrict__ stream = a.stream;
  const uint2 *__restrict__ wtab = a.qv.wtab;
  const uint16_t *__restrict__ qpos = a.qv.qpos;
  const int W = kDef ? 3 : a.min_gap;
  const int L = W - 1;  // record lag: lanes v < L are tested against the previous block
  const int A = kDef ? 40 : a.window;
  const unsigned ltmask = lanemask_lt(lane);
  uint32_t *scr = w.scr();

  BlkState st;
  if (kTrace)
    for (int i = 0; i < kNumStats; ++i) st.stat[i] = 0;
  st.qhead = 0;
  st.qcount = 0;
  int frame = kBlkFrameMin;  // frame position of the next work item's first residue
  int base_slot = 0;         // ring slot of (P, q) = base_slot + (P - b) - q (mod M)
  // ring slot of (P, q) = P - q + slotc (mod M): b and base_slot advance
  // together, so slotc only changes when the frame is rebased
  int slotc = (M - kBlkFrameMin % M) % M;
  const unsigned long long nsegs = (unsigned long long)a.nsegs;
  const unsigned long long nitems = nsegs + (unsigned long long)a.nlong;
  for (;;) {
    unsigned long long ci = 0;
    if (lane == 0) ci = atomicAdd(a.chunk_cursor, 1ull);
    ci = __shfl_sync(kFull, ci, 0);
    int64_t wstart, wend;
    int64_t dlo = INT64_MIN, dhi = INT64_MAX;
    if (ci < nsegs) {
      // A long subject cut by diagonal range: segment j owns
      // the diagonals (stream position - q) in [d_j, d_j + seg_len) --
      // segment 0 also those below the chunk start -- and walks the positions
      // [d_j, d_j + seg_len + Lq) where all of their hits lie, so each of its
      // diagonals' whole R6 / R10 history stays inside the segment.
      const LongItem it = a.long_items[a.seg_item[ci]];
      const int j = int(ci) - it.seg0;
      const int64_t d0 = it.c.start + int64_t(j) * a.seg_len;
      dlo = j == 0 ? INT64_MIN : d0;
      dhi = j == it.nseg - 1 ? INT64_MAX : d0 + a.seg_len;
      wstart = d0;
      wend = j == it.nseg - 1 ? it.c.end : min(it.c.end, d0 + a.seg_len + lq);
      st.first_subj = it.c.first_subj;
      st.last_subj = it.c.last_subj;
    } else if (ci < nitems) {
      const LongItem it = a.long_items[ci - nsegs];
      if (it.nseg > 0) continue;  // covered by its diagonal segments
      wstart = it.c.start;
      wend = it.c.end;
      st.first_subj = it.c.first_subj;
      st.last_subj = it.c.last_subj;
    } else {
      const unsigned long long cj = ci - nitems;
      if (cj >= (unsigned long long)a.nchunks) break;
      const Chunk ch = a.chunks[cj];
      wstart = ch.start;
      wend = ch.end;
      st.first_subj = ch.first_subj;
      st.last_subj = ch.last_subj;
    }

    st.spbase = wstart - frame;
    const bool seg = dlo != INT64_MIN || dhi != INT64_MAX;
    int dlo_f = dlo != INT64_MIN ? int(dlo - st.spbase) : INT_MIN;
    int dhi_f = dhi != INT64_MAX ? int(dhi - st.spbase) : INT_MAX;
    int b = frame;             // frame position of lane 0 (block start)
    int lastsent = frame - 1;  // the sentinel before the work item
    int end = int(wend - st.spbase);

    // REGION: window
    // Software pipeline over windows: residues two windows ahead (one byte
    // per lane + two of overlap), the table lookup one window ahead.
    uint32_t pf_r = 0, pf_x = 0;
    auto load_res = [&](int wn) {
      const int64_t pp = st.spbase + wn;
      pf_r = __ldg(stream + pp + lane);
      pf_x = lane < 2 ? __ldg(stream + pp + 32 + lane) : 0u;
    };
    uint32_t nx_o = 0, nx_c = 0;
    bool nx_s = false;
    auto lookup = [&](int wn) {  // consumes pf_* (residues of window wn)
      const uint32_t r0 = pf_r;
      uint32_t r1 = __shfl_down_sync(kFull, pf_r, 1), r2 = __shfl_down_sync(kFull, pf_r, 2);
      const uint32_t x0 = __shfl_sync(kFull, pf_x, 0), x1 = __shfl_sync(kFull, pf_x, 1);
      if (lane == 31) {
        r1 = x0;
        r2 = x1;
      }
      if (lane == 30) r2 = x0;
      load_res(wn + 32);
      const bool in = wn + lane < end;
      nx_s = in && r0 == uint32_t(kSentinel);
      uint2 t = make_uint2(0u, 0u);
      if (in) t = __ldg(wtab + ((r0 << 10) | (r1 << 5) | r2));
      nx_o = t.x;
      nx_c = t.y;
    };
    load_res(b);
    lookup(b);

    while (b < end) {
      // ---- rebase the frame before positions outgrow 14 bits -------------
      if (b >= kBlkFrameMin + kBlkFrameSpan) {
        while (st.qcount > 0)
          blk_flush<kTrace, kHit, kPssm>(a, w, st, min(st.qcount, 32), qc, b62, lane, slotc, M, pssm);
        slotc = (slotc + kBlkFrameSpan) % M;
        for (int i = lane; i < M; i += 32) {
          const uint32_t e = w.ring()[i];
          // a state whose block starts before the new frame origin is older
          // than any window A can reach back to: dropped
          w.ring()[i] = be_bid(e) > kBlkFrameSpan ? e - uint32_t(kBlkFrameSpan) : 0u;
          const uint32_t r = w.reach()[i];
          w.reach()[i] = uint16_t(r > uint32_t(kBlkFrameSpan) ? r - kBlkFrameSpan : 0u);
        }
        __syncwarp();
        st.spbase += kBlkFrameSpan;
        b -= kBlkFrameSpan;
        lastsent -= kBlkFrameSpan;
        end -= kBlkFrameSpan;
        if (dlo_f != INT_MIN) dlo_f -= kBlkFrameSpan;
        if (dhi_f != INT_MAX) dhi_f -= kBlkFrameSpan;
      }
      bstat<kTrace>(st, kStatIterations, 1);
      // ---- this window's lookup (issued last iteration); issue the next ---
      const uint32_t o = nx_o, cnt = nx_c;
      const unsigned sm = __ballot_sync(kFull, nx_s);
      lookup(b + 32);
      uint32_t incl = cnt;
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) {
        const uint32_t t = __shfl_up_sync(kFull, incl, d);
        if (lane >= d) incl += t;
      }
      const uint32_t excl = incl - cnt;
      const uint32_t Hn = __shfl_sync(kFull, incl, 31);
      // last sentinel at or before each lane (before the window: lastsent)
      const unsigned prior = sm & ((lane == 31) ? kFull : ((2u << lane) - 1u));
      const int ls_lane = prior ? (b + 31 - __clz(prior)) : lastsent;

      if (Hn) {
        // Owner lane and query position of hit kb + lane: each lane whose run
        // of hits intersects [kb, kb + 32) stores (lane, table offset -
        // excl) at the slot of its run's first hit in the round; a hit's
        // owner is the last run start at or before it (OR-reduced mask).
        // REGION: locate
        auto locate = [&](uint32_t kb, uint32_t lim, int &own_out, int &q_out) {
          const bool wr = cnt != 0u && excl < kb + 32u && incl > kb;
          const int p0 = wr ? max(int(excl) - int(kb), 0) : 0;
          // (table offset - excl) << 5 | lane: the offset difference is
          // taken mod 2^27 (tables < 2^27 entries)
          if (wr) scr[p0] = uint32_t(lane) | ((o - excl) << 5);
          const unsigned S = __reduce_or_sync(kFull, wr ? (1u << p0) : 0u);
          __syncwarp();
          const int src = 31 - __clz(S & (kFull >> (31 - lane)));
          const uint32_t vv = scr[src];
          own_out = int(vv & 31u);
          const uint32_t k = kb + uint32_t(lane);
          q_out = k < lim ? int(__ldg(qpos + (((vv >> 5) + k) & 0x7ffffffu))) : 0;
          __syncwarp();
        };
        // hits of lanes v < L (tested against the previous block's state)
#ifdef BLK_LAST3  // exact recent positions: no lag, no prepass
        const uint32_t CL = 0u;
        const bool pre_ok = true;
#else
        const uint32_t CL = L > 0 ? __shfl_sync(kFull, incl, L - 1) : 0u;
        const bool pre_ok = CL <= 32u;  // all of them in the first round
#endif
        // REGION: enqueue
        auto enqueue = [&](bool enq, int P, int q) {
          const unsigned bal = __ballot_sync(kFull, enq);
          if (bal) {
            if (enq)
              w.queue()[(st.qhead + st.qcount + __popc(bal & ltmask)) & (kBlkQcap - 1)] =
                  uint32_t(P) | (uint32_t(q) << 16);
            st.qcount += __popc(bal);
            __syncwarp();
            if (st.qcount >= 32)
              blk_flush<kTrace, kHit, kPssm>(a, w, st, 32, qc, b62, lane, slotc, M, pssm);
          }
        };
        // REGION: prepass
        if (!pre_ok) {
          // rare (> 32 hits on the first L positions): test those hits
          // before any of this window's records, in rounds of their own
          for (uint32_t k0 = 0; k0 < CL; k0 += 32) {
            int v, q;
            locate(k0, CL, v, q);
            const int P = b + v;
            bool act = k0 + uint32_t(lane) < CL;
            if (seg) act = act && P - q >= dlo_f && P - q < dhi_f;
            int slot = base_slot + v - q;
            slot += slot < 0 ? M : 0;
            slot -= slot >= M ? M : 0;
            const int lsv = __shfl_sync(kFull, ls_lane, v);
            const uint32_t e = act ? w.ring()[slot] : 0u;
            const int ebid = be_bid(e);
            const int bt = max(b - 32, lsv + 1);
            const int lo_ok = max(P - A + 1, lsv + 1);
            int pv = ebid ? ebid + be_maxoff(e) : 0;
            bool pin = false;
            if (ebid == bt) {
              pin = ebid + be_minoff(e) <= P - W;
              pv = be_prevoff(e) ? ebid - be_prevoff(e) : 0;
            }
            const bool pass = act && (pin || pv >= lo_ok);
            bool enq = pass;
            if (!kHit && pass) enq = P > int(w.reach()[slot]);
            if (kTrace) {
              bstat<kTrace>(st, kStatPassing, __popc(__ballot_sync(kFull, pass)));
              bstat<kTrace>(st, kStatEnqueued, __popc(__ballot_sync(kFull, enq)));
              if (pass) trace_push(a, 1, st.spbase + P, q, 0, 0, 0);
            }
            enqueue(enq, P, q);
            __syncwarp();
          }
        }
        const bool multi_bid_possible = sm != 0u;
        // Round pipeline: round r's (v, q) are located at the start of round
        // r - 1 (the query-position load, an L2 hit, overlaps a round), its
        // MATCH (the (slot, bid) groups) is issued at the end of round r - 1
        // and overlaps the next locate.
        // REGION: prep
        auto prep = [&](uint32_t k0, int v, int q, int &slot_o, int &lsv_o, bool &act_o) {
          bool act = k0 + uint32_t(lane) < Hn;
          if (seg) act = act && b + v - q >= dlo_f && b + v - q < dhi_f;
          int slot = base_slot + v - q;
          slot += slot < 0 ? M : 0;
          slot -= slot >= M ? M : 0;
          int lsv = lastsent;
          if (multi_bid_possible) lsv = __shfl_sync(kFull, ls_lane, v);
          const int bid = max(b, lsv + 1);  // record block (split at subject starts)
          slot_o = slot;
          lsv_o = lsv;
          act_o = act;
#ifdef BLK_FAKE_MATCH  // experiment only (wrong results): the cost of MATCH.ANY
          (void)bid;
          return (1u << lane) | (__shfl_xor_sync(kFull, slot, 1) == slot ? (1u << (lane ^ 1)) : 0u);
#else
          return __match_any_sync(
              kFull, act ? (unsigned(slot) | (unsigned(bid) << 14)) : 0xffffffffu);
#endif
        };
        int cv = 0, cq = 0, nv = 0, nq = 0, cslot = 0, clsv = 0;
        bool cact = false;
        locate(0u, Hn, cv, cq);
        unsigned cG = prep(0u, cv, cq, cslot, clsv, cact);
        if (32u < Hn) locate(32u, Hn, nv, nq);
        // REGION: round
        for (uint32_t k0 = 0; k0 < Hn; k0 += 32) {
          const int v = cv, q = cq, slot = cslot, lsv = clsv;
          const bool act = cact;
          const unsigned G = cG;
          const int P = b + v;
          const int bid = max(b, lsv + 1);  // record block (split at subject starts)
          uint32_t e = 0;
          if (act) e = w.ring()[slot];
#ifdef BLK_LAST3
          // The diagonal's three most recent hits p1 > p2 > p3 (p1 a frame
          // position, g1 = p1 - p2, g2 = p2 - p3; 255: none or farther than
          // A): the largest of them <= h - W, or an earlier member of h's
          // round group (its first, >= h - 31 >= h - A + 1), decides R6.
          const int lo_ok = max(P - A + 1, lsv + 1);  // within A, same subject
          const int hiP = P - W;
          const int Pf = __shfl_sync(kFull, P, __ffs(G) - 1);  // the group's first hit
          const int p1 = int(e & 0x3fffu), g1 = int((e >> 14) & 0xffu);
          int pq = p1;
          if (pq > hiP) {
            if (g1 == 255) {
              pq = 0;
            } else {
              pq -= g1;
              if (pq > hiP) {
                const int g2 = int(e >> 22);
                pq = g2 == 255 ? 0 : pq - g2;
              }
            }
          }
          const bool pass = act && ((pq >= lo_ok && pq <= hiP) || Pf <= hiP);
          unsigned Gw = G;
          if (multi_bid_possible && __any_sync(kFull, act && bid != b))
            Gw = __match_any_sync(kFull, act ? slot : -1);
          // the state write: the slot's last member, with its two
          // predecessors in the round (else the old state's)
          const bool wrl = act && lane == 31 - __clz(Gw);
          const int d1 = p1 ? min(P - p1, 255) : 255;
          if (__any_sync(kFull, act && (Gw & ltmask) != 0u)) {
            const unsigned bef = Gw & ltmask;
            const int j1 = bef ? 31 - __clz(bef) : lane;
            const unsigned bef2 = bef & ~(0xffffffffu << j1);
            const int j2 = bef2 ? 31 - __clz(bef2) : lane;
            const int x1 = __shfl_sync(kFull, P, j1), x2 = __shfl_sync(kFull, P, j2);
            if (wrl) {
              int n1 = d1, n2 = g1;
              if (bef2) {
                n1 = P - x1;
                n2 = x1 - x2;
              } else if (bef) {
                n1 = P - x1;
                n2 = p1 ? min(x1 - p1, 255) : 255;
              }
              w.ring()[slot] = uint32_t(P) | (uint32_t(n1) << 14) | (uint32_t(n2) << 22);
            }
          } else if (wrl) {
            w.ring()[slot] = uint32_t(P) | (uint32_t(d1) << 14) | (uint32_t(g1) << 22);
          }
#else
          const bool pre = v < L;
          const int lo_ok = max(P - A + 1, lsv + 1);  // within A, same subject
          const int Pf = __shfl_sync(kFull, P, __ffs(G) - 1);  // the group's first hit
          const int ebid = be_bid(e);
          const int emax = ebid + be_maxoff(e);
          const bool tst = act && (!pre || pre_ok);
          const int bt = pre ? max(b - 32, lsv + 1) : bid;  // the block h is tested against
          const bool same = ebid == bt;
          const int mn = same ? ebid + be_minoff(e) : (pre ? INT_MAX : Pf);
          const int po = be_prevoff(e);
          const int pv = same ? (po ? ebid - po : 0) : (ebid ? emax : 0);
          const bool pass = tst && (mn <= P - W || pv >= lo_ok);
          // the state write: the last member of the slot's group (of the
          // slot's last group when a subject starts inside the round)
          unsigned Gw = G;
          if (multi_bid_possible && __any_sync(kFull, act && bid != b))
            Gw = __match_any_sync(kFull, act ? slot : -1);
          if (act && lane == 31 - __clz(Gw)) {
            const bool sw = ebid == bid;
            const int dp = bid - emax;
            const uint32_t nmin = sw ? uint32_t(be_minoff(e)) : uint32_t(Pf - bid);
            const uint32_t npo =
                sw ? uint32_t(po) : ((ebid != 0 && dp <= 255) ? uint32_t(dp) : 0u);
            w.ring()[slot] =
                uint32_t(bid) | (nmin << 14) | (uint32_t(P - bid) << 19) | (npo << 24);
          }
#endif
          // every passing hit is queued: the flush's ext_reach chain (R10)
          // rejects the covered ones (0.5% of passing hits are covered by an
          // already resolved extension at this point on config 3; a reach
          // load per round costs more)
#ifdef BLK_ENQ_REACH  // A/B knob: skip passing hits already covered at enqueue
          const bool enq = pass && (kHit || P > int(w.reach()[slot]));
#else
          const bool enq = pass;
#endif
          if (kTrace) {
            bstat<kTrace>(st, kStatRounds, 1);
            bstat<kTrace>(st, kStatConflictRounds,
                          __any_sync(kFull, act && __popc(G) > 1) ? 1 : 0);
            bstat<kTrace>(st, kStatHits, __popc(__ballot_sync(kFull, act)));
            bstat<kTrace>(st, kStatPassing, __popc(__ballot_sync(kFull, pass)));
            bstat<kTrace>(st, kStatEnqueued, __popc(__ballot_sync(kFull, enq)));
            if (act) trace_push(a, 0, st.spbase + P, q, 0, 0, 0);
            if (pass) trace_push(a, 1, st.spbase + P, q, 0, 0, 0);
          }
          // the queue first (a flush here keeps only the next round's
          // (v, q) live across the X-drop), then the next round's MATCH and
          // the locate of the one after
          enqueue(enq, P, q);
          __syncwarp();
          if (k0 + 32u < Hn) {
            cv = nv;
            cq = nq;
            cG = prep(k0 + 32u, cv, cq, cslot, clsv, cact);
            if (k0 + 64u < Hn) locate(k0 + 64u, Hn, nv, nq);
          }
        }
      }
      // REGION: window
      // ---- advance the window ---------------------------------------------
      if (sm) lastsent = b + 31 - __clz(sm);
      b += 32;
      base_slot += 32;
      if (base_slot >= M) base_slot -= M;
    }
    while (st.qcount > 0)
      blk_flush<kTrace, kHit, kPssm>(a, w, st, min(st.qcount, 32), qc, b62, lane, slotc, M, pssm);
    // the next work item continues the frame after a gap (stale state ages out)
    frame = b + 64;
    base_slot = (base_slot + 64) % M;
  }
  if (kTrace && a.stats && lane == 0)
    for (int i = 0; i < kNumStats; ++i)
      if (st.stat[i]) atomicAdd(a.stats + i, st.stat[i]);
}

// REGION: host
size_t blk_smem_bytes(int lq, int ring, int warps, bool pssm_smem) {
  return kBlkTab + align16(size_t(lq) + 2 * kBlkQPad) +
         (pssm_smem ? align16(size_t(lq + 2 * kBlkQPad) * 32) : 0) +
         size_t(warps) * blk_area_bytes(ring);
}

// Warps per CTA: the most resident warps per SM (occupancy of this kernel
// instance at each CTA size up to warps_max whose shared memory fits),
// larger CTAs on ties.
template <bool kTrace, bool kDef, bool kHit, bool kPssm>
cudaError_t blk_launch(const SearchArgs &a, int warps_max, bool pssm_smem, int optin,
                       int num_sms, cudaStream_t s) {
  void (*k)(const SearchArgs) = search_block_kernel<kTrace, kDef, kHit, kPssm>;
  cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, optin);
  if (e != cudaSuccess) return e;
  int warps = 0, per_sm = 0;
  for (int w = warps_max; w >= 1; --w) {
    const size_t sm = blk_smem_bytes(a.qv.lq, a.ring, w, pssm_smem);
    if (sm > size_t(optin)) continue;
    int per = 0;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k, w * 32, sm);
    if (e != cudaSuccess) return e;
    if (per * w > per_sm * warps) {
      warps = w;
      per_sm = per;
    }
  }
  if (warps < 1 || per_sm < 1) return cudaErrorInvalidConfiguration;
  const size_t smem = blk_smem_bytes(a.qv.lq, a.ring, warps, pssm_smem);
  int64_t grid = int64_t(num_sms) * per_sm;
  const int64_t need = (int64_t(a.nchunks) + a.nlong + a.nsegs + warps - 1) / warps;
  if (grid > need) grid = need < 1 ? 1 : need;
  SearchArgs g = a;
  e = pool_malloc_async(reinterpret_cast<void **>(&g.reach_scratch),
                        size_t(grid) * warps * size_t(a.ring) * 2, s);
  if (e != cudaSuccess) return e;
  k<<<unsigned(grid), warps * 32, smem, s>>>(g);
  e = cudaGetLastError();
  cudaFreeAsync(g.reach_scratch, s);
  return e;
}

template <bool kTrace, bool kPssm>
cudaError_t blk_pick(const SearchArgs &a, int warps_max, bool pssm_smem, int optin, int num_sms,
                     cudaStream_t s) {
  const bool hit = a.ext_mode == BLASTP_EXT_HIT;
  if (a.min_gap == 3 && a.window == 40)
    return hit ? blk_launch<kTrace, true, true, kPssm>(a, warps_max, pssm_smem, optin, num_sms, s)
               : blk_launch<kTrace, true, false, kPssm>(a, warps_max, pssm_smem, optin, num_sms, s);
  return hit ? blk_launch<kTrace, false, true, kPssm>(a, warps_max, pssm_smem, optin, num_sms, s)
             : blk_launch<kTrace, false, false, kPssm>(a, warps_max, pssm_smem, optin, num_sms, s);
}

}  // namespace

bool block_kernel_eligible(const SearchArgs &a) {
  return a.filter_mode == BLASTP_FILTER_LEFT &&
         (a.ext_mode == BLASTP_EXT_DIAGONAL || a.ext_mode == BLASTP_EXT_HIT) &&
#ifdef BLK_LAST3
         a.min_gap >= 1 && a.min_gap <= 3 && a.window >= 32 && a.window <= 255 &&
#else
         a.min_gap >= 1 && a.min_gap <= 8 && a.window >= 31 + a.min_gap && a.window <= 256 &&
#endif
         a.qv.lq <= 16000 && a.qv.wtab != nullptr &&
         a.table_entries < (int64_t(1) << 27);  // the owner lookup's 27-bit offsets
}

cudaError_t launch_search_block(const SearchArgs &a_in, int num_sms, cudaStream_t s) {
  static unsigned long long b62_ready = 0;  // one bit per device
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if (!(b62_ready >> dev & 1ull)) {
    int8_t h[32 * 32];
    fill_b62(h);
    e = cudaMemcpyToSymbol(c_b62_blk, h, sizeof(h));
    if (e != cudaSuccess) return e;
    b62_ready |= 1ull << dev;
  }
  SearchArgs a = a_in;
  a.ring = search_ring_slots(a.qv.lq, a.window);
  a.pssm = nullptr;
  int optin = 0;
  e = cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  if (e != cudaSuccess) return e;
  // X-drop scores (perf only, identical results; paper E2, Fig. 15):
  // BLASTP_SCORE=pssm (PSSM in shared memory, fewer warps if it costs room),
  // pssm_global (PSSM in global memory, L1/L2), default: BLOSUM62 + query codes
  const char *score_env = std::getenv("BLASTP_SCORE");
  const bool pssm = score_env && !std::strncmp(score_env, "pssm", 4);
  const bool pssm_smem = pssm && std::strcmp(score_env, "pssm_global") != 0;
  const char *warps_env = std::getenv("BLASTP_WARPS");
  const int warps = warps_env ? std::max(1, std::min(kBlkWarps, std::atoi(warps_env))) : kBlkWarps;
  const bool trace = a.trace[0] != nullptr;
  if (!pssm)
    return trace ? blk_pick<true, false>(a, warps, false, optin, num_sms, s)
                 : blk_pick<false, false>(a, warps, false, optin, num_sms, s);
  int8_t *g = nullptr;
  if (!pssm_smem) {
    const size_t bytes = size_t(a.qv.lq + 2 * kBlkQPad) * 32;
    if ((e = pool_malloc_async(reinterpret_cast<void **>(&g), bytes, s)) != cudaSuccess) return e;
    pssm_fill_kernel<<<int((bytes + 255) / 256), 256, 0, s>>>(a.qv.qcodes, a.qv.lq, g);
    a.pssm = g;
  }
  e = trace ? blk_pick<true, true>(a, warps, pssm_smem, optin, num_sms, s)
            : blk_pick<false, true>(a, warps, pssm_smem, optin, num_sms, s);
  if (g) cudaFreeAsync(g, s);
  return e;
}

}  // namespace blastp
