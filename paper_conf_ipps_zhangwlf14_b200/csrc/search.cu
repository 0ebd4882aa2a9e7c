// search.cu -- "warp" variant of the fused BLASTP ungapped hot path (sm_100a).
//
// The general kernel: every filter reading (LEFT, EITHER, STATEFUL,
// STATEFUL_RB) and extension strategy (DIAGONAL, HIT, WINDOW), any window A;
// the block kernel (search_block.cu) replaces it for LEFT with A >= 31 + W.
// Each warp owns a chunk of whole subjects at a time (work-stealing over
// chunks) and walks it in ascending subject position:
//
//   hit detection     Alg. 2: a 32-lane window of consecutive
//                     word positions, one residue byte per lane per load
//                     (coalesced) plus two of overlap, prefetched
//                     two windows ahead; the lookup table (R3) is read through
//                     L1/L2, or from shared memory when it fits beside the
//                     rings without costing resident warps (P:L1702-1730
//                     hierarchical buffering).  Every window is 32 positions;
//                     its hits are processed in 32-hit rounds.
//   binning/sorting   P:L967-1343: replaced by a per-warp diagonal ring in
//                     shared memory indexed by (s - q) mod M.  Positions are
//                     visited in ascending s, so each diagonal's hits arrive
//                     in the order the paper's segmented sort establishes.
//                     Hits of one round on the same diagonal are grouped by
//                     __match_any_sync and ordered by lane (= s).
//   two-hit filter    P:L1344-1351 (R6): exists p on the same diagonal and
//                     subject with W <= h - p < A (ring state: last, far, near);
//                     Alg. 1's lasthit walk for STATEFUL (R15, R16).
//   extension         Alg. 3/5 + Fig. 8 (R7-R10): passing hits
//                     not covered by ext_reach are queued; 32 at a time are
//                     X-dropped lane-parallel and the ext_reach chain is
//                     resolved per diagonal in queue order.
//   output            P:L1352-1353: one global atomic per emitted HSP.
#include <cuda_runtime.h>

#include <algorithm>
#include <climits>
#include <cstdlib>
#include <cstring>

#include "search_common.cuh"

namespace blastp {

using namespace dev;

namespace {

constexpr int kMaxWarps = 32;   // warps per CTA (each independent)
constexpr int kQcap = 64;       // extension queue slots per warp
constexpr int kFrameMin = 1024;    // first frame position (> window + margin)
constexpr int kFrameSpan = 32768;  // rebase step

__constant__ int8_t c_b62[32 * 32];

// Ring slot two-hit state, 32 bits: bits 0..15 last hit, 16..23 last - far
// (0: none; a far hit more than 255 positions before `last` can never be
// within the window A <= 256 of a later hit), 24..31 near mask.  The
// ext_reach of the slot is a separate 16-bit array.
__device__ __forceinline__ uint32_t st_last(uint32_t e) { return e & 0xffffu; }
__device__ __forceinline__ uint32_t st_far(uint32_t e) {
  const uint32_t fd = (e >> 16) & 0xffu;
  return fd ? (e & 0xffffu) - fd : 0u;
}
__device__ __forceinline__ uint32_t st_near(uint32_t e) { return e >> 24; }
__device__ __forceinline__ uint32_t st_make(uint32_t last, uint32_t far, uint32_t near) {
  const uint32_t fd = (far != 0 && last - far <= 255u) ? last - far : 0u;
  return last | (fd << 16) | (near << 24);
}

// Per-warp shared-memory area: the fixed-size parts first, so that every
// address is the warp's base plus a constant (reach: plus a launch-uniform
// offset) -- one base register, no per-array pointers to keep or recompute.
//   [0, 256)     queue[kQcap]: P | q << 16 (the slot is recomputed at flush)
//   [256, 448)   flush scratch fs_p, fs_end, fs_acc [32] u16 (also the
//                owner-lookup scratch, 32 u32 over fs_p/fs_end)
//   [448, 480)   wk[8]: walker state: item, segment, entry, slot offset;
//                [4] segment being filtered (-1: none), [5] its list length
//   [480, ...)   ring[M] two-hit state, then reach[M] ext_reach (16-bit)
constexpr int kRingOff = 480;
struct WarpSmem {
  uint8_t *base;
  int reach_off;  // kRingOff + align16(4 M)
  __device__ __forceinline__ uint32_t *queue() const { return reinterpret_cast<uint32_t *>(base); }
  __device__ __forceinline__ uint16_t *fs_p() const { return reinterpret_cast<uint16_t *>(base + 256); }
  __device__ __forceinline__ uint16_t *fs_end() const { return fs_p() + 32; }
  __device__ __forceinline__ uint16_t *fs_acc() const { return fs_p() + 64; }
  __device__ __forceinline__ int *wk() const { return reinterpret_cast<int *>(base + 448); }
  __device__ __forceinline__ uint32_t *ring() const {
    return reinterpret_cast<uint32_t *>(base + kRingOff);
  }
  __device__ __forceinline__ uint16_t *reach() const {
    return reinterpret_cast<uint16_t *>(base + reach_off);
  }
};

// Per-warp shared memory: 6 B per diagonal slot + 480 B; small enough for
// 30+ resident warps per SM at Lq ~ 1000 (occupancy is what this latency-
// bound kernel runs on, profiles/r01).
__host__ __device__ size_t warp_smem_bytes(int ring) {
  return kRingOff + align16(size_t(ring) * 4) + align16(size_t(ring) * 2);
}

__device__ __forceinline__ WarpSmem carve(uint8_t *base, int ring) {
  WarpSmem w;
  w.base = base;
  w.reach_off = kRingOff + int(align16(size_t(ring) * 4));
  return w;
}

struct WarpState {
  int64_t spbase;  // stream position of frame position 0
  int64_t first_subj, last_subj;
  int qhead, qcount;
  unsigned long long stat[kNumStats];  // tracing variant only
};

template <bool kStats>
__device__ __forceinline__ void stat_add(WarpState &st, int i, unsigned long long v) {
  if (kStats) st.stat[i] += v;
}

// One direction of the window-based X-drop (Alg. 5 / Fig. 8):
// the warp scores 32 consecutive positions of the diagonal at a time, lane i
// the position t0 + i (step +1 right from (q0, s0), -1 left), then forms the
// PrefixSum (inclusive scan seeded with the running sum), the running best
// (inclusive max scan seeded with the best so far) and the DropFlag
// (best - prefix >= X); the first flagged lane stops the scan.  The best is
// the largest prefix at or before the stop, its length the first lane that
// reaches it (strict >, R8).  Returns (best, length); warp-uniform.
__device__ __forceinline__ void window_xdrop(const uint8_t *__restrict__ stream, int64_t s0,
                                             const uint8_t *qq, int q0, int step,
                                             const int8_t *b62, int X, int lane, int &best_out,
                                             int &len_out) {
  int run = 0, best = 0, blen = 0;
  for (int t0 = 0;; t0 += 32) {
    const int t = t0 + lane;
    const int64_t sp = s0 + int64_t(step) * t;
    const int qi = q0 + step * t;
    // lanes past a sentinel (sequence end) read clamped addresses: the scan
    // stops at the sentinel, so their values are never used
    const uint32_t sc = __ldg(stream + (sp < 0 ? 0 : sp));
    const uint32_t qcv = qq[qi < -kQPad ? -kQPad : qi];
    int P = score(b62, qcv, sc);
    if (lane == 0) P += run;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const int v = __shfl_up_sync(kFull, P, d);
      if (lane >= d) P += v;
    }
    int Mx = max(P, best);
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const int v = __shfl_up_sync(kFull, Mx, d);
      if (lane >= d) Mx = max(Mx, v);
    }
    const unsigned drop = __ballot_sync(kFull, Mx - P >= X);
    const int stop = drop ? __ffs(drop) - 1 : 31;  // last lane that counts
    const int mx = __shfl_sync(kFull, Mx, stop);
    if (mx > best) {
      const unsigned at = __ballot_sync(kFull, lane <= stop && P == mx);
      blen = t0 + __ffs(at);
      best = mx;
    }
    if (drop) break;
    run = __shfl_sync(kFull, P, 31);
  }
  best_out = best;
  len_out = blen;
}

// Alg. 5 (ext_mode WINDOW): the queued passing hits in queue (= s) order, one
// at a time; a hit covered by its diagonal's ext_reach is skipped before any
// work (Alg. 3 L19), otherwise the warp extends it with window_xdrop in both
// directions and sets ext_reach = the HSP's subject end (R10).
template <bool kTrace>
__device__ void flush_queue_window(const SearchArgs &a, const WarpSmem &w, WarpState &st, int n,
                                   const uint8_t *qc, const int8_t *b62, int lane, int slotc,
                                   int M) {
  const uint8_t *qq = qc + kQPad;
  for (int j = 0; j < n; ++j) {
    const uint32_t ent = w.queue()[(st.qhead + j) & (kQcap - 1)];
    const int P = int(ent & 0xffffu), q = int(ent >> 16);
    int slot = (P - q + slotc) % M;
    slot += slot < 0 ? M : 0;
    if (P <= int(w.reach()[slot])) continue;  // covered (warp-uniform)
    const int64_t sp = st.spbase + P;
    const int seed = score(b62, qq[q], __ldg(a.stream + sp)) +
                     score(b62, qq[q + 1], __ldg(a.stream + sp + 1)) +
                     score(b62, qq[q + 2], __ldg(a.stream + sp + 2));
    int br, rlen, bl, llen;
    window_xdrop(a.stream, sp + 3, qq, q + 3, 1, b62, a.xdrop, lane, br, rlen);
    window_xdrop(a.stream, sp - 1, qq, q - 1, -1, b62, a.xdrop, lane, bl, llen);
    const int total = seed + br + bl;
    __syncwarp();
    if (lane == 0) w.reach()[slot] = uint16_t(min(P + 2 + rlen, 0xffff));
    __syncwarp();
    if (kTrace) {
      stat_add<kTrace>(st, kStatExtended, 1);
      stat_add<kTrace>(st, kStatAccepted, 1);
      stat_add<kTrace>(st, kStatEmitted, total >= a.cutoff ? 1 : 0);
    }
    if (lane == 0) {
      if (kTrace) trace_push(a, 2, sp, q, llen, rlen, total);
      emit_hsp(a, sp, q, llen, rlen, total, st.first_subj, st.last_subj);
    }
  }
  __syncwarp();
  st.qhead = (st.qhead + n) & (kQcap - 1);
  st.qcount -= n;
}

// Extend up to 32 queued passing hits lane-parallel, then resolve the
// ext_reach chain (Alg. 3 L19-23, R10) per diagonal in queue (= s) order.
// Speculation (extending entries the chain may then reject, 22% of them on
// config 3) is cheaper than extending only each diagonal's first uncovered
// entry and keeping the rest queued: +8.7% per config-3 step measured
// (profiles/r01/ab_flush_defer_rejected.txt).
// kWin: ext_mode WINDOW, a kernel instantiation of its own (the window scan
// inlined into the default kernel cost it 15% through register allocation).
// kSt: filter mode STATEFUL (Alg. 1 L8-19, R15): the queued entries' walk
// is finished here (see the round code in search_warp_kernel).
template <bool kTrace, bool kWin, int kSt>
__device__ void flush_queue(const SearchArgs &a, const WarpSmem &w, WarpState &st, int n,
                            const uint8_t *qc, const int8_t *b62, int lane, int slotc, int M) {
  if constexpr (kWin) {
    flush_queue_window<kTrace>(a, w, st, n, qc, b62, lane, slotc, M);
    return;
  }
  const bool act = lane < n;
  uint32_t ent = 0;
  if (act) ent = w.queue()[(st.qhead + lane) & (kQcap - 1)];
  const int P = int(ent & 0xffffu);
  const int q = kSt ? int((ent >> 16) & 0x3fffu) : int(ent >> 16);
  // ring slot of the diagonal: (base_slot - win) + P - q (mod M), slotc given
  int slot = (P - q + slotc) % M;
  slot += slot < 0 ? M : 0;
  const int64_t sp = st.spbase + P;
  int total = 0, llen = 0, rlen = 0, scanned = 0;
  if (act) xdrop_extend(a.stream, sp, q, qc, b62, a.xdrop, total, llen, rlen, scanned);
  if (kTrace) {
    stat_add<kTrace>(st, kStatFlushes, 1);
    stat_add<kTrace>(st, kStatExtended, n);
    stat_add<kTrace>(st, kStatXdropSteps, __reduce_add_sync(kFull, unsigned(scanned)));
    stat_add<kTrace>(st, kStatXdropLaneSlots, 32ull * __reduce_max_sync(kFull, unsigned(scanned)));
  }
  const int endp = min(P + 2 + rlen, 0xffff);  // HSP subject end (inclusive), frame
  bool acc = false;
  uint16_t *reach16 = w.reach() + slot;
  if constexpr (kSt) {
    // Finish Alg. 1's walk over the flushed entries of each diagonal, in
    // queue (= s) order, from the slot's lasthit: a trigger (bit 31) was
    // decided at enqueue; a fresh entry (bit 30) starts a new subject (no
    // lasthit); any other entry applies L11-19 to the lasthit the walk has
    // reached.  An accepted extension sets lasthit = its subject end.
    const unsigned grp = __match_any_sync(kFull, act ? slot : -1);
    const uint32_t e = act ? w.ring()[slot] : 0u;
    uint32_t cur = e & 0xffffu;
    const int gmax = __reduce_max_sync(kFull, act ? __popc(grp) : 0);
    const uint32_t fl = ent >> 30;
    const int sst = P - llen;  // the extension's subject start (frame), for R16
    unsigned rem = act ? grp : 0u;
    for (int it = 0; it < gmax; ++it) {
      const int src = rem ? __ffs(rem) - 1 : lane;
      const bool valid = rem != 0;
      rem &= rem - 1;
      const int Pj = __shfl_sync(kFull, P, src);
      const int Ej = __shfl_sync(kFull, endp, src);
      const uint32_t fj = __shfl_sync(kFull, fl, src);
      const int Sj = kSt == 2 ? __shfl_sync(kFull, sst, src) : 0;
      if (valid) {
        bool aj;
        if (fj & 2u) {
          aj = true;
        } else {
          if (fj & 1u) cur = 0;
          const int d = Pj - int(cur);
          aj = false;
          if (cur == 0 || d >= a.window) cur = uint32_t(Pj);
          else if (d >= a.min_gap) aj = true;
        }
        // R16 (filter_mode STATEFUL_RB, Alg. 1 L13 ungapped_ext(hit, lasthit)):
        // an extension not reaching back to the lasthit is dropped and the hit
        // becomes the lasthit (L19)
        if (kSt == 2 && aj && Sj > int(cur)) {
          aj = false;
          cur = uint32_t(Pj);
        }
        if (aj) cur = uint32_t(Ej);
        if (src == lane) acc = aj;
      }
    }
    __syncwarp();
    if (act && (grp >> lane) == 1u) w.ring()[slot] = cur | (((e >> 16) - __popc(grp)) << 16);
    __syncwarp();
    if (kTrace) {
      stat_add<kTrace>(st, kStatPassing, __popc(__ballot_sync(kFull, acc)));
      if (acc) trace_push(a, 1, sp, q, 0, 0, 0);
    }
  } else if (a.ext_mode == BLASTP_EXT_HIT) {
    // Alg. 4: every passing hit is extended and kept; ext_reach
    // is never written, so every passing hit was also queued
    acc = act;
  } else if (const unsigned grp = __match_any_sync(kFull, act ? slot : -1),
             uniq = (grp == (1u << lane));
             __all_sync(kFull, uniq || !act)) {
    if (act) {
      acc = P > int(*reach16);
      if (acc) *reach16 = uint16_t(endp);
    }
  } else {
    w.fs_p()[lane] = uint16_t(P);
    w.fs_end()[lane] = uint16_t(endp);
    __syncwarp();
    if (act) {
      if (uniq) {
        acc = P > int(*reach16);
        if (acc) *reach16 = uint16_t(endp);
      } else if (lane == __ffs(grp) - 1) {
        int r = *reach16;
        unsigned g = grp;
        while (g) {
          const int j = __ffs(g) - 1;
          g &= g - 1;
          const bool aj = int(w.fs_p()[j]) > r;
          if (aj) r = w.fs_end()[j];
          w.fs_acc()[j] = aj;
        }
        *reach16 = uint16_t(r);
      }
    }
    __syncwarp();
    if (act && !uniq) acc = w.fs_acc()[lane] != 0;
  }
  if (kTrace) {
    stat_add<kTrace>(st, kStatAccepted, __popc(__ballot_sync(kFull, acc)));
    stat_add<kTrace>(st, kStatEmitted, __popc(__ballot_sync(kFull, acc && total >= a.cutoff)));
  }
  if (acc) {
    if (kTrace) trace_push(a, 2, sp, q, llen, rlen, total);
    emit_hsp(a, sp, q, llen, rlen, total, st.first_subj, st.last_subj);
  }
  __syncwarp();
  st.qhead = (st.qhead + n) & (kQcap - 1);
  st.qcount -= n;
}

// kF: filter mode, BLASTP_FILTER_LEFT / _EITHER / _STATEFUL;
// OffT: uint16_t (table in shared memory) or uint32_t (table in global memory);
// kW: min_gap fixed at compile time (3, the default) or 0 (runtime value).
template <bool kTrace, int kF, typename OffT, int kW, bool kWin>
__global__ void __launch_bounds__(kMaxWarps * 32) search_warp_kernel(const SearchArgs a) {
  constexpr bool kEither = kF == BLASTP_FILTER_EITHER;
  // 1: STATEFUL (R15); 2: STATEFUL_RB (R15 + R16's reach-back)
  constexpr int kSt = kF == BLASTP_FILTER_STATEFUL ? 1 : kF == BLASTP_FILTER_STATEFUL_RB ? 2 : 0;
  extern __shared__ __align__(16) uint8_t smem[];
  const int lq = a.qv.lq;
  int8_t *b62 = reinterpret_cast<int8_t *>(smem);
  uint8_t *qc = smem + 1024;
  const size_t qc_bytes = align16(size_t(lq) + 2 * kQPad + 8);
  uint8_t *after_qc = qc + qc_bytes;
  const OffT *woff;
  const uint16_t *qpos;
  size_t table_bytes = 0;
  if constexpr (sizeof(OffT) == 2) {
    // Hierarchical buffering: the whole lookup table in smem.
    uint16_t *woff_s = reinterpret_cast<uint16_t *>(after_qc);
    const int nw = kWords + 1;
    uint16_t *qpos_s = woff_s + ((nw + 7) & ~7);
    const uint32_t entries = uint32_t(a.table_entries);
    for (int i = threadIdx.x; i < nw; i += blockDim.x) woff_s[i] = uint16_t(__ldg(a.qv.woff + i));
    for (uint32_t i = threadIdx.x; i < entries; i += blockDim.x) qpos_s[i] = __ldg(a.qv.qpos + i);
    woff = reinterpret_cast<const OffT *>(woff_s);
    qpos = qpos_s;
    table_bytes = align16(size_t((nw + 7) & ~7) * 2 + size_t(entries) * 2);
  } else {
    woff = reinterpret_cast<const OffT *>(a.qv.woff);
    qpos = a.qv.qpos;
  }
  for (int i = threadIdx.x; i < 1024; i += blockDim.x) b62[i] = c_b62[i];
  for (int i = threadIdx.x; i < int(qc_bytes); i += blockDim.x) {
    const int k = i - kQPad;
    qc[i] = (k >= 0 && k < lq) ? a.qv.qcodes[k] : uint8_t(kSentinel);
  }
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int M = a.ring;
  WarpSmem w = carve(after_qc + table_bytes + size_t(warp) * warp_smem_bytes(M), M);
  for (int i = lane; i < M; i += 32) {
    w.ring()[i] = 0;
    w.reach()[i] = 0;
  }
  __syncthreads();

  const uint8_t *__restrict__ stream = a.stream;
  const int W = kW ? kW : a.min_gap, A = a.window;  // kW: compile-time min_gap
  const uint32_t nearmask = (1u << W) - 2u;  // bits 1 .. W-1
  const int warm = (A + 31) & ~31;           // segment warm-up, whole windows

  WarpState st;
  if (kTrace)
    for (int i = 0; i < kNumStats; ++i) st.stat[i] = 0;
  st.qhead = 0;
  st.qcount = 0;
  int frame = kFrameMin;  // frame position of the next chunk's first residue
  int base_slot = 0;      // ring slot of diagonal (win - q + const) at q = lane = 0
  // subtract kFrameSpan from every stored frame position (0 = none stays 0)
  auto rebase_ring = [&]() {
    for (int i = lane; i < M; i += 32) {
      const uint32_t e = w.ring()[i];
      auto rb = [](uint32_t v) { return v > uint32_t(kFrameSpan) ? v - kFrameSpan : 0u; };
      const uint32_t nl = rb(st_last(e));
      w.ring()[i] = nl ? st_make(nl, rb(st_far(e)), st_near(e)) : 0u;
      w.reach()[i] = uint16_t(rb(w.reach()[i]));
    }
    __syncwarp();
    st.spbase += kFrameSpan;
  };
  const unsigned long long nsegs = (unsigned long long)a.nsegs;
  const unsigned long long nitems = nsegs + (unsigned long long)a.nlong;
  // Work items: segments (walk, queue spilled to a list), long items (walker, or a plain
  // walk), regular chunks (walk).  Every queue drain outside the hot round
  // loop happens at the single site at the bottom of this loop, so the
  // X-drop code exists in three copies only (instruction-cache footprint);
  // the walker therefore runs in steps that end whenever the queue must be
  // drained, its state parked in shared memory (w.wk()), not in registers.
  int mode = 0;  // 0: take the next work item; 1: a walker is active
  for (;;) {
    int64_t wstart = 0, wend = 0, wemit = 0;
    int64_t dlo = INT64_MIN, dhi = INT64_MAX;  // STATEFUL segment: its diagonals
    bool walk = false;
    bool retrace = false;  // fallback walk: its hits were traced by the segments
    int sg = -1;
    int sc = 0;  // slot offset of the queued entries, for the drain below
    if (mode == 0) {
      unsigned long long ci = 0;
      if (lane == 0) ci = atomicAdd(a.chunk_cursor, 1ull);
      ci = __shfl_sync(kFull, ci, 0);
      // a walk covers stream positions [wstart, wend); hits before wemit
      // only warm the two-hit state (segments); a segment's queue is
      // spilled to its list instead of being extended
      if (ci < nsegs) {
        sg = int(ci);
        const LongItem &it = a.long_items[a.seg_item[sg]];
        if constexpr (kSt) {
          // STATEFUL: segment j owns the diagonals (stream position - q) in
          // [dlo, dhi); every hit of such a diagonal lies in [dlo, dhi + lq),
          // so the segment walks that range, keeps the hits of its own
          // diagonals and holds each diagonal's whole lasthit walk (R15)
          // (segment 0 also owns the diagonals below the chunk start: hits
          // at its first positions with large q)
          const int j = sg - it.seg0;
          const int64_t d0 = it.c.start + int64_t(j) * a.seg_len;
          dlo = j == 0 ? INT64_MIN : d0;
          dhi = j == it.nseg - 1 ? INT64_MAX : d0 + a.seg_len;
          wstart = wemit = d0;
          wend = j == it.nseg - 1 ? it.c.end : min(it.c.end, d0 + a.seg_len + lq);
          sg = -1;  // extends and emits itself (no list, no walker)
        } else {
          wemit = it.c.start + int64_t(sg - it.seg0) * a.seg_len;
          wend = min(it.c.end, wemit + a.seg_len);
          // R6 looks back < A positions: a warm-up of A rounded up to whole
          // windows (seg_len >= 256 >= A keeps it inside the chunk)
          wstart = sg == it.seg0 ? it.c.start : wemit - warm;
        }
        st.first_subj = it.c.first_subj;
        st.last_subj = it.c.last_subj;
        walk = true;
      } else if (ci < nitems) {
        const LongItem it = a.long_items[ci - nsegs];
        st.first_subj = it.c.first_subj;
        st.last_subj = it.c.last_subj;
        if (kSt && it.nseg > 0) continue;  // covered by its diagonal segments
        if (it.nseg > 0 && !kSt) {
          st.spbase = it.c.start - frame;
          if (lane == 0) {
            w.wk()[0] = int(ci - nsegs);
            w.wk()[1] = 0;
            w.wk()[2] = 0;
            w.wk()[3] = ((base_slot - frame) % M + M) % M;  // slot = P - q + offset
          }
          __syncwarp();
          mode = 1;
        } else {
          wstart = wemit = it.c.start;
          wend = it.c.end;
          walk = true;
        }
      } else {
        const unsigned long long cj = ci - nitems;
        if (cj >= (unsigned long long)a.nchunks) break;
        const Chunk ch = a.chunks[cj];
        st.first_subj = ch.first_subj;
        st.last_subj = ch.last_subj;
        wstart = wemit = ch.start;
        wend = ch.end;
        walk = true;
      }
    }
    if (!kSt && mode == 1) {
      // ---- walker step: the segments' passing hits, in s order, into the
      // extension queue (the ext_reach chain resolves at the drain, exactly
      // as in a walk); returns whenever the queue must be drained first
      const LongItem it = a.long_items[__shfl_sync(kFull, w.wk()[0], 0)];
      int k = __shfl_sync(kFull, w.wk()[1], 0), i0 = __shfl_sync(kFull, w.wk()[2], 0),
          slotw = __shfl_sync(kFull, w.wk()[3], 0);
      // a rebase lowers every frame position by kFrameSpan: the slot offset
      // rises by as much, so each diagonal keeps its slot
      auto rebase_w = [&]() {
        rebase_ring();
        slotw = (slotw + kFrameSpan) % M;
      };
      for (;;) {
        if (k == it.nseg) {
          if (st.qcount > 0) break;
          while (it.c.end - st.spbase >= kFrameMin + kFrameSpan) rebase_w();
          frame = int(it.c.end - st.spbase) + 64;
          base_slot = (frame + slotw) % M;
          mode = 0;
          break;
        }
        const int sgk = it.seg0 + k;
        const int64_t emit = it.c.start + int64_t(k) * a.seg_len;
        // wait (warp-uniformly) for the segment's list to be published
        while (__shfl_sync(kFull, ld_acquire(a.seg_done + sgk), 0) != a.seq) __nanosleep(256);
        // values that steer control flow are broadcast from lane 0: the
        // compiler then knows they are warp-uniform (volatile loads are not)
        const int n = __shfl_sync(kFull, *(volatile const int32_t *)(a.seg_count + sgk), 0);
        if (n < 0) {
          // the list overflowed: walk the rest of the chunk directly,
          // continuing this frame and ext_reach state
          if (st.qcount > 0) break;
          wstart = k == 0 ? it.c.start : emit - warm;
          wemit = emit;
          wend = it.c.end;
          while (wstart - st.spbase >= kFrameMin + kFrameSpan) rebase_w();
          frame = int(wstart - st.spbase);
          base_slot = (frame + slotw) % M;
          walk = true;
          retrace = true;
          mode = 0;
          break;
        }
        if (i0 >= n) {
          ++k;
          i0 = 0;
          continue;
        }
        const volatile uint32_t *L = a.seg_list + int64_t(sgk) * a.seg_cap;
        const uint32_t e0 = __shfl_sync(kFull, lane == 0 ? L[i0] : 0u, 0);
        if (emit + int64_t(e0 & 0xffffu) - st.spbase >= kFrameMin + kFrameSpan) {
          if (st.qcount > 0) break;
          rebase_w();
          continue;
        }
        const int i = i0 + lane;
        const uint32_t e = i < n ? L[i] : 0u;
        const int64_t P64 = emit + int64_t(e & 0xffffu) - st.spbase;
        const bool act = i < n && P64 < kFrameMin + kFrameSpan + 32;  // a prefix
        const int P = int(P64), q = int(e >> 16);
        uint32_t rch = 0;
        if (act) {
          int slot = (P - q + slotw) % M;
          slot += slot < 0 ? M : 0;
          rch = w.reach()[slot];
        }
        const bool enq = act && P > int(rch);
        const unsigned bal = __ballot_sync(kFull, enq);
        stat_add<kTrace>(st, kStatEnqueued, __popc(bal));
        const int pos = st.qcount + __popc(bal & lanemask_lt(lane));
        if (enq) w.queue()[(st.qhead + pos) & (kQcap - 1)] = uint32_t(P) | (uint32_t(q) << 16);
        st.qcount += __popc(bal);
        i0 += __popc(__ballot_sync(kFull, act));
        if (st.qcount >= 32) break;
      }
      __syncwarp();
      if (lane == 0) {
        w.wk()[1] = k;
        w.wk()[2] = i0;
        w.wk()[3] = slotw;
      }
      __syncwarp();
      sc = slotw;
    }
    if (walk) {
    __syncwarp();
    if (lane == 0) {
      w.wk()[4] = sg;
      w.wk()[5] = 0;
    }
    __syncwarp();
    st.spbase = wstart - frame;
    // frame-relative diagonal range (P - q) of a STATEFUL segment
    int dlo_f = INT_MIN, dhi_f = INT_MAX;
    if (kSt && dlo != INT64_MIN) dlo_f = int(dlo - st.spbase);
    if (kSt && dhi != INT64_MAX) dhi_f = int(dhi - st.spbase);
    int win = frame;                           // frame position of lane 0 of the window
    int lastsent = frame - 1;                  // the sentinel before the chunk
    int64_t end = wend - st.spbase;            // frame position of the chunk end (exclusive)
    int emit_f = int(wemit - st.spbase);       // first frame position whose hits count
    // Segment: move n queued entries to the segment's list as (s - emit) |
    // q << 16 (passing hits in s order; ext_reach holds only stale values
    // older than the frame there, so every passing hit was queued)
    auto spill = [&](int n) {
      const int sgw = __shfl_sync(kFull, w.wk()[4], 0);
      const int nl = __shfl_sync(kFull, w.wk()[5], 0);
      if (lane < n && nl + lane < a.seg_cap) {
        const uint32_t ent = w.queue()[(st.qhead + lane) & (kQcap - 1)];
        a.seg_list[int64_t(sgw) * a.seg_cap + nl + lane] =
            ((ent & 0xffffu) - uint32_t(emit_f)) | (ent & 0xffff0000u);
      }
      __syncwarp();
      if (lane == 0) w.wk()[5] = nl + n;
      __syncwarp();
      st.qhead = (st.qhead + n) & (kQcap - 1);
      st.qcount -= n;
    };
    // Software pipeline over windows: residues are loaded two windows ahead
    // (one coalesced byte per lane + 2 bytes of overlap), the table lookup is
    // issued one window ahead and consumed by the next iteration.
    uint32_t pf_r = 0, pf_x = 0;  // residues of the window after the next
    auto load_res = [&](int wn) {
      const int64_t pp = st.spbase + wn;
      pf_r = __ldg(stream + pp + lane);
      pf_x = lane < 2 ? __ldg(stream + pp + 32 + lane) : 0u;
    };
    uint32_t nx_r0 = 0, nx_o = 0, nx_c = 0;
    auto lookup = [&](int wn) {  // consumes pf_* (residues of window wn)
      const uint32_t r0 = pf_r;
      uint32_t r1 = __shfl_down_sync(kFull, pf_r, 1), r2 = __shfl_down_sync(kFull, pf_r, 2);
      const uint32_t x0 = __shfl_sync(kFull, pf_x, 0), x1 = __shfl_sync(kFull, pf_x, 1);
      if (lane == 31) { r1 = x0; r2 = x1; }
      if (lane == 30) r2 = x0;
      load_res(wn + 32);
      const bool ok = (wn + lane < end) && (max(r0, max(r1, r2)) < uint32_t(kNumLetters));
      nx_r0 = (wn + lane < end) ? r0 : 0u;
      nx_o = 0;
      nx_c = 0;
      if (ok) {
        const uint32_t c = (r0 * kNumLetters + r1) * kNumLetters + r2;
        nx_o = woff[c];
        nx_c = woff[c + 1];
      }
    };
    load_res(win);
    lookup(win);
    auto slotc = [&]() {  // (base_slot - win) mod M: ring slot of (P, q) = P - q + slotc
      int c = (base_slot - win) % M;
      return c < 0 ? c + M : c;
    };

    while (win < end) {
      // ---- rebase the frame before positions outgrow 16 bits --------------
      if (win >= kFrameMin + kFrameSpan) {
        if (__shfl_sync(kFull, w.wk()[4], 0) >= 0) {
          while (st.qcount > 0) spill(min(st.qcount, 32));
        } else {
          const int sc = slotc();
          while (st.qcount > 0)
            flush_queue<kTrace, kWin, kSt>(a, w, st, min(st.qcount, 32), qc, b62, lane, sc, M);
        }
        rebase_ring();
        win -= kFrameSpan;
        lastsent -= kFrameSpan;
        if (kSt && dlo_f != INT_MIN) dlo_f -= kFrameSpan;
        if (kSt && dhi_f != INT_MAX) dhi_f -= kFrameSpan;
        end -= kFrameSpan;
        emit_f -= kFrameSpan;
      }
      stat_add<kTrace>(st, kStatIterations, 1);
      // ---- this window's lookup (issued last iteration); issue the next ---
      const uint32_t o = nx_o, cnt = nx_c - nx_o;
      const unsigned sm = __ballot_sync(kFull, nx_r0 == uint32_t(kSentinel));
      lookup(win + 32);
      uint32_t incl = cnt;
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) {
        const uint32_t t = __shfl_up_sync(kFull, incl, d);
        if (lane >= d) incl += t;
      }
      const uint32_t excl = incl - cnt;
      // all 32 positions are consumed; their hits are processed in 32-hit
      // rounds in lane-major (= s) order.  Hits of one diagonal in different
      // rounds see each other through the ring (rounds are sequential).
      const int npos = 32;
      const uint32_t Hn = __shfl_sync(kFull, incl, 31);
      // last sentinel at or before each lane (before `win`: lastsent)
      const unsigned prior = sm & ((lane == 31) ? kFull : ((2u << lane) - 1u));
      int ls_lane = prior ? (win + 31 - __clz(prior)) : lastsent;
      // a segment's warm-up windows (emit_f is window-aligned): a sentinel
      // "after" every hit makes R6's lower bound unreachable, so no hit passes
      if (win < emit_f) ls_lane = INT_MAX - 1;

      // round r's owner lane and query position are computed (and the query
      // position load issued) one round ahead of its processing
      // Owner lane and query position of hit kb + lane, through a 32-entry
      // per-warp scratch (the flush scratch; free here): each lane whose run
      // of hits intersects [kb, kb + 32) stores (lane, table offset - excl)
      // at the slot of its run's first hit in the round; a hit's owner is the
      // last run start at or before it, from the OR-reduced start mask
      // (measured: 1.1% faster than a 5-step shuffle binary search over the
      // inclusive counts, profiles/r01/ab_locate.txt)
      uint32_t *scr = reinterpret_cast<uint32_t *>(w.fs_p());
      auto locate = [&](uint32_t kb, int &own_out, int &q_out) {
        const bool wr = cnt != 0u && excl < kb + 32u && incl > kb;
        const int p0 = wr ? max(int(excl) - int(kb), 0) : 0;
        if (wr) scr[p0] = uint32_t(lane) | ((o - excl) << 5);
        const unsigned S = __reduce_or_sync(kFull, wr ? (1u << p0) : 0u);
        __syncwarp();
        const int src = 31 - __clz(S & (kFull >> (31 - lane)));
        const uint32_t v = scr[src];
        own_out = int(v & 31u);
        const uint32_t k = kb + uint32_t(lane);
        q_out = k < Hn ? int(qpos[((v >> 5) + k) & 0x7ffffffu]) : 0;
        __syncwarp();
      };
      int nown = 0, nq = 0;
      if (Hn) locate(0u, nown, nq);
      for (uint32_t k0 = 0; k0 < Hn; k0 += 32) {
        const uint32_t k = k0 + uint32_t(lane);
        const int own = nown;
        int q = nq;
        bool act = k < Hn;
        if constexpr (kSt) act = act && win + own - q >= dlo_f && win + own - q < dhi_f;
        if (k0 + 32 < Hn) locate(k0 + 32u, nown, nq);
        const int ls = __shfl_sync(kFull, ls_lane, own);
        int slot = 0;
        const int Ph = win + own;
        if (act) {
          slot = base_slot + own - q;
          slot += (slot < 0) ? M : 0;
          slot -= (slot >= M) ? M : 0;
        }
        const unsigned grp = __match_any_sync(kFull, act ? slot : -1);
        const unsigned earlier = grp & lanemask_lt(lane);
        uint32_t e = 0, rch = 0;
        if (act) {
          e = w.ring()[slot];
          rch = w.reach()[slot];
        }
        bool enq = false;
        uint32_t eflags = 0;  // STATEFUL queue-entry flags (bit 31 trigger, bit 30 fresh)
        if constexpr (kSt) {
          // Alg. 1 L8-19 (R15) at enqueue time.  Slot state: lasthit L (0:
          // none) | count of queued, unresolved entries << 16; reach[] = the
          // position of the last queued entry.  While entries are queued the
          // lasthit depends on their extensions: later hits are queued too
          // (conditional) and the walk finishes at the flush, in queue order.
          // Members of a round group replay the group's walk in lane (= s)
          // order; each keeps its own decision.
          uint32_t L = e & 0xffffu, cnt = e >> 16, rq = rch;
          const int gmax = __reduce_max_sync(kFull, act ? __popc(grp) : 0);
          unsigned rem = act ? grp : 0u;
          for (int it = 0; it < gmax; ++it) {
            const int src = rem ? __ffs(rem) - 1 : lane;
            const bool valid = rem != 0;
            rem &= rem - 1;
            const int Pj = __shfl_sync(kFull, Ph, src);
            const int lsj = __shfl_sync(kFull, ls, src);
            if (valid) {
              bool ej = false;
              uint32_t fj = 0;
              if (cnt > 0) {
                ej = true;
                fj = int(rq) <= lsj ? (1u << 30) : 0u;  // pending entries of an earlier subject
                ++cnt;
                rq = uint32_t(Pj);
              } else {
                const int d = Pj - int(L);
                if (L == 0 || int(L) <= lsj || d >= A) {
                  L = uint32_t(Pj);  // L17-19
                } else if (d >= W) {  // L11-14: extend (lasthit from the flush)
                  ej = true;
                  fj = 1u << 31;
                  cnt = 1;
                  rq = uint32_t(Pj);
                }
              }
              if (src == lane) {
                enq = ej;
                eflags = fj;
              }
            }
          }
          if (kTrace) {
            stat_add<kTrace>(st, kStatRounds, 1);
            stat_add<kTrace>(st, kStatHits, __popc(__ballot_sync(kFull, act)));
            stat_add<kTrace>(st, kStatEnqueued, __popc(__ballot_sync(kFull, enq)));
            if (act) trace_push(a, 0, st.spbase + Ph, q, 0, 0, 0);
          }
          __syncwarp();
          if (act && (grp >> lane) == 1u) {
            w.ring()[slot] = L | (cnt << 16);
            w.reach()[slot] = uint16_t(rq);
          }
        } else {
          const uint32_t last = st_last(e), near = st_near(e);
          // R6 predecessor among stored hits: the largest one <= Ph - W
          const int hi_ok = Ph - W;
          const int lo_ok = max(Ph - A + 1, ls + 1);  // within A, same subject
          const int cand_s = st_pred(last, st_far(e), near, hi_ok);
          // earlier hits of this round on the same diagonal (rare per lane, but
          // some in almost every round): the best predecessor among them and
          // the mask of those within W of this hit
          int cand_e = 0;
          uint32_t nb = 0;
          if (const int nearly = __reduce_max_sync(kFull, act ? __popc(earlier) : 0); nearly) {
            unsigned rem = earlier;
            for (int it = 0; it < nearly; ++it) {
              const int src = rem ? __ffs(rem) - 1 : lane;
              rem &= rem - 1;
              const int Pj = __shfl_sync(kFull, Ph, src);
              if (act && src != lane) {
                if (Pj <= hi_ok) cand_e = max(cand_e, Pj);
                const int d = Ph - Pj;
                if (d < W) nb |= 1u << d;
              }
            }
          }
          const int cand = max(cand_s, cand_e);
          // not a segment's warm-up (the LEFT test fails there by ls above)
          const bool counts = act && (kTrace || kEither ? Ph >= emit_f : true);
          bool pass = counts && cand >= lo_ok;
          const int64_t sph = st.spbase + Ph;
          if (kEither && counts && !pass)
            pass = has_successor(stream, sph, q, qc, b62, lq, W, A, a.threshold);
          if (kTrace) {
            stat_add<kTrace>(st, kStatRounds, 1);
            stat_add<kTrace>(st, kStatConflictRounds, __any_sync(kFull, act && earlier != 0) ? 1 : 0);
            if (!retrace) {
              stat_add<kTrace>(st, kStatHits, __popc(__ballot_sync(kFull, counts)));
              stat_add<kTrace>(st, kStatPassing, __popc(__ballot_sync(kFull, pass)));
            }
            if (w.wk()[4] < 0)
              stat_add<kTrace>(st, kStatEnqueued,
                               __popc(__ballot_sync(kFull, pass && Ph > int(rch))));
            if (counts && !retrace) {
              trace_push(a, 0, sph, q, 0, 0, 0);
              if (pass) trace_push(a, 1, sph, q, 0, 0, 0);
            }
          }
          // the group's last member writes the diagonal state with its own hit:
          // last = Ph, far = largest hit <= Ph - W (= cand), near = every hit
          // (stored or earlier in the round) within W of Ph
          if (act && (grp >> lane) == 1u) {
            if (last != 0) {
              const int d = Ph - int(last);
              if (d < W) nb |= ((near << d) | (1u << d));
            }
            w.ring()[slot] = st_make(uint32_t(Ph), uint32_t(cand), nb & nearmask);
          }
          enq = pass && Ph > int(rch);
        }
        const unsigned bal = __ballot_sync(kFull, enq);
        if (bal) {
          const int pos = st.qcount + __popc(bal & lanemask_lt(lane));
          if (enq)
            w.queue()[(st.qhead + pos) & (kQcap - 1)] = uint32_t(Ph) | (uint32_t(q) << 16) | eflags;
          st.qcount += __popc(bal);
          __syncwarp();
          while (st.qcount >= 32) {  // a flush may keep entries queued
            if (__shfl_sync(kFull, w.wk()[4], 0) >= 0)
              spill(32);  // segment: to its list
            else
              flush_queue<kTrace, kWin, kSt>(a, w, st, 32, qc, b62, lane, slotc(), M);
          }
        }
        __syncwarp();
      }
      // ---- advance the window ---------------------------------------------
      const unsigned sl = sm & ((npos == 32) ? kFull : ((1u << npos) - 1u));
      if (sl) lastsent = win + 31 - __clz(sl);
      win += npos;
      base_slot += npos;
      if (base_slot >= M) base_slot -= M;
    }
    if (const int sgw = __shfl_sync(kFull, w.wk()[4], 0); sgw >= 0) {
      while (st.qcount > 0) spill(min(st.qcount, 32));
      const int nl = __shfl_sync(kFull, w.wk()[5], 0);
      __threadfence();
      __syncwarp();
      if (lane == 0) {
        a.seg_count[sgw] = nl > a.seg_cap ? -1 : nl;
        st_release(a.seg_done + sgw, a.seq);
      }
    }
    sc = slotc();
    // the next chunk continues the frame after a gap (stale state ages out)
    frame = win + 64;
    base_slot = (base_slot + 64) % M;
    }  // walk
    // ---- the single drain site (chunk end, walker steps) -------------------
    while (st.qcount > 0)
      flush_queue<kTrace, kWin, kSt>(a, w, st, min(st.qcount, 32), qc, b62, lane, sc, M);
  }
  if (kTrace && a.stats && lane == 0)
    for (int i = 0; i < kNumStats; ++i)
      if (st.stat[i]) atomicAdd(a.stats + i, st.stat[i]);
}

size_t smem_bytes(int lq, int ring, int64_t table_entries, int warps) {
  const size_t fixed = 1024 + align16(size_t(lq) + 2 * kQPad + 8);
  const size_t table = table_entries < 0 ? 0
                                         : align16(size_t((kWords + 1 + 7) & ~7) * 2 +
                                                   size_t(table_entries) * 2);
  return fixed + table + size_t(warps) * warp_smem_bytes(ring);
}

template <bool kTrace, int kF, typename OffT>
cudaError_t launch_variant(const SearchArgs &a, int warps, size_t smem, int num_sms,
                           cudaStream_t s) {
  void (*k)(const SearchArgs) = search_warp_kernel<kTrace, kF, OffT, 0, false>;
  if constexpr (kF != BLASTP_FILTER_STATEFUL && kF != BLASTP_FILTER_STATEFUL_RB) {
    if (a.ext_mode == BLASTP_EXT_WINDOW) k = search_warp_kernel<kTrace, kF, OffT, 0, true>;
    else if (a.min_gap == 3) k = search_warp_kernel<kTrace, kF, OffT, 3, false>;
  }
  cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
  if (e != cudaSuccess) return e;
  int per_sm = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, warps * 32, smem);
  if (e != cudaSuccess) return e;
  if (per_sm < 1) return cudaErrorInvalidConfiguration;
  int64_t grid = int64_t(num_sms) * per_sm;
  const int64_t need = (int64_t(a.nchunks) + a.nlong + a.nsegs + warps - 1) / warps;
  if (grid > need) grid = need < 1 ? 1 : need;
  k<<<unsigned(grid), warps * 32, smem, s>>>(a);
  return cudaGetLastError();
}

}  // namespace

int search_ring_slots(int lq, int window) {
  // Diagonal d and d - M share a slot.  A stored hit of d - M lies before
  // d - M + lq, so it can never be within `window` of a hit of d when
  // M >= lq + window; and two diagonals hit inside one 32-position window
  // are distinct slots when M >= lq + 32.
  const int need = lq + (window > 32 ? window : 32) + 8;
  return (need + 7) & ~7;
}

cudaError_t launch_search_warp(const SearchArgs &a_in, int num_sms, cudaStream_t s) {
  static unsigned long long b62_ready = 0;  // one bit per device
  int dev = 0;
  cudaGetDevice(&dev);
  if (!(b62_ready >> dev & 1ull)) {
    int8_t h[32 * 32];
    fill_b62(h);
    cudaError_t e = cudaMemcpyToSymbol(c_b62, h, sizeof(h));
    if (e != cudaSuccess) return e;
    b62_ready |= 1ull << dev;
  }
  SearchArgs a = a_in;
  a.ring = search_ring_slots(a.qv.lq, a.window);
  int optin = 0;
  cudaError_t e = cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  if (e != cudaSuccess) return e;
  const bool trace = a.trace[0] != nullptr;
  const int fm = a.filter_mode;
  const char *tab_env = std::getenv("BLASTP_TABLE");
  const bool force_global = tab_env && !std::strcmp(tab_env, "global");
  const char *warps_env = std::getenv("BLASTP_WARPS");
  const int max_warps = warps_env ? std::max(1, std::min(kMaxWarps, std::atoi(warps_env))) : kMaxWarps;
  int warps_s = 0;
  if (a.table_entries < 65536 && !force_global) {
    warps_s = max_warps;
    while (warps_s > 0 && smem_bytes(a.qv.lq, a.ring, a.table_entries, warps_s) > size_t(optin))
      --warps_s;
  }
  int warps_g = max_warps;
  while (warps_g > 0 && smem_bytes(a.qv.lq, a.ring, -1, warps_g) > size_t(optin)) --warps_g;
  // More resident warps beat a shared-memory table once the table would cost
  // more than a few warps (profiles/r01: q1054, 16 warps + L1/L2 table is
  // faster than 11 warps + shared-memory table).
  const bool force_smem = tab_env && !std::strcmp(tab_env, "smem");
  const bool use_s = warps_s > 0 && (force_smem || warps_s >= std::min(warps_g, 24));
  if (!use_s && warps_g < 1) return cudaErrorInvalidConfiguration;
  const int warps = use_s ? warps_s : warps_g;
  const size_t smem = smem_bytes(a.qv.lq, a.ring, use_s ? a.table_entries : -1, warps);
  auto pick = [&](auto off_tag) -> cudaError_t {
    using OffT = decltype(off_tag);
    if (trace) {
      if (fm == BLASTP_FILTER_EITHER) return launch_variant<true, 1, OffT>(a, warps, smem, num_sms, s);
      if (fm == BLASTP_FILTER_STATEFUL) return launch_variant<true, 2, OffT>(a, warps, smem, num_sms, s);
      if (fm == BLASTP_FILTER_STATEFUL_RB) return launch_variant<true, 3, OffT>(a, warps, smem, num_sms, s);
      return launch_variant<true, 0, OffT>(a, warps, smem, num_sms, s);
    }
    if (fm == BLASTP_FILTER_EITHER) return launch_variant<false, 1, OffT>(a, warps, smem, num_sms, s);
    if (fm == BLASTP_FILTER_STATEFUL) return launch_variant<false, 2, OffT>(a, warps, smem, num_sms, s);
    if (fm == BLASTP_FILTER_STATEFUL_RB) return launch_variant<false, 3, OffT>(a, warps, smem, num_sms, s);
    return launch_variant<false, 0, OffT>(a, warps, smem, num_sms, s);
  };
  return use_s ? pick(uint16_t{}) : pick(uint32_t{});
}

}  // namespace blastp
