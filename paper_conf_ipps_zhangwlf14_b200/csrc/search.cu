// search.cu -- the fused BLASTP ungapped hot path for sm_100a.
//
// One kernel does the whole path of PAPER.md Sec. 3.2-3.4 for a chunk of
// whole subjects per warp:
//
//   hit detection     Alg. 2: lanes = consecutive subject
//                     words, coalesced byte loads, CSR table lookup (R3/R4)
//   "binning/sorting" P:L967-1343: replaced by a per-warp diagonal ring in
//                     shared memory indexed by (s - q) mod M; because the
//                     warp walks its subjects in ascending s, each diagonal's
//                     hits arrive already sorted -- the order the paper's
//                     segmented sort establishes, without materialising bins
//   two-hit filter    P:L1344-1351 (R6): exists p on the same diagonal with
//                     W <= h - p < A; in-iteration predecessors via a 32-bit
//                     lane mask per diagonal, earlier ones via ring.last
//   extension         Alg. 3/5 + Fig. 8 (R7-R10): passing hits
//                     not covered by ext_reach are queued; 32 at a time are
//                     X-dropped lane-parallel and the ext_reach chain is then
//                     resolved per diagonal in queue (= s) order
//   output            P:L1352-1353: one global atomic per emitted HSP
//
// Per-iteration layout: a warp covers 32 consecutive stream positions
// s0-CTX .. s0-CTX+31, CTX = min_gap-1 "context" lanes that were already
// processed by the previous iteration (so that every new hit sees all hits
// at distance < min_gap in the same lane mask).  Each iteration advances
// 32-CTX positions.
#include <cuda_runtime.h>

#include "common.cuh"

namespace blastp {

namespace {

constexpr int kWarps = 4;       // warps per CTA (each independent)
constexpr int kQcap = 64;       // extension queue slots per warp
constexpr int kNeg = -(1 << 30);
constexpr unsigned kFull = 0xffffffffu;

__constant__ int8_t c_b62[32 * 32];

__host__ __device__ constexpr size_t align16(size_t x) { return (x + 15) & ~size_t(15); }

struct WarpSmem {
  int2 *ring;         // [M]: .x = last hit (virtual pos) at <= s0-W, .y = ext_reach
  uint32_t *imask;    // [M]: lanes of the current iteration with a hit on the slot
  uint32_t *hbuf;     // [hb]: flattened hits of the iteration, (q << 5) | lane
  uint32_t *mbuf;     // [hb]: imask value seen by each hit (pass C)
  int2 *queue;        // [kQcap]: (vpos, slot << 16 | q)
  int *fs_vp, *fs_end, *fs_acc;  // [32] flush scratch
};

__host__ __device__ size_t warp_smem_bytes(int ring, int hb) {
  return align16(size_t(ring) * 8) + align16(size_t(ring) * 4) + 2 * align16(size_t(hb) * 4) +
         size_t(kQcap) * 8 + 3 * 32 * 4;
}

__device__ __forceinline__ WarpSmem carve(uint8_t *base, int ring, int hb) {
  WarpSmem w;
  w.ring = reinterpret_cast<int2 *>(base);
  base += align16(size_t(ring) * 8);
  w.imask = reinterpret_cast<uint32_t *>(base);
  base += align16(size_t(ring) * 4);
  w.hbuf = reinterpret_cast<uint32_t *>(base);
  base += align16(size_t(hb) * 4);
  w.mbuf = reinterpret_cast<uint32_t *>(base);
  base += align16(size_t(hb) * 4);
  w.queue = reinterpret_cast<int2 *>(base);
  base += size_t(kQcap) * 8;
  w.fs_vp = reinterpret_cast<int *>(base);
  w.fs_end = w.fs_vp + 32;
  w.fs_acc = w.fs_vp + 64;
  return w;
}

__device__ __forceinline__ unsigned lanemask_lt(int lane) { return (1u << lane) - 1u; }
// bits lo..hi inclusive (0 <= lo <= hi <= 31)
__device__ __forceinline__ unsigned bit_range(int lo, int hi) {
  unsigned upto = (hi >= 31) ? kFull : ((2u << hi) - 1u);
  return upto & ~((1u << lo) - 1u);
}

__device__ __forceinline__ int score(const int8_t *b62, uint32_t qcode, uint32_t scode) {
  return b62[(qcode << 5) | scode];
}

// R7/R8: X-drop extension from the seed word at (q, sp) (sp = stream pos).
// Subject boundaries are sentinels scoring -128, which stops the walk.
__device__ void xdrop_extend(const uint8_t *__restrict__ stream, int64_t sp, int q,
                             const uint8_t *qc, const int8_t *b62, int lq, int wl, int X,
                             int &total, int &llen, int &rlen) {
  int seed = 0;
  for (int i = 0; i < wl; ++i) seed += score(b62, qc[q + i], __ldg(stream + sp + i));
  // right: from (q+wl, sp+wl)
  int run = 0, best = 0, bl = 0;
  {
    const int qi = q + wl;
    const int n = lq - qi;
    const uint8_t *sptr = stream + sp + wl;
    for (int t = 0; t < n; ++t) {
      run += score(b62, qc[qi + t], __ldg(sptr + t));
      if (run > best) { best = run; bl = t + 1; }
      if (best - run >= X) break;
    }
  }
  const int best_r = best;
  rlen = bl;
  run = 0; best = 0; bl = 0;
  {
    const uint8_t *sptr = stream + sp - 1;
    for (int t = 0; t < q; ++t) {
      run += score(b62, qc[q - 1 - t], __ldg(sptr - t));
      if (run > best) { best = run; bl = t + 1; }
      if (best - run >= X) break;
    }
  }
  llen = bl;
  total = seed + best_r + best;
}

// EITHER mode (R6, Fig. 7 reading): does a hit exist at (q+k, sp+k) for some
// k in [W, A-1]?  Scored directly along the diagonal (the definition of a hit).
__device__ bool has_successor(const uint8_t *__restrict__ stream, int64_t sp, int q,
                              const uint8_t *qc, const int8_t *b62, int lq, int W, int A, int T) {
  const int kmax = min(A - 1, lq - 3 - q);
  if (kmax < W) return false;
  // rolling pair scores at offsets j-2, j-1 (offsets 1, 2 lie in the hit word)
  int s1 = score(b62, qc[q + 1], __ldg(stream + sp + 1));
  int s2 = score(b62, qc[q + 2], __ldg(stream + sp + 2));
  for (int j = 3; j <= kmax + 2; ++j) {
    const uint32_t c = __ldg(stream + sp + j);
    if (c == uint32_t(kSentinel)) return false;  // the subject ends: no later word
    const int s3 = score(b62, qc[q + j], c);
    if (j - 2 >= W && s1 + s2 + s3 >= T) return true;
    s1 = s2;
    s2 = s3;
  }
  return false;
}

__device__ __forceinline__ void trace_push(const SearchArgs &a, int which, int64_t sp, int q,
                                           int llen, int rlen, int sc) {
  unsigned long long i = atomicAdd(a.trace_count + which, 1ull);
  if ((long long)i < a.trace_cap[which]) {
    TraceRec r;
    r.sp = sp; r.q = q; r.llen = llen; r.rlen = rlen; r.score = sc;
    r.query_id = a.qv.query_id; r.pad = 0;
    a.trace[which][i] = r;
  }
}

struct WarpState {
  int64_t voff;        // vpos = stream pos + voff
  int64_t first_subj, last_subj;
  int qhead, qcount;
};

// Extend up to 32 queued passing hits lane-parallel, then resolve the
// ext_reach chain (Alg. 3 L19-23, R10) per diagonal in queue order.
__device__ void flush_queue(const SearchArgs &a, const WarpSmem &w, WarpState &st, int n,
                            const uint8_t *qc, const int8_t *b62, int lane) {
  const bool act = lane < n;
  int2 ent = make_int2(0, 0);
  if (act) ent = w.queue[(st.qhead + lane) & (kQcap - 1)];
  const int vp = ent.x;
  const int slot = int(uint32_t(ent.y) >> 16);
  const int q = int(uint32_t(ent.y) & 0xffffu);
  const int64_t sp = int64_t(vp) - st.voff;
  int total = 0, llen = 0, rlen = 0;
  if (act) xdrop_extend(a.stream, sp, q, qc, b62, a.qv.lq, a.word_len, a.xdrop, total, llen, rlen);
  const int endv = vp + a.word_len - 1 + rlen;  // HSP subject end (inclusive), virtual
  const unsigned grp = __match_any_sync(kFull, act ? slot : -1 - lane);
  w.fs_vp[lane] = vp;
  w.fs_end[lane] = endv;
  __syncwarp();
  bool acc = false;
  const bool uniq = (grp == (1u << lane));
  if (act) {
    if (uniq) {
      const int r = w.ring[slot].y;
      acc = vp > r;
      if (acc) w.ring[slot].y = endv;
    } else if (lane == __ffs(grp) - 1) {
      int r = w.ring[slot].y;
      unsigned g = grp;
      while (g) {
        const int j = __ffs(g) - 1;
        g &= g - 1;
        const bool aj = w.fs_vp[j] > r;
        if (aj) r = w.fs_end[j];
        w.fs_acc[j] = aj;
      }
      w.ring[slot].y = r;
    }
  }
  __syncwarp();
  if (act && !uniq) acc = w.fs_acc[lane] != 0;
  if (acc) {
    if (a.trace[2]) trace_push(a, 2, sp, q, llen, rlen, total);
    if (total >= a.cutoff) {
      // subject of the seed: largest i with sstart[i] <= sp
      int64_t lo = st.first_subj, hi = st.last_subj - 1;
      while (lo < hi) {
        const int64_t mid = (lo + hi + 1) >> 1;
        if (__ldg(a.sstart + mid) <= sp) lo = mid; else hi = mid - 1;
      }
      const int64_t s_local = sp - __ldg(a.sstart + lo);
      blastp_hsp h;
      h.query_id = a.qv.query_id;
      h.subject_id = int32_t(a.subject_base + lo);
      h.q_start = q - llen;
      h.s_start = int32_t(s_local) - llen;
      h.diagonal = h.s_start - h.q_start;
      h.length = llen + a.word_len + rlen;
      h.score = total;
      const unsigned long long idx = atomicAdd(a.hsp_count, 1ull);
      if ((long long)idx < a.out_cap) a.out[idx] = h;
    }
  }
  __syncwarp();
  st.qhead = (st.qhead + n) & (kQcap - 1);
  st.qcount -= n;
}

__global__ void __launch_bounds__(kWarps * 32) search_kernel(const SearchArgs a) {
  extern __shared__ __align__(16) uint8_t smem[];
  int8_t *b62 = reinterpret_cast<int8_t *>(smem);
  uint8_t *qc = smem + 1024;
  const int lq = a.qv.lq;
  for (int i = threadIdx.x; i < 1024; i += blockDim.x) b62[i] = c_b62[i];
  for (int i = threadIdx.x; i < lq; i += blockDim.x) qc[i] = a.qv.qcodes[i];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int M = a.ring, HB = a.hitbuf;
  WarpSmem w = carve(smem + 1024 + align16(lq) + size_t(warp) * warp_smem_bytes(M, HB), M, HB);
  for (int i = lane; i < M; i += 32) {
    w.ring[i] = make_int2(kNeg, kNeg);
    w.imask[i] = 0;
  }
  __syncthreads();

  const uint32_t *__restrict__ woff = a.qv.woff;
  const uint16_t *__restrict__ qpos = a.qv.qpos;
  const uint8_t *__restrict__ stream = a.stream;
  const int W = a.min_gap, A = a.window, CTX = W - 1, step = 32 - CTX;
  const unsigned lastmask = (CTX == 0) ? kFull : (kFull >> CTX);  // lanes <= 31-CTX
  const bool either = a.filter_mode == BLASTP_FILTER_EITHER;
  const bool tracing = a.trace[0] != nullptr;

  WarpState st;
  int vbase = 1 << 20;
  for (;;) {
    unsigned long long ci = 0;
    if (lane == 0) ci = atomicAdd(a.chunk_cursor, 1ull);
    ci = __shfl_sync(kFull, ci, 0);
    if (ci >= (unsigned long long)a.nchunks) break;
    const Chunk ch = a.chunks[ci];
    if (vbase > (1 << 30)) {  // re-base the virtual positions (ring ages out)
      for (int i = lane; i < M; i += 32) w.ring[i] = make_int2(kNeg, kNeg);
      __syncwarp();
      vbase = 1 << 20;
    }
    st.voff = int64_t(vbase) - ch.start;
    st.first_subj = ch.first_subj;
    st.last_subj = ch.last_subj;
    st.qhead = 0;
    st.qcount = 0;
    int lastsent = vbase - 1;  // virtual pos of the last sentinel before the iteration
    int base_slot = int((int64_t(vbase) - CTX + lq) % M);

    for (int64_t s0 = ch.start; s0 < ch.end; s0 += step) {
      const int64_t p = s0 - CTX + lane;
      const int vp0 = int(s0 - CTX + st.voff);  // virtual pos of lane 0
      // residues p, p+1, p+2 (one coalesced byte load + shuffles)
      const uint32_t r0 = __ldg(stream + p);
      uint32_t xr = 0;
      if (lane < 2) xr = __ldg(stream + s0 - CTX + 32 + lane);
      uint32_t r1 = __shfl_down_sync(kFull, r0, 1);
      uint32_t r2 = __shfl_down_sync(kFull, r0, 2);
      const uint32_t x0 = __shfl_sync(kFull, xr, 0), x1 = __shfl_sync(kFull, xr, 1);
      if (lane == 31) { r1 = x0; r2 = x1; }
      if (lane == 30) r2 = x0;
      const bool inrange = (p >= ch.start) && (p < ch.end);
      const bool valid = inrange && (max(r0, max(r1, r2)) < uint32_t(kNumLetters));
      const unsigned sm = __ballot_sync(kFull, r0 == uint32_t(kSentinel));

      uint32_t o = 0, cnt = 0;
      if (valid) {
        const uint32_t c = (r0 * kNumLetters + r1) * kNumLetters + r2;
        o = __ldg(woff + c);
        cnt = __ldg(woff + c + 1) - o;
      }
      uint32_t incl = cnt;
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) {
        const uint32_t t = __shfl_up_sync(kFull, incl, d);
        if (lane >= d) incl += t;
      }
      const uint32_t H = __shfl_sync(kFull, incl, 31);

      if (H != 0) {
        // per-hit helpers ------------------------------------------------
        auto slot_of = [&](int l, int q) {
          int s = base_slot + l - q;
          s += (s < 0) ? M : 0;
          s -= (s >= M) ? M : 0;
          return s;
        };
        auto seg_lo_of = [&](int l) {
          const unsigned prior = sm & ((l == 31) ? kFull : ((2u << l) - 1u));
          return prior ? (32 - __clz(prior)) : 0;
        };
        // pass B body: two-hit test (R6) + coverage pre-check; returns enqueue
        auto test_hit = [&](int l, int q, int slot, unsigned m, int &vpk) -> bool {
          if (l < CTX) return false;  // context lane: already tested last iteration
          const int P = vp0 + l;
          const int lo_seg = seg_lo_of(l);
          const int lo = max(lo_seg, l - A + 1), hi = l - W;
          bool pass = (hi >= lo) && (m & bit_range(lo, hi)) != 0;
          const int2 rr = w.ring[slot];
          if (!pass && lo_seg == 0 && rr.x > lastsent && rr.x >= P - A + 1) pass = true;
          const int64_t sp = s0 - CTX + l;
          if (!pass && either) pass = has_successor(stream, sp, q, qc, b62, lq, W, A, a.threshold);
          if (tracing) {
            trace_push(a, 0, sp, q, 0, 0, 0);
            if (pass) trace_push(a, 1, sp, q, 0, 0, 0);
          }
          vpk = P;
          return pass && P > rr.y;
        };
        auto enqueue_round = [&](bool enq, int vpk, int slot, int q) {
          const unsigned bal = __ballot_sync(kFull, enq);
          if (bal) {
            const int pos = st.qcount + __popc(bal & lanemask_lt(lane));
            if (enq) w.queue[(st.qhead + pos) & (kQcap - 1)] = make_int2(vpk, (slot << 16) | q);
            st.qcount += __popc(bal);
            __syncwarp();
            if (st.qcount >= 32) flush_queue(a, w, st, 32, qc, b62, lane);
          }
        };

        if (H <= uint32_t(HB)) {
          // ---- fast path: flatten the iteration's hits into smem -------
          const uint32_t excl = incl - cnt;
          for (uint32_t i = 0; i < cnt; ++i)
            w.hbuf[excl + i] = (uint32_t(__ldg(qpos + o + i)) << 5) | uint32_t(lane);
          __syncwarp();
          const int rounds = int((H + 31) >> 5);
          // pass A: mark the lanes that hit each diagonal slot
          for (int r = 0; r < rounds; ++r) {
            const uint32_t k = uint32_t(r * 32 + lane);
            if (k < H) {
              const uint32_t e = w.hbuf[k];
              const int l = int(e & 31), q = int(e >> 5);
              atomicOr(&w.imask[slot_of(l, q)], 1u << l);
            }
          }
          __syncwarp();
          // pass B: two-hit test, coverage pre-check, enqueue in s order
          for (int r = 0; r < rounds; ++r) {
            const uint32_t k = uint32_t(r * 32 + lane);
            bool enq = false;
            int vpk = 0, slot = 0, q = 0;
            if (k < H) {
              const uint32_t e = w.hbuf[k];
              const int l = int(e & 31);
              q = int(e >> 5);
              slot = slot_of(l, q);
              const unsigned m = w.imask[slot];
              w.mbuf[k] = m;
              enq = test_hit(l, q, slot, m, vpk);
            }
            enqueue_round(enq, vpk, slot, q);
          }
          __syncwarp();
          // pass C: ring.last <- last hit at lanes <= 31-CTX; clear masks
          for (int r = 0; r < rounds; ++r) {
            const uint32_t k = uint32_t(r * 32 + lane);
            if (k < H) {
              const uint32_t e = w.hbuf[k];
              const int l = int(e & 31), q = int(e >> 5);
              const int slot = slot_of(l, q);
              const unsigned m2 = w.mbuf[k] & lastmask;
              if (m2 && l == 31 - __clz(m2)) w.ring[slot].x = vp0 + l;
              w.imask[slot] = 0;
            }
          }
          __syncwarp();
        } else {
          // ---- slow path (hit-dense iteration): lane-major cooperative --
          for (int pass = 0; pass < 4; ++pass) {
            for (int j = 0; j < 32; ++j) {
              const uint32_t cj = __shfl_sync(kFull, cnt, j);
              const uint32_t oj = __shfl_sync(kFull, o, j);
              for (uint32_t kk = 0; kk < cj; kk += 32) {
                const uint32_t k = kk + uint32_t(lane);
                const bool active = k < cj;
                const int q = active ? int(__ldg(qpos + oj + k)) : 0;
                const int slot = active ? slot_of(j, q) : 0;
                if (pass == 0) {
                  if (active) atomicOr(&w.imask[slot], 1u << j);
                } else if (pass == 1) {
                  bool enq = false;
                  int vpk = 0;
                  if (active) enq = test_hit(j, q, slot, w.imask[slot], vpk);
                  enqueue_round(enq, vpk, slot, q);
                } else if (pass == 2) {
                  if (active) {
                    const unsigned m2 = w.imask[slot] & lastmask;
                    if (m2 && j == 31 - __clz(m2)) w.ring[slot].x = vp0 + j;
                  }
                } else {
                  if (active) w.imask[slot] = 0;
                }
              }
            }
            __syncwarp();
          }
        }
      }
      // carry the last sentinel before the next iteration's first lane
      const unsigned sl = sm & lastmask;
      if (sl) lastsent = vp0 + (31 - __clz(sl));
      base_slot += step;
      if (base_slot >= M) base_slot -= M;
    }
    while (st.qcount > 0) flush_queue(a, w, st, min(st.qcount, 32), qc, b62, lane);
    vbase += int(ch.end - ch.start) + M + A + 128;
  }
}

}  // namespace

int search_ring_slots(int lq, int window) {
  // M > lq + window + 32 keeps aliased slots (diagonal d and d+M) from ever
  // looking recent; multiple of 32.
  return ((lq + window + 64) + 31) & ~31;
}

int search_hitbuf(int lq) { return lq <= 1100 ? 256 : 512; }

size_t search_smem_bytes(int lq, int ring, int hitbuf, int warps) {
  return 1024 + align16(size_t(lq)) + size_t(warps) * warp_smem_bytes(ring, hitbuf);
}

cudaError_t launch_search(const SearchArgs &a, int num_sms, cudaStream_t s) {
  static unsigned long long b62_ready = 0;  // one bit per device
  int dev = 0;
  cudaGetDevice(&dev);
  if (!(b62_ready >> dev & 1ull)) {
    int8_t h[32 * 32];
    for (int i = 0; i < 32; ++i)
      for (int j = 0; j < 32; ++j)
        h[i * 32 + j] = (i < kNumLetters && j < kNumLetters) ? kBlosum62[i][j]
                                                              : int8_t(kSentinelScore);
    cudaError_t e = cudaMemcpyToSymbol(c_b62, h, sizeof(h));
    if (e != cudaSuccess) return e;
    b62_ready |= 1ull << dev;
  }
  int optin = 0;
  cudaError_t e = cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  if (e != cudaSuccess) return e;
  // as many independent warps per CTA as the per-warp diagonal rings allow
  int warps = kWarps;
  while (warps > 1 && search_smem_bytes(a.qv.lq, a.ring, a.hitbuf, warps) > size_t(optin)) warps >>= 1;
  const size_t smem = search_smem_bytes(a.qv.lq, a.ring, a.hitbuf, warps);
  if (smem > size_t(optin)) return cudaErrorInvalidConfiguration;
  e = cudaFuncSetAttribute(search_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
  if (e != cudaSuccess) return e;
  int per_sm = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, search_kernel, warps * 32, smem);
  if (e != cudaSuccess) return e;
  if (per_sm < 1) return cudaErrorInvalidConfiguration;
  int64_t grid = int64_t(num_sms) * per_sm;
  const int64_t need = (int64_t(a.nchunks) + warps - 1) / warps;
  if (grid > need) grid = need < 1 ? 1 : need;
  search_kernel<<<unsigned(grid), warps * 32, smem, s>>>(a);
  return cudaGetLastError();
}

}  // namespace blastp
