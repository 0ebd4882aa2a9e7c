// search_cta.cu -- "cta" variant of the fused BLASTP ungapped hot path (sm_100a).
//
// One persistent CTA per SM, warp-specialised:
//
//  * NP producer warps walk a chunk of whole subjects in windows of
//    32*NP word positions (group g = warp g = 32 consecutive positions):
//      hit detection  Alg. 2: lane = word position, coalesced
//                     residue loads prefetched one window ahead, lookup table
//                     (R3) in shared memory;
//      binning        P:L837-948 / Fig. 5: hits are binned by diagonal into a
//                     shared-memory counting sort (one bin per diagonal of the
//                     window, atomicAdd on the bin counter as in Alg. 2 L18);
//      filtering      P:L1344-1360 (R6): each hit scans its diagonal's bin for a
//                     left neighbour with W <= h - p < A in the same subject;
//                     older hits come from a per-diagonal state ring (last hit,
//                     last hit <= last - W, bit mask of those in between);
//      hand-off       the bin's owner (its rightmost hit) updates the ring and
//                     appends the bin's passing hits, in ascending s, to the
//                     FIFO of the consumer warp that owns the diagonal.
//  * NC consumer warps drain their FIFOs 32 entries at a time: lane-parallel
//    X-drop extension (Alg. 3/5 + Fig. 8, R7-R9), then the
//    ext_reach chain (Alg. 3 L19-23, R10) resolved per diagonal in FIFO (= s)
//    order; HSPs with score >= cutoff are appended to the output.
//
// Producer-only synchronisation uses named barrier 1; producers and consumers
// communicate only through the FIFOs (sequence-numbered slots) and the
// per-diagonal ext_reach array.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>

#include "search_common.cuh"

namespace blastp {

cudaError_t launch_search_warp(const SearchArgs &a, int num_sms, cudaStream_t s);

using namespace dev;

namespace {

constexpr int kThreads = 1024;
constexpr int kFrameMin = 1024;    // first frame position (> window A)
constexpr int kFrameSpan = 32768;  // rebase step of 16-bit frame positions
constexpr uint32_t kOwnerBit = 0x80000000u;

__constant__ int8_t c_b62[32 * 32];

struct CtaConfig {
  int np, nc;       // producer / consumer warps
  int nmax;         // positions per window (32 * np)
  int cap;          // hits per window (bin storage)
  int nb;           // bins per window (diagonals): nmax + lq
  int M;            // diagonal ring slots
  int qcap;         // FIFO slots per consumer (power of 2)
  int smem_table;   // 1: lookup table staged in shared memory
};

// Shared control block (producers write, everybody may read).
struct Ctrl {
  int64_t spbase;      // stream position of frame position 0
  int64_t end;         // frame position of the chunk end (exclusive)
  int64_t first_subj, last_subj;
  unsigned int vbase;  // vpos (CTA-monotonic) of frame position 0
  int win;             // frame position of the window start
  int lastsent;        // frame position of the last sentinel before `win`
  int base_slot;       // ring slot of bin 0 of the window
  int have_chunk;
  int ngroups;         // groups consumed by this window (0: slow path)
  unsigned int H;      // hits of this window
  volatile int done;   // producers finished
};

struct Smem {
  int8_t *b62;
  uint8_t *qc;
  const uint16_t *woff16;
  const uint16_t *qpos;
  uint64_t *ring;      // [M] last | far << 16 | near << 32
  unsigned int *reach; // [M] ext_reach as vpos (0 = none)
  uint32_t *rec;       // [cap] bin << 11 | pos-in-window (| owner bit)
  uint16_t *rank;      // [cap]
  uint16_t *bucketed;  // [cap] positions in window, grouped by bin
  uint8_t *pflag;      // [cap] pass flag by bin slot
  uint32_t *cnt;       // [nb + 1] bin counters, then exclusive starts
  uint32_t *gtot;      // [32] hits per group
  uint32_t *gsent;     // [32] sentinel lane mask per group
  int *gcarry;         // [32] last sentinel before group
  uint32_t *scan_tmp;  // [32] warp totals of the bin scan
  uint32_t *gO, *gC;   // [32] group-0 offsets / counts (slow path)
  uint32_t *posI;      // [nmax] inclusive hit count within the group, per position
  uint32_t *posO;      // [nmax] lookup-table offset, per position
  Ctrl *ctrl;
  uint4 *fifo;         // [nc * qcap]: vpos, sp, q | slot << 16, seq
  unsigned int *ftail; // [nc] reservation counters
  volatile unsigned int *fhead;  // [nc] consumer heads
  int *fs;             // [nc * 96] consumer flush scratch
};

__host__ __device__ size_t smem_layout(const CtaConfig &c, int lq, int64_t entries, size_t *off) {
  size_t o = 0;
  auto take = [&](int i, size_t bytes) {
    if (off) off[i] = o;
    o += align16(bytes);
  };
  take(0, 1024);                                          // b62
  take(1, size_t(lq) + 2 * kQPad + 8);                    // qc
  take(2, c.smem_table ? size_t((kWords + 1 + 7) & ~7) * 2 + size_t(entries) * 2 : 0);
  take(3, size_t(c.M) * 8);                               // ring
  take(4, size_t(c.M) * 4);                               // reach
  take(5, size_t(c.cap) * 4);                             // rec
  take(6, size_t(c.cap) * 2);                             // rank
  take(7, size_t(c.cap) * 2);                             // bucketed
  take(8, size_t(c.cap));                                 // pflag
  take(9, size_t(c.nb + 1) * 4);                          // cnt
  take(10, 32 * 4 * 7);                                   // group arrays + scan tmp
  take(11, sizeof(Ctrl));
  take(12, size_t(c.nc) * c.qcap * 16);                   // fifo
  take(13, size_t(c.nc) * 4 * 2);                         // ftail, fhead
  take(14, size_t(c.nc) * 96 * 4);                        // fs
  take(15, size_t(c.nmax) * 8);                           // posI, posO
  return o;
}

__device__ __forceinline__ void pbar(int np) {
  asm volatile("bar.sync 1, %0;\n" ::"r"(np * 32) : "memory");
}

template <bool kStats>
struct Stats {
  unsigned long long v[kNumStats];
  __device__ void zero() {
    if (kStats)
      for (int i = 0; i < kNumStats; ++i) v[i] = 0;
  }
  __device__ void add(int i, unsigned long long x) {
    if (kStats) v[i] += x;
  }
  __device__ void flush(const SearchArgs &a) {
    if (kStats && a.stats)
      for (int i = 0; i < kNumStats; ++i)
        if (v[i]) atomicAdd(a.stats + i, v[i]);
  }
};

// ------------------------------------------------------------ consumers

template <bool kTrace>
__device__ void consumer(const SearchArgs &a, const CtaConfig &c, const Smem &S, int cidx,
                         int lane) {
  Stats<kTrace> st;
  st.zero();
  uint4 *fifo = S.fifo + size_t(cidx) * c.qcap;
  int *fs = S.fs + cidx * 96;
  unsigned int head = 0;
  const unsigned qmask = unsigned(c.qcap) - 1u;
  for (;;) {
    // entries are ready when their sequence number matches the slot's index;
    // idle consumers probe one slot and sleep (they must not steal issue
    // slots from the producers)
    // the producers' completion flag: written once by producer warp 0 after
    // its __threadfence_block (release), read here volatile (acquire side);
    // racecheck reports this flag handshake as a shared-memory hazard, the
    // only one in the library (profiles/r02/sanitizer_*.log)
    const bool done = *reinterpret_cast<volatile int *>(&S.ctrl->done) != 0;
    if (!done) {
      unsigned probe = 0;
      if (lane == 0)
        probe = reinterpret_cast<volatile unsigned int *>(&fifo[(head + 31u) & qmask].w)[0];
      probe = __shfl_sync(kFull, probe, 0);
      if (probe != head + 32u) {
        __nanosleep(1000);
        continue;
      }
    }
    const volatile unsigned int *seqp =
        reinterpret_cast<volatile unsigned int *>(&fifo[(head + lane) & qmask].w);
    const bool ready = (*seqp == head + unsigned(lane) + 1u);
    const unsigned rb = __ballot_sync(kFull, ready);
    const int n = __popc(~rb) == 0 ? 32 : (__ffs(~rb) - 1);  // contiguous ready prefix
    if (n < 32 && !done) {
      __nanosleep(200);
      continue;
    }
    if (n == 0) break;  // done and drained
    __threadfence_block();
    const uint4 ent = fifo[(head + lane) & qmask];
    const bool act = lane < n;
    const unsigned vpos = ent.x;
    const int64_t sp = int64_t(ent.y);
    const int q = int(ent.z & 0xffffu);
    const int slot = int(ent.z >> 16);
    // skip hits already covered by an extension resolved in an earlier batch
    // (ext_mode HIT, Alg. 4: ext_reach stays 0, every passing hit is extended)
    const bool hitm = a.ext_mode == BLASTP_EXT_HIT;
    const bool pre = act && (hitm || vpos > S.reach[slot]);
    int total = 0, llen = 0, rlen = 0, scanned = 0;
    if (pre) xdrop_extend(a.stream, sp, q, S.qc, S.b62, a.xdrop, total, llen, rlen, scanned);
    if (kTrace) {
      st.add(kStatFlushes, 1);
      st.add(kStatExtended, __popc(__ballot_sync(kFull, pre)));
      st.add(kStatXdropSteps, __reduce_add_sync(kFull, unsigned(scanned)));
      st.add(kStatXdropLaneSlots, 32ull * __reduce_max_sync(kFull, unsigned(scanned)));
    }
    const unsigned endv = vpos + 2u + unsigned(rlen);  // subject end of the HSP (vpos)
    bool acc = false;
    if (hitm) {
      acc = pre;
    } else if (const unsigned grp = __match_any_sync(kFull, pre ? slot : -1),
               uniq = grp == (1u << lane);
               __all_sync(kFull, uniq || !pre)) {
      if (pre) {
        acc = vpos > S.reach[slot];
        if (acc) S.reach[slot] = endv;
      }
    } else {
      fs[lane] = int(vpos);
      fs[32 + lane] = int(endv);
      __syncwarp();
      if (pre) {
        if (uniq) {
          acc = vpos > S.reach[slot];
          if (acc) S.reach[slot] = endv;
        } else if (lane == __ffs(grp) - 1) {
          unsigned r = S.reach[slot];
          unsigned g = grp;
          while (g) {
            const int j = __ffs(g) - 1;
            g &= g - 1;
            const bool aj = unsigned(fs[j]) > r;
            if (aj) r = unsigned(fs[32 + j]);
            fs[64 + j] = aj;
          }
          S.reach[slot] = r;
        }
      }
      __syncwarp();
      if (pre && !uniq) acc = fs[64 + lane] != 0;
    }
    if (kTrace) {
      st.add(kStatAccepted, __popc(__ballot_sync(kFull, acc)));
      st.add(kStatEmitted, __popc(__ballot_sync(kFull, acc && total >= a.cutoff)));
      if (acc) trace_push(a, 2, sp, q, llen, rlen, total);
    }
    if (acc) emit_hsp(a, sp, q, llen, rlen, total, 0, a.nseq);
    __syncwarp();
    head += unsigned(n);
    if (lane == 0) S.fhead[cidx] = head;
  }
  if (lane == 0) st.flush(a);
}

// ------------------------------------------------------------ producers

// Append a passing hit to its diagonal's consumer FIFO (blocks while full).
__device__ __forceinline__ void fifo_push(const CtaConfig &c, const Smem &S, int slot,
                                          unsigned vpos, unsigned sp, int q) {
  const int cidx = slot % c.nc;
  const unsigned t = atomicAdd(&S.ftail[cidx], 1u);
  while (t - S.fhead[cidx] >= unsigned(c.qcap)) __nanosleep(100);
  uint4 *f = &S.fifo[size_t(cidx) * c.qcap + (t & unsigned(c.qcap - 1))];
  f->x = vpos;
  f->y = sp;
  f->z = unsigned(q) | (unsigned(slot) << 16);
  __threadfence_block();
  reinterpret_cast<volatile unsigned int *>(&f->w)[0] = t + 1u;
}

template <bool kTrace, bool kEither, typename OffT>
__device__ void producer(const SearchArgs &a, const CtaConfig &c, const Smem &S, const OffT *woff,
                         const uint16_t *qpos, int warp, int lane) {
  Stats<kTrace> st;
  st.zero();
  Ctrl &C = *S.ctrl;
  const uint8_t *__restrict__ stream = a.stream;
  const int lq = a.qv.lq, W = a.min_gap, A = a.window, M = c.M, NP = c.np;
  const int ptid = warp * 32 + lane, NPT = NP * 32;
  const uint32_t nearmask = (1u << W) - 2u;
  // residue prefetch for this warp's group of the next window (valid for any
  // window that starts at the same stream position)
  int64_t pf_sp = -1;
  uint32_t pf_r0 = 0, pf_x = 0;

  for (;;) {
    // ---- chunk management ---------------------------------------------------
    if (ptid == 0 && !C.have_chunk) {
      const unsigned long long ci = atomicAdd(a.chunk_cursor, 1ull);
      Chunk ch;
      if (!fetch_chunk(a, ci, ch)) {
        C.have_chunk = -1;
      } else {
        const int frame = C.win;  // continue the frame (stale state ages out)
        C.spbase = ch.start - frame;
        C.end = ch.end - C.spbase;
        C.first_subj = ch.first_subj;
        C.last_subj = ch.last_subj;
        C.lastsent = frame - 1;  // the sentinel before the chunk
        C.have_chunk = 1;
      }
    }
    pbar(NP);
    if (C.have_chunk < 0) break;
    // ---- rebase 16-bit frame positions --------------------------------------
    if (C.win >= kFrameMin + kFrameSpan) {
      for (int i = ptid; i < M; i += NPT) {
        const uint64_t e = S.ring[i];
        auto rb = [](uint32_t v) { return v > uint32_t(kFrameSpan) ? v - kFrameSpan : 0u; };
        const uint32_t last = rb(uint32_t(e) & 0xffffu), far = rb(uint32_t(e) >> 16);
        S.ring[i] = uint64_t(last | (far << 16)) | (e & 0xffff00000000ull);
      }
      pbar(NP);
      if (ptid == 0) {
        C.win -= kFrameSpan;
        C.lastsent -= kFrameSpan;
        C.end -= kFrameSpan;
        C.spbase += kFrameSpan;
        C.vbase += kFrameSpan;
      }
      pbar(NP);
    }
    const int win = C.win;
    const int64_t spbase = C.spbase, end = C.end;
    const int lastsent = C.lastsent;
    const unsigned vbase = C.vbase;
    const int base_slot = C.base_slot;
    if (kTrace && ptid == 0) st.add(kStatIterations, 1);

    // ---- (C) lookup: group g = warp ------------------------------------------
    const int Pg = win + 32 * warp;  // frame position of lane 0 of the group
    const int64_t sp0 = spbase + Pg;
    uint32_t r0, xr;
    if (pf_sp == sp0) {
      r0 = pf_r0;
      xr = pf_x;
    } else {
      r0 = __ldg(stream + sp0 + lane);
      xr = lane < 2 ? __ldg(stream + sp0 + 32 + lane) : 0u;
    }
    uint32_t r1 = __shfl_down_sync(kFull, r0, 1), r2 = __shfl_down_sync(kFull, r0, 2);
    {
      const uint32_t x0 = __shfl_sync(kFull, xr, 0), x1 = __shfl_sync(kFull, xr, 1);
      if (lane == 31) { r1 = x0; r2 = x1; }
      if (lane == 30) r2 = x0;
    }
    const bool inchunk = int64_t(Pg + lane) < end;
    const bool valid = inchunk && (max(r0, max(r1, r2)) < uint32_t(kNumLetters));
    const unsigned sm = __ballot_sync(kFull, inchunk && r0 == uint32_t(kSentinel));
    uint32_t o = 0, cnt = 0;
    if (valid) {
      const uint32_t code = (r0 * kNumLetters + r1) * kNumLetters + r2;
      o = woff[code];
      cnt = uint32_t(woff[code + 1]) - o;
    }
    uint32_t incl = cnt;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const uint32_t t = __shfl_up_sync(kFull, incl, d);
      if (lane >= d) incl += t;
    }
    if (lane == 31) S.gtot[warp] = incl;
    if (lane == 0) S.gsent[warp] = sm;
    S.posI[32 * warp + lane] = incl;
    S.posO[32 * warp + lane] = o;
    if (warp == 0) {
      S.gO[lane] = o;
      S.gC[lane] = cnt;
    }
    pbar(NP);
    // ---- (D) window plan (every producer warp computes it redundantly) -------
    const uint32_t gt = lane < NP ? S.gtot[lane] : 0u;
    uint32_t gincl = gt;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const uint32_t t = __shfl_up_sync(kFull, gincl, d);
      if (lane >= d) gincl += t;
    }
    const unsigned fit = __ballot_sync(kFull, lane < NP && gincl <= uint32_t(c.cap));
    const int ngroups = __popc(fit);  // groups are a prefix (gincl non-decreasing)
    const uint32_t H = ngroups ? __shfl_sync(kFull, gincl, ngroups - 1) : 0u;
    if (warp == 0) {
      // last sentinel before each group
      const uint32_t gs = lane < NP ? S.gsent[lane] : 0u;
      const unsigned nz = __ballot_sync(kFull, gs != 0) & lanemask_lt(lane);
      int carry = lastsent;
      // every lane fetches the sentinel mask of the last earlier group having one
      const int src = nz ? 31 - __clz(nz) : lane;
      const uint32_t msrc = __shfl_sync(kFull, gs, src);
      if (nz) carry = win + 32 * src + (31 - __clz(msrc));
      if (lane < NP) S.gcarry[lane] = carry;
    }
    // prefetch this warp's residues of the next window (advance by ngroups or 1)
    {
      const int nwin = win + 32 * (ngroups ? ngroups : 1);
      const int64_t nsp = spbase + nwin + 32 * warp;
      pf_r0 = __ldg(stream + nsp + lane);
      pf_x = lane < 2 ? __ldg(stream + nsp + 32 + lane) : 0u;
      pf_sp = nsp;
    }

    if (ngroups == 0) {
      // ---- slow path: group 0 alone has more than `cap` hits -----------------
      // Positions one at a time: the hits of one position lie on distinct
      // diagonals, and all earlier positions are already in the ring state.
      pbar(NP);
      const uint32_t gs0 = S.gsent[0];
      for (int l = 0; l < 32; ++l) {
        const uint32_t ol = S.gO[l], cl = S.gC[l];
        const int P = win + l;
        const uint32_t prior = gs0 & ((l == 31) ? kFull : ((2u << l) - 1u));
        const int ls = prior ? (win + 31 - __clz(prior)) : lastsent;
        for (uint32_t k = ptid; k < cl; k += NPT) {
          const int q = qpos[ol + k];
          int slot = (base_slot + l - q + lq - 1) % M;
          if (slot < 0) slot += M;
          const uint64_t e = S.ring[slot];
          uint32_t last = uint32_t(e) & 0xffffu, far = (uint32_t(e) >> 16) & 0xffffu,
                   near = uint32_t(e >> 32) & 0xffu;
          const int cand = st_pred(last, far, near, P - W);
          bool pass = cand >= max(P - A + 1, ls + 1);
          const int64_t sph = spbase + P;
          if (kEither && !pass)
            pass = has_successor(stream, sph, q, S.qc, S.b62, lq, W, A, a.threshold);
          if (kTrace) {
            trace_push(a, 0, sph, q, 0, 0, 0);
            if (pass) trace_push(a, 1, sph, q, 0, 0, 0);
            st.add(kStatHits, 1);
            st.add(kStatPassing, pass);
          }
          st_append(last, far, near, P, W, nearmask);
          S.ring[slot] = uint64_t(last | (far << 16)) | (uint64_t(near) << 32);
          const unsigned vp = vbase + unsigned(P);
          if (pass && vp > S.reach[slot]) {
            if (kTrace) st.add(kStatEnqueued, 1);
            fifo_push(c, S, slot, vp, unsigned(sph), q);
          }
        }
        pbar(NP);
      }
    } else {
      // ---- (E) generate + bin by diagonal --------------------------------------
      // 32-hit rounds of all consumed groups, dealt round-robin to the warps
      // (groups differ in hit count; this keeps the phase balanced).
      {
        const uint32_t rg = (lane < ngroups) ? (gt + 31u) >> 5 : 0u;
        uint32_t rincl = rg;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
          const uint32_t t = __shfl_up_sync(kFull, rincl, d);
          if (lane >= d) rincl += t;
        }
        const uint32_t rounds = __shfl_sync(kFull, rincl, 31);
        for (uint32_t rho = warp; rho < rounds; rho += NP) {
          const int gg = __popc(__ballot_sync(kFull, rincl <= rho));  // group of the round
          const uint32_t r0g = __shfl_sync(kFull, rincl - rg, gg);
          const uint32_t gofs = __shfl_sync(kFull, gincl - gt, gg);
          const uint32_t Hg = __shfl_sync(kFull, gt, gg);
          const uint32_t k = (rho - r0g) * 32u + uint32_t(lane);
          const uint32_t *pi = S.posI + 32 * gg;
          int own = 0;
#pragma unroll
          for (int b = 16; b >= 1; b >>= 1)
            if (pi[own + b - 1] <= k) own += b;
          if (k < Hg) {
            const uint32_t e_own = own ? pi[own - 1] : 0u;
            const int q = qpos[S.posO[32 * gg + own] + (k - e_own)];
            const int prel = 32 * gg + own;
            const int bin = prel - q + lq - 1;
            const uint32_t idx = gofs + k;
            S.rec[idx] = (uint32_t(bin) << 11) | uint32_t(prel);
            S.rank[idx] = uint16_t(atomicAdd(&S.cnt[bin], 1u));
          }
        }
      }
      if (kTrace && ptid == 0) st.add(kStatRounds, 1);
      pbar(NP);
      // ---- (F) exclusive scan of the bin counters --------------------------------
      {
        const int nb1 = c.nb + 1;
        const int per = (nb1 + NPT - 1) / NPT;
        const int lo = ptid * per, hi = min(lo + per, nb1);
        uint32_t sum = 0;
        for (int i = lo; i < hi; ++i) sum += S.cnt[i];
        uint32_t inc = sum;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
          const uint32_t t = __shfl_up_sync(kFull, inc, d);
          if (lane >= d) inc += t;
        }
        if (lane == 31) S.scan_tmp[warp] = inc;
        pbar(NP);
        uint32_t wsum = lane < NP ? S.scan_tmp[lane] : 0u;
        uint32_t winc = wsum;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
          const uint32_t t = __shfl_up_sync(kFull, winc, d);
          if (lane >= d) winc += t;
        }
        const uint32_t wbase = __shfl_sync(kFull, winc - wsum, warp);
        uint32_t run = wbase + inc - sum;
        for (int i = lo; i < hi; ++i) {
          const uint32_t v = S.cnt[i];
          S.cnt[i] = run;
          run += v;
        }
      }
      pbar(NP);
      // ---- (G) scatter positions into their bins --------------------------------
      for (uint32_t idx = ptid; idx < H; idx += NPT) {
        const uint32_t r = S.rec[idx];
        S.bucketed[S.cnt[r >> 11] + S.rank[idx]] = uint16_t(r & 0x7ffu);
      }
      pbar(NP);
      // ---- (H) two-hit test (R6) -------------------------------------------------
      for (uint32_t idx = ptid; idx < H; idx += NPT) {
        const uint32_t r = S.rec[idx];
        const int bin = int(r >> 11), prel = int(r & 0x7ffu);
        const int P = win + prel;
        const int q = prel - bin + lq - 1;
        const int g = prel >> 5, l = prel & 31;
        const uint32_t gm = S.gsent[g] & ((l == 31) ? kFull : ((2u << l) - 1u));
        const int ls = gm ? (win + 32 * g + 31 - __clz(gm)) : S.gcarry[g];
        const int lo_ok = max(prel - A + 1, ls - win + 1);  // window-relative bounds
        const int hi_ok = prel - W;
        const uint32_t s = S.cnt[bin], e = S.cnt[bin + 1];
        bool pass = false;
        int maxp = prel;
        if (e - s > 1) {  // most bins hold a single hit
          for (uint32_t j = s; j < e; ++j) {
            const int p = S.bucketed[j];
            maxp = max(maxp, p);
            pass |= (p >= lo_ok) && (p <= hi_ok);
          }
        }
        int slot = base_slot + bin;
        slot -= (slot >= M) ? M : 0;
        if (!pass) {
          const uint64_t st8 = S.ring[slot];
          const int cand = st_pred(uint32_t(st8) & 0xffffu, (uint32_t(st8) >> 16) & 0xffffu,
                                   uint32_t(st8 >> 32) & 0xffu, P - W);
          pass = cand >= max(P - A + 1, ls + 1);
        }
        const int64_t sph = spbase + P;
        if (kEither && !pass)
          pass = has_successor(stream, sph, q, S.qc, S.b62, lq, W, A, a.threshold);
        S.pflag[s + S.rank[idx]] = pass;
        if (maxp == prel) S.rec[idx] = r | kOwnerBit;  // the bin's rightmost hit owns it
        if (kTrace) {
          trace_push(a, 0, sph, q, 0, 0, 0);
          if (pass) trace_push(a, 1, sph, q, 0, 0, 0);
          st.add(kStatHits, 1);
          st.add(kStatPassing, pass);
        }
      }
      pbar(NP);
      // ---- (I) bin owners: ring update + hand-off of passing hits in s order ---
      for (uint32_t idx = ptid; idx < H; idx += NPT) {
        const uint32_t r = S.rec[idx];
        if (!(r & kOwnerBit)) continue;
        const int bin = int((r & ~kOwnerBit) >> 11), prel = int(r & 0x7ffu);
        const uint32_t s = S.cnt[bin], e = S.cnt[bin + 1];
        int slot = base_slot + bin;
        slot -= (slot >= M) ? M : 0;
        const int P = win + prel;
        // new state: last = P; near = hits in (P-W, P); far = largest <= P-W
        const uint64_t old = S.ring[slot];
        const uint32_t olast = uint32_t(old) & 0xffffu, ofar = (uint32_t(old) >> 16) & 0xffffu,
                       onear = uint32_t(old >> 32) & 0xffu;
        const unsigned reach_now = S.reach[slot];
        if (e - s == 1) {  // single-hit bin: append to the old state, hand off
          uint32_t last = olast, far = ofar, near = onear;
          st_append(last, far, near, P, W, nearmask);
          S.ring[slot] = uint64_t(last | (far << 16)) | (uint64_t(near) << 32);
          const unsigned vp = vbase + unsigned(P);
          if (S.pflag[s] && vp > reach_now) {
            if (kTrace) st.add(kStatEnqueued, 1);
            fifo_push(c, S, slot, vp, unsigned(spbase + P), prel - bin + lq - 1);
          }
          continue;
        }
        uint32_t nnear = 0, nfar = 0;
        int npass = 0;
        auto add = [&](int x) {
          if (x <= 0) return;
          const int d = P - x;
          if (d >= W) nfar = max(nfar, uint32_t(x));
          else if (d >= 1) nnear |= 1u << d;
        };
        if (olast) {
          add(int(olast));
          for (uint32_t m = onear; m; m &= m - 1) add(int(olast) - (__ffs(m) - 1));
          add(int(ofar));
        }
        for (uint32_t j = s; j < e; ++j) {
          add(win + int(S.bucketed[j]));
          npass += S.pflag[j];
        }
        S.ring[slot] = uint64_t(uint32_t(P) | (nfar << 16)) | (uint64_t(nnear) << 32);
        // passing hits of the bin, ascending s, not covered by a resolved reach
        int prev = -1;
        for (int it = 0; it < npass; ++it) {
          int best = 0x7fffffff;
          for (uint32_t j = s; j < e; ++j) {
            const int p = S.bucketed[j];
            if (S.pflag[j] && p > prev && p < best) best = p;
          }
          if (best == 0x7fffffff) break;
          prev = best;
          const int Pb = win + best;
          const unsigned vp = vbase + unsigned(Pb);
          if (vp > reach_now) {
            if (kTrace) st.add(kStatEnqueued, 1);
            fifo_push(c, S, slot, vp, unsigned(spbase + Pb), best - bin + lq - 1);
          }
        }
      }
      pbar(NP);
      // ---- (J) clear the bin counters ------------------------------------------
      for (int i = ptid; i <= c.nb; i += NPT) S.cnt[i] = 0;
    }
    // ---- advance the window ---------------------------------------------------
    if (ptid == 0) {
      const int used = ngroups ? ngroups : 1;
      unsigned nzm = 0;
      for (int g = 0; g < used; ++g)
        if (S.gsent[g]) nzm |= 1u << g;
      if (nzm) {
        const int g = 31 - __clz(nzm);
        C.lastsent = win + 32 * g + 31 - __clz(S.gsent[g]);
      }
      C.win = win + 32 * used;
      int bs = base_slot + 32 * used;
      while (bs >= M) bs -= M;
      C.base_slot = bs;
      if (int64_t(C.win) >= end) {
        C.have_chunk = 0;
        C.win += 64;  // gap before the next chunk's frame
        C.base_slot = (C.base_slot + 64) % M;
      }
    }
    pbar(NP);
  }
  st.flush(a);  // producer counters are per thread
}

template <bool kTrace, bool kEither, typename OffT>
__global__ void __launch_bounds__(kThreads, 1) search_cta_kernel(const SearchArgs a,
                                                                 const CtaConfig c) {
  extern __shared__ __align__(16) uint8_t smem[];
  size_t off[16];
  smem_layout(c, a.qv.lq, a.table_entries, off);
  Smem S;
  S.b62 = reinterpret_cast<int8_t *>(smem + off[0]);
  S.qc = smem + off[1];
  uint16_t *woff_s = reinterpret_cast<uint16_t *>(smem + off[2]);
  const int nwp = (kWords + 1 + 7) & ~7;
  S.woff16 = woff_s;
  S.qpos = woff_s + nwp;
  S.ring = reinterpret_cast<uint64_t *>(smem + off[3]);
  S.reach = reinterpret_cast<unsigned int *>(smem + off[4]);
  S.rec = reinterpret_cast<uint32_t *>(smem + off[5]);
  S.rank = reinterpret_cast<uint16_t *>(smem + off[6]);
  S.bucketed = reinterpret_cast<uint16_t *>(smem + off[7]);
  S.pflag = smem + off[8];
  S.cnt = reinterpret_cast<uint32_t *>(smem + off[9]);
  uint32_t *g = reinterpret_cast<uint32_t *>(smem + off[10]);
  S.gtot = g;
  S.gsent = g + 32;
  S.gcarry = reinterpret_cast<int *>(g + 64);
  S.scan_tmp = g + 96;
  S.gO = g + 128;
  S.gC = g + 160;
  S.posI = reinterpret_cast<uint32_t *>(smem + off[15]);
  S.posO = S.posI + c.nmax;
  S.ctrl = reinterpret_cast<Ctrl *>(smem + off[11]);
  S.fifo = reinterpret_cast<uint4 *>(smem + off[12]);
  S.ftail = reinterpret_cast<unsigned int *>(smem + off[13]);
  S.fhead = S.ftail + c.nc;
  S.fs = reinterpret_cast<int *>(smem + off[14]);

  const int tid = threadIdx.x, lq = a.qv.lq;
  for (int i = tid; i < 1024; i += kThreads) S.b62[i] = c_b62[i];
  const int qcb = int(align16(size_t(lq) + 2 * kQPad + 8));
  for (int i = tid; i < qcb; i += kThreads) {
    const int k = i - kQPad;
    S.qc[i] = (k >= 0 && k < lq) ? a.qv.qcodes[k] : uint8_t(kSentinel);
  }
  if (c.smem_table) {
    const uint32_t entries = uint32_t(a.table_entries);
    for (int i = tid; i < kWords + 1; i += kThreads) woff_s[i] = uint16_t(__ldg(a.qv.woff + i));
    for (uint32_t i = tid; i < entries; i += kThreads)
      const_cast<uint16_t *>(S.qpos)[i] = __ldg(a.qv.qpos + i);
  }
  for (int i = tid; i < c.M; i += kThreads) {
    S.ring[i] = 0;
    S.reach[i] = 0;
  }
  for (int i = tid; i <= c.nb; i += kThreads) S.cnt[i] = 0;
  for (int i = tid; i < c.nc * c.qcap; i += kThreads) S.fifo[i] = make_uint4(0, 0, 0, 0);
  if (tid < c.nc) {
    S.ftail[tid] = 0;
    S.fhead[tid] = 0;
  }
  if (tid == 0) {
    Ctrl &C = *S.ctrl;
    C.spbase = 0;
    C.end = 0;
    C.vbase = 0;
    C.win = kFrameMin;
    C.lastsent = kFrameMin - 1;
    C.base_slot = 0;
    C.have_chunk = 0;
    C.done = 0;
  }
  __syncthreads();

  const int warp = tid >> 5, lane = tid & 31;
  if (warp < c.np) {
    const OffT *woff;
    const uint16_t *qpos;
    if constexpr (sizeof(OffT) == 2) {
      woff = reinterpret_cast<const OffT *>(S.woff16);
      qpos = S.qpos;
    } else {
      woff = reinterpret_cast<const OffT *>(a.qv.woff);
      qpos = a.qv.qpos;
    }
    producer<kTrace, kEither, OffT>(a, c, S, woff, qpos, warp, lane);
    pbar(c.np);
    if (warp == 0 && lane == 0) {
      __threadfence_block();
      *reinterpret_cast<volatile int *>(&S.ctrl->done) = 1;
    }
  } else if (warp < c.np + c.nc) {
    consumer<kTrace>(a, c, S, warp - c.np, lane);
  }
}

template <bool kTrace, bool kEither, typename OffT>
cudaError_t launch_variant(const SearchArgs &a, const CtaConfig &c, size_t smem, int num_sms,
                           cudaStream_t s) {
  auto k = search_cta_kernel<kTrace, kEither, OffT>;
  cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
  if (e != cudaSuccess) return e;
  int grid = num_sms;
  const int items = a.nchunks + a.nlong;
  if (grid > items) grid = items < 1 ? 1 : items;
  k<<<unsigned(grid), kThreads, smem, s>>>(a, c);
  return cudaGetLastError();
}

// 0: pick automatically, 1: force the warp variant, 2: force the CTA variant
int kernel_choice() {
  const char *v = std::getenv("BLASTP_KERNEL");
#ifdef BLASTP_DEFAULT_WARP  // A/B builds: the warp kernel by default
  if (!v) return 1;
#endif
  if (!v) return 0;
  if (!std::strcmp(v, "warp")) return 1;
  if (!std::strcmp(v, "cta")) return 2;
  if (!std::strcmp(v, "block")) return 3;
  return 0;
}

}  // namespace

cudaError_t launch_search(const SearchArgs &a_in, int num_sms, cudaStream_t s) {
  // Default: the block kernel (search_block.cu) where its state encoding
  // applies (filter LEFT, ext_mode DIAGONAL/HIT, window >= 31 + min_gap),
  // else the warp kernel; BLASTP_KERNEL=warp|cta|block forces a variant
  // (block falls back to warp outside its domain; tests cover all three).
  const int choice = kernel_choice();
  if ((choice == 0 || choice == 3) && block_kernel_eligible(a_in))
    return launch_search_block(a_in, num_sms, s);
  if (choice != 2 || a_in.filter_mode == BLASTP_FILTER_STATEFUL ||
      a_in.filter_mode == BLASTP_FILTER_STATEFUL_RB)
    return launch_search_warp(a_in, num_sms, s);  // STATEFUL: warp variant only
  static unsigned long long b62_ready = 0;  // one bit per device
  int dev = 0;
  cudaGetDevice(&dev);
  int optin = 0;
  cudaError_t e = cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  if (e != cudaSuccess) return e;
  SearchArgs a = a_in;
  a.nsegs = 0;  // no segment pipeline: long items are walked whole
  CtaConfig c{};
  c.np = 24;
  c.nc = 8;
  // E1 knobs (the paper's bins-per-warp sweep):
  // producer / consumer warps; a window of 32 * np positions is binned into
  // 32 * np + Lq diagonal bins, i.e. (32 * np + Lq) / np bins per producer warp
  if (const char *v = std::getenv("BLASTP_CTA_NP")) c.np = std::max(1, std::min(31, std::atoi(v)));
  if (const char *v = std::getenv("BLASTP_CTA_NC")) c.nc = std::max(1, std::min(32 - c.np, std::atoi(v)));
  if (c.np + c.nc > 32) c.nc = 32 - c.np;
  c.nmax = 32 * c.np;
  c.cap = std::max(4096, 4096 * c.np / 24);
  c.nb = c.nmax + a.qv.lq;
  c.M = ((a.qv.lq + c.nmax + a.window + 64) + 31) & ~31;
  c.qcap = 256;
  c.smem_table = a.table_entries < 65536 ? 1 : 0;
  a.ring = c.M;
  size_t smem = smem_layout(c, a.qv.lq, a.table_entries, nullptr);
  if (smem > size_t(optin) && c.smem_table) {
    c.smem_table = 0;
    smem = smem_layout(c, a.qv.lq, a.table_entries, nullptr);
  }
  // the CTA variant addresses the shard with 32-bit stream positions
  const bool fits = smem <= size_t(optin) && a.stream_len < (int64_t(1) << 32) && c.M < 65536;
  if (!fits) {
    if (choice == 2) return cudaErrorInvalidConfiguration;
    return launch_search_warp(a_in, num_sms, s);
  }
  if (!(b62_ready >> dev & 1ull)) {
    int8_t h[32 * 32];
    fill_b62(h);
    e = cudaMemcpyToSymbol(c_b62, h, sizeof(h));
    if (e != cudaSuccess) return e;
    b62_ready |= 1ull << dev;
  }
  const bool trace = a.trace[0] != nullptr;
  const bool either = a.filter_mode == BLASTP_FILTER_EITHER;
  if (c.smem_table) {
    if (trace)
      return either ? launch_variant<true, true, uint16_t>(a, c, smem, num_sms, s)
                    : launch_variant<true, false, uint16_t>(a, c, smem, num_sms, s);
    return either ? launch_variant<false, true, uint16_t>(a, c, smem, num_sms, s)
                  : launch_variant<false, false, uint16_t>(a, c, smem, num_sms, s);
  }
  if (trace)
    return either ? launch_variant<true, true, uint32_t>(a, c, smem, num_sms, s)
                  : launch_variant<true, false, uint32_t>(a, c, smem, num_sms, s);
  return either ? launch_variant<false, true, uint32_t>(a, c, smem, num_sms, s)
                : launch_variant<false, false, uint32_t>(a, c, smem, num_sms, s);
}

}  // namespace blastp
