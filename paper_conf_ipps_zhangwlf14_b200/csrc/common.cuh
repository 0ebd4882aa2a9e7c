// common.cuh -- product-side constants and device structs of libblastp.so.
//
// This is the CUDA path's own copy of the alphabet (R1) and BLOSUM62 (R2);
// it shares nothing with oracle/ (the oracle has its own literal).
#pragma once

#include <cstdint>
#include <mutex>

#include <cuda_runtime.h>

#include "../../include/blastp.h"

namespace blastp {

// R1 alphabet: NCBI order; code = index.  Code 31 separates subjects in the
// packed stream ("sentinel"); codes 24..30 are never produced.
constexpr char kAlphabet[] = "ARNDCQEGHILKMFPSTWYVBZX*";
constexpr int kNumLetters = 24;
constexpr int kSentinel = 31;
constexpr int kWords = kNumLetters * kNumLetters * kNumLetters;  // 13824
// Scores involving a sentinel (or an unused code).  An extension that steps
// onto a sentinel drops by >= 128 - 11*2 > X (X <= 127 is validated), so the
// X-drop stops exactly at a subject boundary (R8 "end of either sequence").
constexpr int kSentinelScore = -128;

// Leading / trailing sentinel padding of the packed stream (bytes).
constexpr int64_t kStreamPadFront = 16;
constexpr int64_t kStreamPadBack = 2048;  // covers the 512-B staging prefetch

// NCBI BLOSUM62, order kAlphabet.
constexpr int8_t kBlosum62[kNumLetters][kNumLetters] = {
    {4, -1, -2, -2, 0, -1, -1, 0, -2, -1, -1, -1, -1, -2, -1, 1, 0, -3, -2, 0, -2, -1, 0, -4},
    {-1, 5, 0, -2, -3, 1, 0, -2, 0, -3, -2, 2, -1, -3, -2, -1, -1, -3, -2, -3, -1, 0, -1, -4},
    {-2, 0, 6, 1, -3, 0, 0, 0, 1, -3, -3, 0, -2, -3, -2, 1, 0, -4, -2, -3, 3, 0, -1, -4},
    {-2, -2, 1, 6, -3, 0, 2, -1, -1, -3, -4, -1, -3, -3, -1, 0, -1, -4, -3, -3, 4, 1, -1, -4},
    {0, -3, -3, -3, 9, -3, -4, -3, -3, -1, -1, -3, -1, -2, -3, -1, -1, -2, -2, -1, -3, -3, -2, -4},
    {-1, 1, 0, 0, -3, 5, 2, -2, 0, -3, -2, 1, 0, -3, -1, 0, -1, -2, -1, -2, 0, 3, -1, -4},
    {-1, 0, 0, 2, -4, 2, 5, -2, 0, -3, -3, 1, -2, -3, -1, 0, -1, -3, -2, -2, 1, 4, -1, -4},
    {0, -2, 0, -1, -3, -2, -2, 6, -2, -4, -4, -2, -3, -3, -2, 0, -2, -2, -3, -3, -1, -2, -1, -4},
    {-2, 0, 1, -1, -3, 0, 0, -2, 8, -3, -3, -1, -2, -1, -2, -1, -2, -2, 2, -3, 0, 0, -1, -4},
    {-1, -3, -3, -3, -1, -3, -3, -4, -3, 4, 2, -3, 1, 0, -3, -2, -1, -3, -1, 3, -3, -3, -1, -4},
    {-1, -2, -3, -4, -1, -2, -3, -4, -3, 2, 4, -2, 2, 0, -3, -2, -1, -2, -1, 1, -4, -3, -1, -4},
    {-1, 2, 0, -1, -3, 1, 1, -2, -1, -3, -2, 5, -1, -3, -1, 0, -1, -3, -2, -2, 0, 1, -1, -4},
    {-1, -1, -2, -3, -1, 0, -2, -3, -2, 1, 2, -1, 5, 0, -2, -1, -1, -1, -1, 1, -3, -1, -1, -4},
    {-2, -3, -3, -3, -2, -3, -3, -3, -1, 0, 0, -3, 0, 6, -4, -2, -2, 1, 3, -1, -3, -3, -1, -4},
    {-1, -2, -2, -1, -3, -1, -1, -2, -2, -3, -3, -1, -2, -4, 7, -1, -1, -4, -3, -2, -2, -1, -2, -4},
    {1, -1, 1, 0, -1, 0, 0, 0, -1, -2, -2, 0, -1, -2, -1, 4, 1, -3, -2, -2, 0, 0, 0, -4},
    {0, -1, 0, -1, -1, -1, -1, -2, -2, -1, -1, -1, -1, -2, -1, 1, 5, -2, -2, 0, -1, -1, 0, -4},
    {-3, -3, -4, -4, -2, -2, -3, -2, -2, -3, -2, -3, -1, 1, -4, -3, -2, 11, 2, -3, -4, -3, -2, -4},
    {-2, -2, -2, -3, -2, -1, -2, -3, 2, -1, -1, -2, -1, 3, -3, -2, -2, 2, 7, -1, -3, -2, -1, -4},
    {0, -3, -3, -3, -1, -2, -2, -3, -3, 3, 1, -2, 1, -1, -2, -2, 0, -3, -1, 4, -3, -2, -1, -4},
    {-2, -1, 3, 4, -3, 0, 1, -1, 0, -3, -4, 0, -3, -3, -2, 0, -1, -4, -3, -3, 4, 1, -1, -4},
    {-1, 0, 0, 1, -3, 3, 4, -2, 0, -3, -3, 1, -1, -3, -1, 0, -1, -3, -2, -2, 1, 4, -1, -4},
    {0, -1, -1, -1, -2, -1, -1, -1, -1, -1, -1, -1, -1, -1, -2, 0, 0, -2, -1, -1, -1, -1, -1, -4},
    {-4, -4, -4, -4, -4, -4, -4, -4, -4, -4, -4, -4, -4, -4, -4, -4, -4, -4, -4, -4, -4, -4, -4, 1},
};

// A contiguous range of whole subjects searched by one warp.  Positions are
// byte offsets in the packed stream; stream[start-1] and stream[end] are
// sentinels.  Subjects [first_subj, last_subj) (shard-local indices).
struct Chunk {
  int64_t start, end;
  int64_t first_subj, last_subj;
};

// A chunk longer than 2C (it ends in a long subject), scheduled before the
// regular chunks.  With nseg > 0 the warp variant splits it (DESIGN.md "Long
// subjects"): segment k covers emit positions [start + k*seg_len, +seg_len)
// and is two-hit filtered by its own warp after a `window`-position warm-up,
// writing its passing hits to a list; one walker warp then feeds the lists,
// in s order, through extension and the ext_reach chain.  nseg == 0: the
// chunk is walked whole by one warp.
struct LongItem {
  Chunk c;
  int32_t seg0, nseg;  // segments [seg0, seg0 + nseg) of the segment arrays
  int64_t pad;
};

// Trace record (debug entry points only): stream position of the hit /
// seed, query position, and for extensions llen/rlen/score.
struct TraceRec {
  int64_t sp;
  int32_t q, llen, rlen, score, query_id, pad;
};

// Per-query device view of a lookup table (R3): CSR word -> query positions.
struct QueryView {
  const uint32_t *woff;   // [kWords + 1]
  const uint2 *wtab;      // [32^3] radix-32 code -> (woff, count) (table.cu)
  const uint16_t *qpos;   // [entries], ascending within a word
  const uint8_t *qcodes;  // [lq] query codes
  int32_t lq, query_id;
  // a query group (nsub >= 2): member k starts at combined position sub[k]
  // and is batch query sub[nsub + k]; 0 for a single query
  int32_t nsub;
  const int32_t *sub;
};

struct SearchArgs {
  const uint8_t *stream;
  const int64_t *sstart;  // [nseq]: stream position of each subject's first residue
  int64_t nseq;           // subjects of the shard
  int64_t stream_len;     // bytes of the packed stream
  int64_t subject_base;
  const Chunk *chunks;
  int32_t nchunks;
  // Work items of the chunk cursor, in order: segments [0, nsegs) (warp
  // variant only), long items [0, nlong), regular chunks [0, nchunks).
  const LongItem *long_items;
  int32_t nlong;
  int32_t nsegs;               // 0: no segment pipeline
  const int32_t *seg_item;     // [nsegs] long item of each segment
  uint32_t *seg_list;          // [nsegs * seg_cap] passing hits: (s - emit) | q << 16
  int32_t *seg_count;          // [nsegs] list length, -1 = overflow
  unsigned *seg_done;          // [nsegs] == seq once the segment's list is published
  int32_t seg_len, seg_cap;
  unsigned seq;                // launch sequence number of this search
  QueryView qv;
  int32_t word_len, threshold, window, min_gap, xdrop, cutoff, filter_mode;
  int32_t ext_mode;  // BLASTP_EXT_DIAGONAL (Alg. 3 ext_reach chain) / BLASTP_EXT_HIT (Alg. 4)
  int32_t ring;      // M: per-warp diagonal ring slots
  int64_t table_entries;  // CSR entries of the query table (positions)
  blastp_hsp *out;
  int64_t out_cap;
  unsigned long long *hsp_count;     // one counter
  unsigned long long *chunk_cursor;  // work-stealing cursor
  TraceRec *trace[3];                // hits, passing, extensions (or null)
  int64_t trace_cap[3];
  unsigned long long *trace_count;   // [3]
  unsigned long long *stats;         // [kNumStats] event counters (trace runs only)
  int32_t emit_seed;                 // ext_mode HIT_DEDUP: every extension as a seed record
  int32_t out_fence;                 // blastp_search_ungapped_append: out may be peer memory
  const int8_t *pssm;                // block kernel, BLASTP_SCORE=pssm_global: the PSSM
  uint16_t *reach_scratch;           // block kernel: per-warp ext_reach regions (launch-owned)
};

// Event counters collected by the tracing kernel variant (blastp_debug_stats).
enum StatIndex {
  kStatIterations = 0,   // 32-position windows
  kStatRounds,           // 32-hit rounds
  kStatConflictRounds,   // rounds with >= 2 hits on one diagonal
  kStatHits,             // hits (R4)
  kStatPassing,          // hits passing the two-hit test (R6)
  kStatEnqueued,         // passing hits not covered at enqueue time
  kStatFlushes,          // extension batches
  kStatExtended,         // extensions computed (speculative included)
  kStatAccepted,         // extensions accepted by the ext_reach chain (R10)
  kStatEmitted,          // HSPs with score >= cutoff
  kStatXdropSteps,       // residues scored by X-drop (both sides, all lanes)
  kStatXdropLaneSlots,   // lanes x steps of the X-drop loops (utilisation)
  kNumStats = 16
};

// Stream-ordered device allocations of the library come from its own memory
// pool per device (created on first use, release threshold = keep
// everything), so repeated pack / search / format calls do not pay cudaMalloc
// again -- without changing the device's default pool, which belongs to the
// caller (PyTorch and others allocate from it).  Freed with cudaFreeAsync.
struct LibPools {
  cudaMemPool_t pools[64] = {};
  std::mutex mu;
};
inline LibPools &lib_pools() {
  static LibPools p;
  return p;
}
inline cudaError_t pool_malloc_async(void **ptr, size_t bytes, cudaStream_t s) {
  cudaMemPool_t *pools = lib_pools().pools;
  std::mutex &mu = lib_pools().mu;
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if (dev < 0 || dev >= 64) return cudaMallocAsync(ptr, bytes, s);
  std::lock_guard<std::mutex> lock(mu);
  if (!pools[dev]) {
    cudaMemPoolProps props = {};
    props.allocType = cudaMemAllocationTypePinned;
    props.location.type = cudaMemLocationTypeDevice;
    props.location.id = dev;
    cudaMemPool_t pool;
    if ((e = cudaMemPoolCreate(&pool, &props)) != cudaSuccess) return e;
    uint64_t thr = ~uint64_t(0);
    cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
    pools[dev] = pool;
  }
  return cudaMallocFromPoolAsync(ptr, bytes, pools[dev], s);
}
// Returns the memory the library's pool of `device` holds to the device
// (blastp_trim_memory); allocations still alive are kept.
inline cudaError_t pool_trim(int device) {
  if (device < 0 || device >= 64) return cudaSuccess;
  std::lock_guard<std::mutex> lock(lib_pools().mu);
  cudaMemPool_t pool = lib_pools().pools[device];
  if (!pool) return cudaSuccess;
  cudaError_t e = cudaDeviceSynchronize();
  return e == cudaSuccess ? cudaMemPoolTrimTo(pool, 0) : e;
}
template <typename T>
inline cudaError_t pool_malloc_async(T **ptr, size_t bytes, cudaStream_t s) {
  return pool_malloc_async(reinterpret_cast<void **>(ptr), bytes, s);
}

// Launch helpers implemented in search.cu / pack.cu / sort.cu.
int search_ring_slots(int lq, int window);
// Picks the kernel variant (search_cta.cu, else search.cu); the environment
// variable BLASTP_KERNEL=warp|cta forces one (tests cover both).
cudaError_t launch_search(const SearchArgs &a, int num_sms, cudaStream_t s);
cudaError_t launch_search_warp(const SearchArgs &a, int num_sms, cudaStream_t s);
// The block kernel (search_block.cu), default for filter_mode LEFT with
// ext_mode DIAGONAL/HIT when window >= 31 + min_gap (block_kernel_eligible).
bool block_kernel_eligible(const SearchArgs &a);
cudaError_t launch_search_block(const SearchArgs &a, int num_sms, cudaStream_t s);
// Query lookup table on the GPU (table.cu): woff (kWords + 1) from the query
// codes, the entry count returned on the host (synchronises s), then qpos.
cudaError_t launch_table_count(const uint8_t *qcodes, int lq, int T, uint32_t *woff,
                               int64_t *total, cudaStream_t s);
cudaError_t launch_table_radix32(const uint32_t *woff, uint2 *wtab, cudaStream_t s);
cudaError_t launch_table_fill(const uint8_t *qcodes, int lq, int T, const uint32_t *woff,
                              uint16_t *qpos, cudaStream_t s);
cudaError_t launch_pack(const uint8_t *ascii, const int64_t *off, int64_t n,
                        const int64_t *sstart, uint8_t *stream, int64_t stream_len, int *err,
                        cudaStream_t s);
// Chunk plan: chunk k covers the subjects whose first residue lies in
// [target(k), target(k+1)) of the shard's residues; chunks [0, K1) are C
// residues apart, the rest (the last ~2 chunks' worth per resident warp) Ct =
// C/4 apart, so the tail of a launch -- warps finishing their last chunk --
// is a fraction of a small chunk.
struct ChunkPlan {
  int64_t C, Ct, K1, nchunks;
};
__host__ __device__ inline int64_t chunk_target(const ChunkPlan &p, int64_t k) {
  return k < p.K1 ? k * p.C : p.K1 * p.C + (k - p.K1) * p.Ct;
}
cudaError_t launch_layout(const int64_t *off, int64_t n, const ChunkPlan &plan, int64_t *sstart,
                          Chunk *chunks, Chunk *long_chunks, int *nlong, int *err,
                          cudaStream_t s);
// Segment length / list capacity of the long-item pipeline.
constexpr int kSegLen = 2048;
constexpr int kSegCap = 2048;
constexpr int kMaxSegments = 32768;  // 256 MB of lists at most
// Gapped-extension consumer (gapped.cu, R18-R22).
struct GappedArgs {
  const blastp_hsp *hsps;  // canonical order (R11), n records
  int64_t n;
  const uint8_t *const *qcodes;  // device: codes of batch query k
  const int32_t *qlens;          // device
  int32_t nq;
  const uint8_t *stream;  // packed shard: subject i at stream[sstart[i]]
  const int64_t *sstart;
  int64_t nseq, subject_base, stream_end, max_subject_len;
  int32_t gap_open, gap_extend, xdrop, cutoff;
};
cudaError_t launch_gapped(const GappedArgs &a, int num_sms, blastp_gapped *d_out, int64_t cap,
                          int64_t *h_count, int *h_err, cudaStream_t s);
cudaError_t measure_alu_peak(double *lane_ops_per_s);  // micro.cu
cudaError_t sort_hsps(blastp_hsp *d, int64_t n, cudaStream_t s);
cudaError_t unique_hsps(blastp_hsp *d, int64_t n, int64_t *d_n_out, cudaStream_t s);
cudaError_t dedup_covered(blastp_hsp *d, int64_t n, int32_t cutoff, int64_t *d_n_out,
                          cudaStream_t s);
void upload_encode_table();

}  // namespace blastp
