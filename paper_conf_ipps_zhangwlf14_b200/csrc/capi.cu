// capi.cu -- the extern "C" boundary of libblastp.so (include/blastp.h).
//
// Host logic only: argument validation, the query lookup-table builder (R3),
// the database packer / sharder, launch drivers and result marshalling.
// Every step of the search itself runs in the kernels of search.cu.
#include <algorithm>
#include <chrono>
#include <cstdarg>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <limits>
#include <string>
#include <type_traits>
#include <vector>

#include <cuda_runtime.h>

#include "common.cuh"

using namespace blastp;

// ------------------------------------------------------------------ errors

namespace {

thread_local std::string g_last_error;

int fail(int code, const char *fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  g_last_error = buf;
  return code;
}

#define CUDA_TRY(expr)                                                                    \
  do {                                                                                    \
    cudaError_t _e = (expr);                                                              \
    if (_e != cudaSuccess)                                                                \
      return fail(BLASTP_E_CUDA, "%s failed: %s (%s:%d)", #expr, cudaGetErrorString(_e), \
                  __FILE__, __LINE__);                                                    \
  } while (0)

struct DeviceGuard {
  int prev = -1;
  cudaError_t err = cudaSuccess;
  explicit DeviceGuard(int dev) {
    cudaGetDevice(&prev);
    if (prev != dev) err = cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    if (prev >= 0) cudaSetDevice(prev);
  }
};

// R1 encoding (host side, for queries)
int encode_char(unsigned char c) {
  if (c >= 'a' && c <= 'z') c = static_cast<unsigned char>(c - 'a' + 'A');
  if (c == 'U' || c == 'O' || c == 'J') c = 'X';
  for (int k = 0; k < kNumLetters; ++k)
    if (static_cast<unsigned char>(kAlphabet[k]) == c) return k;
  return -1;
}

int validate_params(const blastp_params *p) {
  if (!p) return fail(BLASTP_E_INVALID_ARG, "params is NULL");
  if (p->word_len != 3) return fail(BLASTP_E_INVALID_ARG, "word_len %d unsupported (3 only)", p->word_len);
  if (p->min_gap < 1 || p->min_gap > 8)
    return fail(BLASTP_E_INVALID_ARG, "min_gap %d outside [1, 8]", p->min_gap);
  if (p->window < 1 || p->window > 256)
    return fail(BLASTP_E_INVALID_ARG, "window %d outside [1, 256]", p->window);
  if (p->xdrop < 1 || p->xdrop > 127)
    return fail(BLASTP_E_INVALID_ARG, "xdrop %d outside [1, 127]", p->xdrop);
  if (p->threshold < -100 || p->threshold > 100)
    return fail(BLASTP_E_INVALID_ARG, "threshold %d outside [-100, 100]", p->threshold);
  if (p->filter_mode != BLASTP_FILTER_LEFT && p->filter_mode != BLASTP_FILTER_EITHER &&
      p->filter_mode != BLASTP_FILTER_STATEFUL && p->filter_mode != BLASTP_FILTER_STATEFUL_RB)
    return fail(BLASTP_E_INVALID_ARG, "filter_mode %d unknown", p->filter_mode);
  if ((p->filter_mode == BLASTP_FILTER_STATEFUL || p->filter_mode == BLASTP_FILTER_STATEFUL_RB) &&
      p->ext_mode != BLASTP_EXT_DIAGONAL)
    return fail(BLASTP_E_INVALID_ARG, "filter_mode STATEFUL decides coverage itself: ext_mode "
                "must be DIAGONAL (got %d)", p->ext_mode);
  if (p->ext_mode != BLASTP_EXT_DIAGONAL && p->ext_mode != BLASTP_EXT_HIT &&
      p->ext_mode != BLASTP_EXT_WINDOW && p->ext_mode != BLASTP_EXT_HIT_DEDUP)
    return fail(BLASTP_E_INVALID_ARG, "ext_mode %d unknown", p->ext_mode);
  return BLASTP_OK;
}

int num_sms(int device) {
  int sms = 0;
  if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device) != cudaSuccess ||
      sms <= 0)
    sms = 148;
  return sms;
}

}  // namespace

// ------------------------------------------------------------------ handles

struct QueryDev {
  uint32_t *woff = nullptr;
  uint2 *wtab = nullptr;  // radix-32 view of woff (launch_table_radix32)
  uint16_t *qpos = nullptr;
  uint8_t *qcodes = nullptr;
  int32_t lq = 0;
  int64_t entries = 0;
  // a group of queries searched as one: the member
  // queries' codes concatenated with sentinel gaps; member k starts at
  // combined position sub_off[k] and is query sub_id[k] of the batch
  int32_t nsub = 0;
  int32_t *sub = nullptr;  // device: sub_off[nsub], then sub_id[nsub]
};

struct blastp_query_table {
  int device = 0;
  blastp_params p{};
  std::vector<QueryDev> q;
  int64_t entries = 0;
  // query groups of a batch and the queries left alone (indices into q)
  std::vector<QueryDev> groups;
  std::vector<int32_t> alone;
  int32_t group_gap = 0;  // sentinel positions between the members of a group
};

struct blastp_db {
  int device = 0;
  int sms = 148;
  int64_t nseq = 0, residues = 0, subject_base = 0, stream_len = 0;
  uint8_t *stream = nullptr;
  int64_t *sstart = nullptr;
  Chunk *chunks = nullptr;
  Chunk *long_chunks = nullptr;  // chunks > 2C residues (count at counters[6]), pack only
  int32_t nchunks = 0;
  // long items, longest first, and their segments
  LongItem *items = nullptr;
  int32_t nlong = 0, nsegs = 0, seg_len = kSegLen, seg_cap = kSegCap;
  int32_t *seg_item = nullptr, *seg_count = nullptr;
  uint32_t *seg_list = nullptr;
  unsigned *seg_done = nullptr;
  unsigned seq = 0;  // search launches on this db (segment publication epoch)
  bool carved = false;  // stream/sstart/chunks/counters live in a caller's arena
  std::vector<int64_t> h_sstart;
  int64_t max_len = -1;  // longest subject (the gapped stage's big-ring width), computed once
  unsigned long long *counters = nullptr;  // [0] hsp count, [1] chunk cursor, [6] long chunks
  blastp_hsp *out = nullptr;               // scratch for the host-array search
  int64_t out_cap = 0;
};

// Long items (chunks > 2C, i.e. ending in a long subject), longest first;
// those longer than 2 segments are split into segments (DESIGN.md "Long
// subjects") while the segment budget lasts.  Knobs for tests/experiments:
// BLASTP_SEGMENTS=0 (off), BLASTP_SEGLEN (256..16384; >= the largest window A
// so a segment's warm-up stays inside its chunk), BLASTP_SEGCAP.
static cudaError_t plan_long_items(blastp_db *db, int nlong, cudaStream_t s) {
  std::vector<Chunk> lc(static_cast<size_t>(nlong));
  cudaError_t e = cudaMemcpyAsync(lc.data(), db->long_chunks, sizeof(Chunk) * lc.size(),
                                  cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return e;
  std::sort(lc.begin(), lc.end(), [](const Chunk &x, const Chunk &y) {
    const int64_t lx = x.end - x.start, ly = y.end - y.start;
    return lx != ly ? lx > ly : x.start < y.start;
  });
  const char *on = std::getenv("BLASTP_SEGMENTS");
  const bool enabled = !(on && std::atoi(on) == 0);
  if (const char *v = std::getenv("BLASTP_SEGLEN")) db->seg_len = std::max(256, std::min(16384, std::atoi(v)));
  if (const char *v = std::getenv("BLASTP_SEGCAP")) db->seg_cap = std::max(1, std::atoi(v));
  std::vector<LongItem> items(lc.size());
  std::vector<int32_t> seg_item;
  for (size_t i = 0; i < lc.size(); ++i) {
    LongItem &it = items[i];
    it = LongItem{};
    it.c = lc[i];
    const int64_t len = lc[i].end - lc[i].start;
    const int64_t nseg = (len + db->seg_len - 1) / db->seg_len;
    if (enabled && len > 2 * int64_t(db->seg_len) &&
        int64_t(seg_item.size()) + nseg <= kMaxSegments) {
      it.seg0 = static_cast<int32_t>(seg_item.size());
      it.nseg = static_cast<int32_t>(nseg);
      seg_item.insert(seg_item.end(), static_cast<size_t>(nseg), static_cast<int32_t>(i));
    }
  }
  db->nlong = nlong;
  db->nsegs = static_cast<int32_t>(seg_item.size());
  const size_t ns = std::max<size_t>(seg_item.size(), 1);
  if ((e = pool_malloc_async(&db->items, sizeof(LongItem) * items.size(), s)) != cudaSuccess) return e;
  if ((e = pool_malloc_async(&db->seg_item, sizeof(int32_t) * ns, s)) != cudaSuccess) return e;
  if ((e = pool_malloc_async(&db->seg_count, sizeof(int32_t) * ns, s)) != cudaSuccess) return e;
  if ((e = pool_malloc_async(&db->seg_done, sizeof(unsigned) * ns, s)) != cudaSuccess) return e;
  if ((e = pool_malloc_async(&db->seg_list, sizeof(uint32_t) * ns * size_t(db->seg_cap), s)) != cudaSuccess)
    return e;
  if ((e = cudaMemcpyAsync(db->items, items.data(), sizeof(LongItem) * items.size(),
                           cudaMemcpyHostToDevice, s)) != cudaSuccess)
    return e;
  if (!seg_item.empty() &&
      (e = cudaMemcpyAsync(db->seg_item, seg_item.data(), sizeof(int32_t) * seg_item.size(),
                           cudaMemcpyHostToDevice, s)) != cudaSuccess)
    return e;
  if ((e = cudaMemsetAsync(db->seg_done, 0, sizeof(unsigned) * ns, s)) != cudaSuccess) return e;
  return cudaStreamSynchronize(s);  // the host vectors die here
}

static void free_query_dev(QueryDev &d) {
  cudaFree(d.woff);
  cudaFree(d.wtab);
  cudaFree(d.qpos);
  cudaFree(d.qcodes);
  cudaFree(d.sub);
  d = QueryDev{};
}

extern "C" {

void blastp_params_default(blastp_params *p) {
  if (!p) return;
  p->word_len = 3;
  p->threshold = 11;
  p->window = 40;
  p->min_gap = 3;
  p->xdrop = 16;
  p->cutoff = 41;
  p->filter_mode = BLASTP_FILTER_LEFT;
  p->ext_mode = BLASTP_EXT_DIAGONAL;
}

const char *blastp_strerror(int status) {
  switch (status) {
    case BLASTP_OK: return "ok";
    case BLASTP_E_INVALID_ARG: return "invalid argument";
    case BLASTP_E_BAD_RESIDUE: return "invalid residue character";
    case BLASTP_E_TOO_LONG: return "sequence too long";
    case BLASTP_E_NOMEM: return "out of memory";
    case BLASTP_E_CUDA: return "CUDA error";
    case BLASTP_E_CAPACITY: return "output capacity exceeded";
    default: return "unknown status";
  }
}

const char *blastp_last_error(void) { return g_last_error.c_str(); }

const char *blastp_version(void) { return "blastp-b200 0.1 (sm_100a)"; }

// ------------------------------------------------------- query table (R3)

static int encode_query(const char *ascii, int32_t len, std::vector<uint8_t> &Q) {
  if (!ascii) return fail(BLASTP_E_INVALID_ARG, "query is NULL");
  if (len < 3) return fail(BLASTP_E_INVALID_ARG, "query length %d < 3", len);
  if (len > BLASTP_MAX_QUERY_LEN)
    return fail(BLASTP_E_TOO_LONG, "query length %d > %d", len, BLASTP_MAX_QUERY_LEN);
  Q.resize(static_cast<size_t>(len));
  for (int32_t i = 0; i < len; ++i) {
    const int c = encode_char(static_cast<unsigned char>(ascii[i]));
    if (c < 0) return fail(BLASTP_E_BAD_RESIDUE, "query byte %d (0x%02x) is not a residue", i,
                           static_cast<unsigned char>(ascii[i]));
    Q[static_cast<size_t>(i)] = static_cast<uint8_t>(c);
  }
  return BLASTP_OK;
}

// Lookup table (R3) of the query codes Q (a query, or a group's members
// separated by sentinel codes: a word touching a sentinel scores -1000 per
// sentinel letter and neighbours nothing).
// The radix-32 (start, count) view the block kernel reads (table.cu).
static int finish_table(QueryDev &out, cudaStream_t s) {
  if (pool_malloc_async(&out.wtab, sizeof(uint2) * 32 * 32 * 32, s) != cudaSuccess) {
    cudaGetLastError();
    free_query_dev(out);
    return fail(BLASTP_E_NOMEM, "device allocation for the query table failed");
  }
  CUDA_TRY(launch_table_radix32(out.woff, out.wtab, s));
  CUDA_TRY(cudaStreamSynchronize(s));
  return BLASTP_OK;
}

static int build_table(const std::vector<uint8_t> &Q, const blastp_params *p, QueryDev &out,
                       cudaStream_t s) {
  const int32_t len = static_cast<int32_t>(Q.size());
  out.lq = len;
  const char *how = std::getenv("BLASTP_TABLE_BUILD");  // "host": the host enumeration below
  if (!(how && !std::strcmp(how, "host"))) {
    // GPU build (table.cu): one thread per word counts, scans, fills
    if (pool_malloc_async(&out.woff, sizeof(uint32_t) * (kWords + 1), s) != cudaSuccess ||
        pool_malloc_async(&out.qcodes, static_cast<size_t>(len) + 16, s) != cudaSuccess) {
      cudaGetLastError();
      free_query_dev(out);
      return fail(BLASTP_E_NOMEM, "device allocation for the query table failed");
    }
    CUDA_TRY(cudaMemcpyAsync(out.qcodes, Q.data(), Q.size(), cudaMemcpyHostToDevice, s));
    int64_t total = 0;
    CUDA_TRY(launch_table_count(out.qcodes, len, p->threshold, out.woff, &total, s));
    out.entries = total;
    if (pool_malloc_async(&out.qpos, sizeof(uint16_t) * size_t(std::max<int64_t>(total, 1)), s) !=
        cudaSuccess) {
      cudaGetLastError();
      free_query_dev(out);
      return fail(BLASTP_E_NOMEM, "device allocation for the query table failed");
    }
    CUDA_TRY(launch_table_fill(out.qcodes, len, p->threshold, out.woff, out.qpos, s));
    return finish_table(out, s);
  }
  // Neighbourhood words by pruned enumeration: for each query word, walk the
  // 24^3 words letter by letter and cut a branch as soon as even the best
  // remaining letters cannot reach T.  Same set as the brute-force
  // definition (R3); lists come out with q ascending.
  int rowmax[kNumLetters];
  for (int a = 0; a < kNumLetters; ++a) {
    int m = -1000;
    for (int b = 0; b < kNumLetters; ++b) m = std::max(m, int(kBlosum62[a][b]));
    rowmax[a] = m;
  }
  const int T = p->threshold;
  std::vector<uint32_t> count(kWords + 1, 0);
  auto enumerate = [&](auto &&emit) {
    for (int32_t q = 0; q + 3 <= len; ++q) {
      const int a0 = Q[q], a1 = Q[q + 1], a2 = Q[q + 2];
      if (a0 >= kNumLetters || a1 >= kNumLetters || a2 >= kNumLetters) continue;  // group gap
      for (int x = 0; x < kNumLetters; ++x) {
        const int s1 = kBlosum62[a0][x];
        if (s1 + rowmax[a1] + rowmax[a2] < T) continue;
        for (int y = 0; y < kNumLetters; ++y) {
          const int s2 = s1 + kBlosum62[a1][y];
          if (s2 + rowmax[a2] < T) continue;
          for (int z = 0; z < kNumLetters; ++z)
            if (s2 + kBlosum62[a2][z] >= T) emit((x * kNumLetters + y) * kNumLetters + z, q);
        }
      }
    }
  };
  enumerate([&](int w, int) { count[static_cast<size_t>(w) + 1]++; });
  for (int w = 0; w < kWords; ++w) count[static_cast<size_t>(w) + 1] += count[static_cast<size_t>(w)];
  const int64_t total = count[kWords];
  std::vector<uint16_t> pos(static_cast<size_t>(std::max<int64_t>(total, 1)));
  std::vector<uint32_t> cur(count.begin(), count.end() - 1);
  enumerate([&](int w, int q) { pos[cur[static_cast<size_t>(w)]++] = static_cast<uint16_t>(q); });

  out.lq = len;
  out.entries = total;
  if (cudaMalloc(&out.woff, sizeof(uint32_t) * (kWords + 1)) != cudaSuccess ||
      cudaMalloc(&out.qpos, sizeof(uint16_t) * pos.size()) != cudaSuccess ||
      cudaMalloc(&out.qcodes, static_cast<size_t>(len) + 16) != cudaSuccess) {
    free_query_dev(out);
    return fail(BLASTP_E_NOMEM, "device allocation for the query table failed");
  }
  CUDA_TRY(cudaMemcpyAsync(out.woff, count.data(), sizeof(uint32_t) * (kWords + 1),
                           cudaMemcpyHostToDevice, s));
  CUDA_TRY(cudaMemcpyAsync(out.qpos, pos.data(), sizeof(uint16_t) * pos.size(),
                           cudaMemcpyHostToDevice, s));
  CUDA_TRY(cudaMemcpyAsync(out.qcodes, Q.data(), Q.size(), cudaMemcpyHostToDevice, s));
  return finish_table(out, s);  // synchronises: the host vectors die here
}

static int build_one_query(const char *ascii, int32_t len, const blastp_params *p, QueryDev &out,
                           cudaStream_t s) {
  std::vector<uint8_t> Q;
  int rc = encode_query(ascii, len, Q);
  return rc ? rc : build_table(Q, p, out, s);
}

// Query groups of a batch (one DB scan for several
// queries).  Members are concatenated with `gap` sentinel codes between
// them, gap >= A + 8: two members' hits that share a combined diagonal lie
// >= A apart in the subject, so no two-hit pair, lasthit or ext_reach ever
// links them, and every X-drop stops at the sentinels of its own member --
// the group's search returns exactly the members' searches.
// First-fit decreasing into groups of combined length <= kGroupLen
// (config 5 sweep, profiles/r01/group_sweep.txt: 768 757 ms, 1024 742,
// 1280 732, 1536 746, 2048 824 -- longer groups cost resident warps --
// vs 786 ms query by query).
constexpr int32_t kGroupLen = 1280;
static int build_groups(blastp_query_table *t, const char *const *queries, const int32_t *lens,
                        int32_t nq, cudaStream_t s) {
  const char *env = std::getenv("BLASTP_GROUP");  // knob: BLASTP_GROUP=0 disables grouping
  if ((env && std::atoi(env) == 0) || nq < 2) {
    for (int32_t i = 0; i < nq; ++i) t->alone.push_back(i);
    return BLASTP_OK;
  }
  const int32_t gap = t->p.window + 8;
  t->group_gap = gap;
  int32_t budget = kGroupLen;  // knob: BLASTP_GROUP_LEN (combined length per group)
  if (const char *v = std::getenv("BLASTP_GROUP_LEN")) budget = std::max(3, std::atoi(v));
  std::vector<int32_t> order(static_cast<size_t>(nq));
  for (int32_t i = 0; i < nq; ++i) order[static_cast<size_t>(i)] = i;
  std::stable_sort(order.begin(), order.end(),
                   [&](int32_t a, int32_t b) { return lens[a] > lens[b]; });
  std::vector<std::vector<int32_t>> bins;
  std::vector<int32_t> used;
  for (int32_t i : order) {
    size_t b = 0;
    for (; b < bins.size(); ++b)
      if (used[b] + gap + lens[i] <= budget) break;
    if (b == bins.size()) {
      bins.push_back({});
      used.push_back(-gap);
    }
    bins[b].push_back(i);
    used[b] += gap + lens[i];
  }
  for (auto &members : bins) {
    if (members.size() == 1) {
      t->alone.push_back(members[0]);
      continue;
    }
    std::sort(members.begin(), members.end());
    std::vector<uint8_t> Q, M;
    std::vector<int32_t> sub;
    for (int32_t i : members) {
      if (!Q.empty()) Q.insert(Q.end(), static_cast<size_t>(gap), uint8_t(kSentinel));
      sub.push_back(static_cast<int32_t>(Q.size()));
      int rc = encode_query(queries[i], lens[i], M);
      if (rc) return rc;
      Q.insert(Q.end(), M.begin(), M.end());
    }
    for (int32_t i : members) sub.push_back(i);
    QueryDev g;
    int rc = build_table(Q, &t->p, g, s);
    if (rc) return rc;
    g.nsub = static_cast<int32_t>(members.size());
    if (cudaMalloc(&g.sub, sizeof(int32_t) * sub.size()) != cudaSuccess) {
      cudaGetLastError();
      free_query_dev(g);
      return fail(BLASTP_E_NOMEM, "device allocation for a query group failed");
    }
    t->groups.push_back(g);
    CUDA_TRY(cudaMemcpy(g.sub, sub.data(), sizeof(int32_t) * sub.size(), cudaMemcpyHostToDevice));
  }
  return BLASTP_OK;
}

int blastp_build_query_batch(const char *const *queries, const int32_t *lens, int32_t nq,
                             const blastp_params *p, int device, void *cuda_stream,
                             blastp_query_table **out) {
  if (!out) return fail(BLASTP_E_INVALID_ARG, "out is NULL");
  *out = nullptr;
  if (!queries || !lens || nq < 1) return fail(BLASTP_E_INVALID_ARG, "no queries");
  int rc = validate_params(p);
  if (rc) return rc;
  DeviceGuard g(device);
  if (g.err != cudaSuccess) return fail(BLASTP_E_CUDA, "cudaSetDevice(%d): %s", device, cudaGetErrorString(g.err));
  auto *t = new (std::nothrow) blastp_query_table;
  if (!t) return fail(BLASTP_E_NOMEM, "host allocation failed");
  t->device = device;
  t->p = *p;
  t->q.resize(static_cast<size_t>(nq));
  for (int32_t i = 0; i < nq; ++i) {
    rc = build_one_query(queries[i], lens[i], p, t->q[static_cast<size_t>(i)],
                         static_cast<cudaStream_t>(cuda_stream));
    if (rc) {
      blastp_query_table_free(t);
      return rc;
    }
    t->entries += t->q[static_cast<size_t>(i)].entries;
  }
  rc = build_groups(t, queries, lens, nq, static_cast<cudaStream_t>(cuda_stream));
  if (rc) {
    blastp_query_table_free(t);
    return rc;
  }
  *out = t;
  return BLASTP_OK;
}

int blastp_build_query_table(const char *query_ascii, int32_t len, const blastp_params *p,
                             int device, void *cuda_stream, blastp_query_table **out) {
  const char *qs[1] = {query_ascii};
  int32_t ls[1] = {len};
  return blastp_build_query_batch(qs, ls, 1, p, device, cuda_stream, out);
}

int blastp_query_table_groups(const blastp_query_table *q, int32_t *groups, int32_t *alone,
                              int32_t *gap) {
  if (!q) return fail(BLASTP_E_INVALID_ARG, "table is NULL");
  if (groups) *groups = static_cast<int32_t>(q->groups.size());
  if (alone) *alone = static_cast<int32_t>(q->alone.size());
  if (gap) *gap = q->group_gap;
  return BLASTP_OK;
}

int blastp_query_table_info(const blastp_query_table *q, int32_t *num_queries,
                            int64_t *table_entries) {
  if (!q) return fail(BLASTP_E_INVALID_ARG, "table is NULL");
  if (num_queries) *num_queries = static_cast<int32_t>(q->q.size());
  if (table_entries) *table_entries = q->entries;
  return BLASTP_OK;
}

void blastp_query_table_free(blastp_query_table *q) {
  if (!q) return;
  DeviceGuard g(q->device);
  for (auto &d : q->q) free_query_dev(d);
  for (auto &d : q->groups) free_query_dev(d);
  delete q;
}

// --------------------------------------------------------- database / shards

int blastp_shard_range(const int64_t *offsets, int64_t nseq, int32_t shard_index,
                       int32_t num_shards, int64_t *lo, int64_t *hi) {
  if (!offsets || !lo || !hi || nseq < 0 || num_shards < 1 || shard_index < 0 ||
      shard_index >= num_shards)
    return fail(BLASTP_E_INVALID_ARG, "bad shard arguments (shard %d of %d, nseq %lld)",
                shard_index, num_shards, static_cast<long long>(nseq));
  const int64_t total = offsets[nseq] - offsets[0];
  auto first_at = [&](int32_t k) -> int64_t {
    if (k <= 0) return 0;
    if (k >= num_shards) return nseq;
    // first i with offsets[i] - offsets[0] >= total * k / num_shards
    const __int128 num = static_cast<__int128>(total) * k;
    const int64_t target = static_cast<int64_t>(num / num_shards);
    int64_t a = 0, b = nseq;
    while (a < b) {
      const int64_t m = (a + b) / 2;
      if (offsets[m] - offsets[0] >= target) b = m; else a = m + 1;
    }
    return a;
  };
  *lo = first_at(shard_index);
  *hi = first_at(shard_index + 1);
  if (*hi < *lo) *hi = *lo;
  return BLASTP_OK;
}

}  // extern "C"

// Packed-stream bytes and chunk plan of n subjects / nres residues.
// Stream layout: kStreamPadFront sentinels, then subject i at
// sstart[i] = pad + (offsets[lo+i] - offsets[lo]) + i, each followed by one
// sentinel; kStreamPadBack trailing sentinels; 512-byte multiple.  Chunks of
// C residues of whole subjects (8 per resident warp, 128 <= C <= 8192: measured
// 1.3% faster than 16384 on config 3), the last 2 C per resident warp in
// chunks of C/4 (ChunkPlan).
static void layout_sizes(int64_t n, int64_t nres, int sms, int64_t *stream_len, ChunkPlan *plan) {
  *stream_len = (kStreamPadFront + nres + n + kStreamPadBack + 511) & ~int64_t(511);
  const int64_t warps = int64_t(sms) * 32;
  int64_t c = nres / (warps * 8);
  // at least 128: a small shard still spreads over many warps (config 1,
  // 250k residues: 0.066 ms vs 0.095 ms with a 1024 minimum; config 2
  // unchanged; profiles/r01/chunk_sweep.txt)
  c = std::min<int64_t>(std::max<int64_t>(c, 128), 8192);
  if (const char *ce = std::getenv("BLASTP_CHUNK")) c = std::max<int64_t>(64, std::atoll(ce));
  plan->C = c;
  plan->Ct = std::min<int64_t>(c, std::max<int64_t>(1024, c / 4));
  if (const char *v = std::getenv("BLASTP_TAIL_CHUNKS")) {  // knob: 0 = uniform chunks
    if (std::atoi(v) == 0) plan->Ct = c;
  }
  plan->K1 = std::max<int64_t>(0, nres - 2 * warps * c) / c;
  const int64_t rest = nres - plan->K1 * c;
  plan->nchunks = n > 0 ? plan->K1 + (rest + plan->Ct - 1) / plan->Ct + 1 : 0;
}

// Bump allocator over one device block: the pipelined host-db search carves
// every part's buffers from a single pool allocation per call (per-part
// allocations let the pool grow or fragment in the middle of the pipeline).
struct Arena {
  uint8_t *base = nullptr;
  size_t cap = 0, used = 0;
  void *take(size_t bytes) {
    used = (used + 255) & ~size_t(255);
    if (used + bytes > cap) return nullptr;
    void *p = base + used;
    used += bytes;
    return p;
  }
};
static size_t arena_bytes(int64_t n, int64_t nres, int sms) {
  int64_t len = 0;
  ChunkPlan plan{};
  layout_sizes(n, nres, sms, &len, &plan);
  const int64_t nchunks = plan.nchunks;
  const auto a = [](size_t b) { return (b + 255) & ~size_t(255); };
  return a(size_t(len)) + a(8 * size_t(std::max<int64_t>(n, 1))) +
         2 * a(sizeof(Chunk) * size_t(std::max<int64_t>(nchunks, 1))) + a(64);
}
// Staging buffers of a pack (ASCII residues, offsets, error flags); shared by
// the parts of one pipelined search, which are packed in order on one stream.
struct PackStaging {
  uint8_t *ascii = nullptr;
  int64_t *off = nullptr;
  int *err = nullptr;
};

// Pack subjects [lo, hi) of the offsets array (the body of blastp_pack_db).
// arena / staging: optional preallocated buffers (blastp_search_host_db).
static int pack_range(const char *residues_ascii, const int64_t *offsets, int64_t lo, int64_t hi,
                      int device, cudaStream_t s, blastp_db **out, Arena *arena = nullptr,
                      const PackStaging *staging = nullptr) {
  const int64_t n = hi - lo;
  const int64_t nres = offsets[hi] - offsets[lo];
  if (nres < 0) return fail(BLASTP_E_INVALID_ARG, "offsets decrease");
  if (nres > 0 && !residues_ascii) return fail(BLASTP_E_INVALID_ARG, "residues is NULL");
  DeviceGuard g(device);
  if (g.err != cudaSuccess) return fail(BLASTP_E_CUDA, "cudaSetDevice(%d): %s", device, cudaGetErrorString(g.err));

  auto *db = new (std::nothrow) blastp_db;
  if (!db) return fail(BLASTP_E_NOMEM, "host allocation failed");
  db->device = device;
  db->sms = num_sms(device);
  db->nseq = n;
  db->residues = nres;
  db->subject_base = lo;
  // Subject starts, length checks and the chunk plan are computed on the GPU.
  ChunkPlan plan{};
  layout_sizes(n, nres, db->sms, &db->stream_len, &plan);
  const int64_t nchunks = plan.nchunks;
  db->nchunks = static_cast<int32_t>(nchunks);
  db->carved = arena != nullptr;

  // stream-ordered allocations from the library's pool, which keeps its
  // memory (repeated pack calls do not pay cudaMalloc again; common.cuh)
  uint8_t *d_ascii = staging ? staging->ascii : nullptr;
  int64_t *d_off = staging ? staging->off : nullptr;
  int *d_err = staging ? staging->err : nullptr;
  auto cleanup = [&](int code) {
    if (!staging) {
      cudaFreeAsync(d_ascii, s);
      cudaFreeAsync(d_off, s);
      cudaFreeAsync(d_err, s);
    }
    if (code != BLASTP_OK) {
      cudaStreamSynchronize(s);
      blastp_db_free(db);
    }
    return code;
  };
  auto dalloc = [&](auto **p, size_t bytes) {
    if (arena) {
      *p = static_cast<std::remove_pointer_t<decltype(p)>>(arena->take(bytes));
      return *p != nullptr;
    }
    return pool_malloc_async(reinterpret_cast<void **>(p), bytes, s) == cudaSuccess;
  };
  if (!dalloc(&db->stream, static_cast<size_t>(db->stream_len)) ||
      !dalloc(&db->sstart, sizeof(int64_t) * static_cast<size_t>(std::max<int64_t>(n, 1))) ||
      !dalloc(&db->chunks, sizeof(Chunk) * static_cast<size_t>(std::max<int64_t>(nchunks, 1))) ||
      !dalloc(&db->long_chunks, sizeof(Chunk) * static_cast<size_t>(std::max<int64_t>(nchunks, 1))) ||
      !dalloc(&db->counters, 64) ||
      (!staging &&
       (pool_malloc_async(&d_ascii, static_cast<size_t>(std::max<int64_t>(nres, 1)), s) != cudaSuccess ||
        pool_malloc_async(&d_off, sizeof(int64_t) * static_cast<size_t>(n + 1), s) != cudaSuccess ||
        pool_malloc_async(&d_err, sizeof(int), s) != cudaSuccess))) {
    cudaGetLastError();
    return cleanup(fail(BLASTP_E_NOMEM, "device allocation for the database failed"));
  }
  upload_encode_table();
  const bool dbg = std::getenv("BLASTP_DEBUG_PIPE") != nullptr;
  const auto t0 = std::chrono::steady_clock::now();
  auto ms = [&]() {
    return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  };
  double t_off = 0, t_enq = 0;
  // The copies come first in stream order: copy engines need no SMs, so they
  // overlap a search still running on another stream; the memsets and
  // kernels after them wait for SMs.  (Pinned host buffers make both copies
  // asynchronous.)
  cudaError_t e = cudaSuccess;
  if (nres > 0)
    e = cudaMemcpyAsync(d_ascii, residues_ascii + offsets[lo], static_cast<size_t>(nres),
                        cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(d_off, offsets + lo, sizeof(int64_t) * static_cast<size_t>(n + 1),
                        cudaMemcpyHostToDevice, s);
  t_off = ms();
  if (e == cudaSuccess) e = cudaMemsetAsync(d_err, 0, sizeof(int), s);
  if (e == cudaSuccess) e = cudaMemsetAsync(db->counters, 0, sizeof(unsigned long long) * 8, s);
  if (e == cudaSuccess)
    e = launch_layout(d_off, n, plan, db->sstart, db->chunks, db->long_chunks,
                      reinterpret_cast<int *>(db->counters + 6), d_err, s);
  if (e == cudaSuccess)
    e = launch_pack(d_ascii, d_off, n, db->sstart, db->stream, db->stream_len, d_err, s);
  t_enq = ms();
  int h_err = 0, h_nlong = 0;
  if (e == cudaSuccess) e = cudaMemcpyAsync(&h_err, d_err, sizeof(int), cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(&h_nlong, db->counters + 6, sizeof(int), cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess)
    return cleanup(fail(BLASTP_E_CUDA, "packing the database failed: %s", cudaGetErrorString(e)));
  if (h_err & 2) return cleanup(fail(BLASTP_E_INVALID_ARG, "offsets decrease inside the shard"));
  if (h_err & 4) return cleanup(fail(BLASTP_E_TOO_LONG, "a subject is longer than %d residues",
                                     BLASTP_MAX_SUBJECT_LEN));
  if (h_err) {
    // find the offending byte on the host for a precise message
    for (int64_t k = offsets[lo]; k < offsets[hi]; ++k)
      if (encode_char(static_cast<unsigned char>(residues_ascii[k])) < 0)
        return cleanup(fail(BLASTP_E_BAD_RESIDUE, "database byte %lld (0x%02x) is not a residue",
                            static_cast<long long>(k), static_cast<unsigned char>(residues_ascii[k])));
    return cleanup(fail(BLASTP_E_BAD_RESIDUE, "database holds an invalid residue"));
  }
  const double t_sync = ms();
  if (h_nlong > 0 && plan_long_items(db, h_nlong, s) != cudaSuccess) {
    cudaGetLastError();
    return cleanup(fail(BLASTP_E_NOMEM, "device allocation for the long-subject plan failed"));
  }
  if (dbg)
    fprintf(stderr, "[pack] %lld subjects %lld residues: offsets copied %.3f, enqueued %.3f, "
            "synced %.3f, planned %.3f ms\n", static_cast<long long>(n),
            static_cast<long long>(nres), t_off, t_enq, t_sync, ms());
  *out = db;
  return cleanup(BLASTP_OK);
}

extern "C" {

int blastp_pack_db(const char *residues_ascii, const int64_t *offsets, int64_t nseq,
                   int32_t shard_index, int32_t num_shards, int device, void *cuda_stream,
                   blastp_db **out) {
  if (!out) return fail(BLASTP_E_INVALID_ARG, "out is NULL");
  *out = nullptr;
  if (!offsets || nseq < 0) return fail(BLASTP_E_INVALID_ARG, "offsets NULL or nseq < 0");
  int64_t lo = 0, hi = 0;
  int rc = blastp_shard_range(offsets, nseq, shard_index, num_shards, &lo, &hi);
  if (rc) return rc;
  return pack_range(residues_ascii, offsets, lo, hi, device, static_cast<cudaStream_t>(cuda_stream),
                    out);
}

// Host copy of the subject starts (debug traces only; fetched lazily).
static const std::vector<int64_t> &host_sstart(const blastp_db *db) {
  auto *mdb = const_cast<blastp_db *>(db);
  if (static_cast<int64_t>(mdb->h_sstart.size()) != db->nseq) {
    mdb->h_sstart.resize(static_cast<size_t>(db->nseq));
    if (db->nseq > 0)
      cudaMemcpy(mdb->h_sstart.data(), db->sstart, sizeof(int64_t) * static_cast<size_t>(db->nseq),
                 cudaMemcpyDeviceToHost);
  }
  return mdb->h_sstart;
}

int blastp_db_long_info(const blastp_db *db, int64_t *long_items, int64_t *segments,
                        int64_t *segment_len) {
  if (!db) return fail(BLASTP_E_INVALID_ARG, "db is NULL");
  if (long_items) *long_items = db->nlong;
  if (segments) *segments = db->nsegs;
  if (segment_len) *segment_len = db->seg_len;
  return BLASTP_OK;
}

int blastp_db_info(const blastp_db *db, int64_t *nseq, int64_t *residues, int64_t *subject_base,
                   int64_t *stream_bytes, int64_t *num_chunks) {
  if (!db) return fail(BLASTP_E_INVALID_ARG, "db is NULL");
  if (nseq) *nseq = db->nseq;
  if (residues) *residues = db->residues;
  if (subject_base) *subject_base = db->subject_base;
  if (stream_bytes) *stream_bytes = db->stream_len;
  if (num_chunks) *num_chunks = db->nchunks;
  return BLASTP_OK;
}

void blastp_db_free(blastp_db *db) {
  if (!db) return;
  DeviceGuard g(db->device);
  if (!db->carved) {
    cudaFree(db->stream);
    cudaFree(db->sstart);
    cudaFree(db->chunks);
    cudaFree(db->long_chunks);
    cudaFree(db->counters);
  }
  cudaFree(db->items);
  cudaFree(db->seg_item);
  cudaFree(db->seg_count);
  cudaFree(db->seg_done);
  cudaFree(db->seg_list);
  cudaFree(db->out);
  delete db;
}

void blastp_hsp_free(blastp_hsp *h) { free(h); }

// ------------------------------------------------------------------ search

static int check_pair(const blastp_query_table *q, const blastp_db *db, const blastp_params *p) {
  if (!q || !db) return fail(BLASTP_E_INVALID_ARG, "table or db is NULL");
  int rc = validate_params(p);
  if (rc) return rc;
  if (q->device != db->device)
    return fail(BLASTP_E_INVALID_ARG, "table on device %d, db on device %d", q->device, db->device);
  if (p->threshold != q->p.threshold || p->word_len != q->p.word_len)
    return fail(BLASTP_E_INVALID_ARG, "threshold/word_len differ from the table's (%d/%d)",
                q->p.threshold, q->p.word_len);
  return BLASTP_OK;
}

// The search launches of a table ("units"): a batch's query groups (one scan
// per group) when the two-hit window fits the sentinel gap they were built
// with, and the queries left alone; traced runs search query by query.
// ids[u] = the query id of a single-query unit, -1 for a group.
static void launch_units(const blastp_query_table *q, const blastp_params *p, bool traced,
                         std::vector<const QueryDev *> *list, std::vector<int32_t> *ids) {
  list->clear();
  ids->clear();
  if (!q->groups.empty() && !traced && p->window + 8 <= q->group_gap) {
    for (const QueryDev &g : q->groups) {
      list->push_back(&g);
      ids->push_back(-1);
    }
    for (int32_t i : q->alone) {
      list->push_back(&q->q[static_cast<size_t>(i)]);
      ids->push_back(i);
    }
  } else {
    for (size_t i = 0; i < q->q.size(); ++i) {
      list->push_back(&q->q[i]);
      ids->push_back(static_cast<int32_t>(i));
    }
  }
}

// Enqueue the search of every query of `q` against `db` (or of the launch
// units [unit_begin, unit_end) only): HSPs appended to
// out (capacity cap) with the count in *count (device).  trace: optional.
static int enqueue_search(const blastp_query_table *q, const blastp_db *db,
                          const blastp_params *p, cudaStream_t s, blastp_hsp *out, int64_t cap,
                          unsigned long long *count, TraceRec *const trace[3],
                          const int64_t trace_cap[3], unsigned long long *trace_count,
                          bool reset_count = true, bool out_fence = false,
                          size_t unit_begin = 0, size_t unit_end = SIZE_MAX) {
  if (reset_count) CUDA_TRY(cudaMemsetAsync(count, 0, sizeof(unsigned long long), s));
  if (trace_count)  // [0..3): trace record counts, [3..3+kNumStats): event counters
    CUDA_TRY(cudaMemsetAsync(trace_count, 0, (3 + kNumStats) * sizeof(unsigned long long), s));
  if (db->nchunks == 0) return BLASTP_OK;
  std::vector<const QueryDev *> list;
  std::vector<int32_t> ids;
  launch_units(q, p, trace != nullptr, &list, &ids);
  for (size_t li = unit_begin; li < list.size() && li < unit_end; ++li) {
    const QueryDev &qd = *list[li];
    SearchArgs a{};
    a.stream = db->stream;
    a.sstart = db->sstart;
    a.subject_base = db->subject_base;
    a.nseq = db->nseq;
    a.stream_len = db->stream_len;
    a.chunks = db->chunks;
    a.nchunks = db->nchunks;
    a.long_items = db->items;
    a.nlong = db->nlong;
    // STATEFUL splits long subjects by diagonal range instead:
    // the same segment plan, no segment lists
    a.nsegs = db->nsegs;
    a.seg_item = db->seg_item;
    a.seg_list = db->seg_list;
    a.seg_count = db->seg_count;
    a.seg_done = db->seg_done;
    a.seg_len = db->seg_len;
    a.seg_cap = db->seg_cap;
    a.seq = ++const_cast<blastp_db *>(db)->seq;
    a.qv.woff = qd.woff;
    a.qv.wtab = qd.wtab;
    a.qv.qpos = qd.qpos;
    a.qv.qcodes = qd.qcodes;
    a.qv.lq = qd.lq;
    a.qv.query_id = ids[li];
    a.qv.nsub = qd.nsub;
    a.qv.sub = qd.sub;
    a.word_len = p->word_len;
    a.threshold = p->threshold;
    a.window = p->window;
    a.min_gap = p->min_gap;
    a.xdrop = p->xdrop;
    a.cutoff = p->cutoff;
    a.filter_mode = p->filter_mode;
    // HIT_DEDUP searches as Alg. 4 and writes every extension's seed record
    // (R17); the de-duplication step runs after the search
    a.ext_mode = p->ext_mode == BLASTP_EXT_HIT_DEDUP ? BLASTP_EXT_HIT : p->ext_mode;
    a.emit_seed = p->ext_mode == BLASTP_EXT_HIT_DEDUP ? 1 : 0;
    a.ring = search_ring_slots(qd.lq, p->window);
    a.table_entries = qd.entries;
    a.out = out;
    a.out_cap = cap;
    a.hsp_count = count;
    a.out_fence = out_fence ? 1 : 0;
    a.chunk_cursor = db->counters + 1;
    for (int k = 0; k < 3; ++k) {
      a.trace[k] = trace ? trace[k] : nullptr;
      a.trace_cap[k] = trace ? trace_cap[k] : 0;
    }
    a.trace_count = trace_count;
    a.stats = trace_count ? trace_count + 3 : nullptr;
    CUDA_TRY(cudaMemsetAsync(db->counters + 1, 0, sizeof(unsigned long long), s));
    CUDA_TRY(launch_search(a, db->sms, s));
  }
  return BLASTP_OK;
}

int blastp_search_ungapped_device(const blastp_query_table *q, const blastp_db *db,
                                  const blastp_params *p, void *cuda_stream, blastp_hsp *d_out,
                                  int64_t capacity, int64_t *d_count) {
  int rc = check_pair(q, db, p);
  if (rc) return rc;
  if (!d_count || capacity < 0 || (capacity > 0 && !d_out))
    return fail(BLASTP_E_INVALID_ARG, "bad output buffer");
  DeviceGuard g(db->device);
  return enqueue_search(q, db, p, static_cast<cudaStream_t>(cuda_stream), d_out, capacity,
                        reinterpret_cast<unsigned long long *>(d_count), nullptr, nullptr, nullptr);
}

int blastp_search_ungapped_append(const blastp_query_table *q, const blastp_db *db,
                                  const blastp_params *p, void *cuda_stream, blastp_hsp *d_out,
                                  int64_t capacity, int64_t *d_count) {
  int rc = check_pair(q, db, p);
  if (rc) return rc;
  if (!d_count || capacity < 0 || (capacity > 0 && !d_out))
    return fail(BLASTP_E_INVALID_ARG, "bad output buffer");
  DeviceGuard g(db->device);
  return enqueue_search(q, db, p, static_cast<cudaStream_t>(cuda_stream), d_out, capacity,
                        reinterpret_cast<unsigned long long *>(d_count), nullptr, nullptr, nullptr,
                        /*reset_count=*/false, /*out_fence=*/true);
}

// Exported device buffers (CUDA IPC).  cudaMalloc'd (not from the stream
// pool: pool memory cannot be exported with cudaIpcGetMemHandle).
static_assert(sizeof(cudaIpcMemHandle_t) <= BLASTP_IPC_HANDLE_BYTES, "IPC handle size");

int blastp_ipc_alloc(int device, int64_t bytes, void **d_ptr, void *handle_out) {
  if (!d_ptr || !handle_out || bytes <= 0) return fail(BLASTP_E_INVALID_ARG, "bad arguments");
  *d_ptr = nullptr;
  DeviceGuard g(device);
  if (g.err != cudaSuccess)
    return fail(BLASTP_E_CUDA, "cudaSetDevice(%d): %s", device, cudaGetErrorString(g.err));
  void *ptr = nullptr;
  if (cudaMalloc(&ptr, size_t(bytes)) != cudaSuccess) {
    cudaGetLastError();
    return fail(BLASTP_E_NOMEM, "cudaMalloc(%lld) for an exported buffer failed",
                static_cast<long long>(bytes));
  }
  cudaIpcMemHandle_t h;
  const cudaError_t e = cudaIpcGetMemHandle(&h, ptr);
  if (e != cudaSuccess) {
    cudaFree(ptr);
    return fail(BLASTP_E_CUDA, "cudaIpcGetMemHandle: %s", cudaGetErrorString(e));
  }
  std::memset(handle_out, 0, BLASTP_IPC_HANDLE_BYTES);
  std::memcpy(handle_out, &h, sizeof(h));
  *d_ptr = ptr;
  return BLASTP_OK;
}

int blastp_ipc_open(int device, const void *handle, void **d_ptr) {
  if (!d_ptr || !handle) return fail(BLASTP_E_INVALID_ARG, "bad arguments");
  *d_ptr = nullptr;
  DeviceGuard g(device);
  if (g.err != cudaSuccess)
    return fail(BLASTP_E_CUDA, "cudaSetDevice(%d): %s", device, cudaGetErrorString(g.err));
  cudaIpcMemHandle_t h;
  std::memcpy(&h, handle, sizeof(h));
  void *ptr = nullptr;
  const cudaError_t e = cudaIpcOpenMemHandle(&ptr, h, cudaIpcMemLazyEnablePeerAccess);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return fail(BLASTP_E_CUDA, "cudaIpcOpenMemHandle: %s", cudaGetErrorString(e));
  }
  *d_ptr = ptr;
  return BLASTP_OK;
}

int blastp_ipc_close(void *d_ptr) {
  if (!d_ptr) return BLASTP_OK;
  const cudaError_t e = cudaIpcCloseMemHandle(d_ptr);
  if (e != cudaSuccess) return fail(BLASTP_E_CUDA, "cudaIpcCloseMemHandle: %s", cudaGetErrorString(e));
  return BLASTP_OK;
}

int blastp_ipc_free(void *d_ptr) {
  if (!d_ptr) return BLASTP_OK;
  const cudaError_t e = cudaFree(d_ptr);
  if (e != cudaSuccess) return fail(BLASTP_E_CUDA, "cudaFree: %s", cudaGetErrorString(e));
  return BLASTP_OK;
}

// Stream-ordered release of a database (its buffers come from the pool):
// safe while kernels enqueued on `s` still read it.
static void db_free_async(blastp_db *db, cudaStream_t s) {
  if (!db) return;
  if (!db->carved)
    for (void *ptr : {static_cast<void *>(db->stream), static_cast<void *>(db->sstart),
                      static_cast<void *>(db->chunks), static_cast<void *>(db->long_chunks),
                      static_cast<void *>(db->counters)})
      if (ptr) cudaFreeAsync(ptr, s);
  for (void *ptr : {static_cast<void *>(db->items), static_cast<void *>(db->seg_item),
                    static_cast<void *>(db->seg_count), static_cast<void *>(db->seg_done),
                    static_cast<void *>(db->seg_list)})
    if (ptr) cudaFreeAsync(ptr, s);
  if (db->out) cudaFree(db->out);
  delete db;
}

// Part boundaries of a streamed shard [lo, hi) (whole subjects, by
// residues): num_parts equal parts, or (num_parts = 0) sizes growing 1.25x
// from a small first part -- its copy is the only one not hidden behind a
// search, and at 1.25x a part's H2D copy (~52 GB/s) takes about as long as
// the previous part's search (~41 G residues/s at q1054): config 3 e2e
// 30.4 ms at 1.2-1.3x vs 31.7 ms at 1.5x (profiles/r02/pipe_e2e_sweep.txt).
static std::vector<int64_t> part_cuts(const int64_t *offsets, int64_t lo, int64_t hi,
                                      int32_t num_parts, int growth = 125) {
  const int64_t total = offsets[hi] - offsets[lo];
  std::vector<int64_t> cut{lo};
  // knobs (tuning): BLASTP_PIPE_FIRST residues of the first part,
  // BLASTP_PIPE_GROWTH percent growth per part
  int64_t want = std::max<int64_t>(int64_t(1) << 24, total / 64);
  int64_t cap = std::numeric_limits<int64_t>::max();
  if (const char *v = std::getenv("BLASTP_PIPE_FIRST")) want = std::max<int64_t>(1, std::atoll(v));
  if (const char *v = std::getenv("BLASTP_PIPE_GROWTH")) growth = std::max(101, std::atoi(v));
  if (const char *v = std::getenv("BLASTP_PIPE_MAXPART")) cap = std::max<int64_t>(1, std::atoll(v));
  int64_t done = 0;
  for (int k = 0; cut.back() < hi; ++k) {
    int64_t size;
    if (num_parts > 0)
      size = (total * (k + 1)) / num_parts - done;
    else {
      size = std::min(want, cap);
      want = std::min(want * growth / 100, cap);
    }
    const int64_t target = offsets[lo] + done + std::max<int64_t>(size, 1);
    // first subject starting at or after target
    int64_t a = cut.back() + 1, b = hi;
    while (a < b) {
      const int64_t m = (a + b) >> 1;
      if (offsets[m] >= target) b = m; else a = m + 1;
    }
    cut.push_back(a);
    done = offsets[a] - offsets[lo];
  }
  return cut;
}

int blastp_search_host_db(const blastp_query_table *q, const char *residues_ascii,
                          const int64_t *offsets, int64_t nseq, int32_t shard_index,
                          int32_t num_shards, const blastp_params *p, int32_t num_parts,
                          void *cuda_stream, blastp_hsp *d_out, int64_t capacity,
                          int64_t *d_count) {
  if (!q) return fail(BLASTP_E_INVALID_ARG, "table is NULL");
  int rc = validate_params(p);
  if (rc) return rc;
  if (p->threshold != q->p.threshold || p->word_len != q->p.word_len)
    return fail(BLASTP_E_INVALID_ARG, "threshold/word_len differ from the table's (%d/%d)",
                q->p.threshold, q->p.word_len);
  if (!d_count || capacity < 0 || (capacity > 0 && !d_out))
    return fail(BLASTP_E_INVALID_ARG, "bad output buffer");
  if (!offsets || nseq < 0) return fail(BLASTP_E_INVALID_ARG, "offsets NULL or nseq < 0");
  if (num_parts < 0) return fail(BLASTP_E_INVALID_ARG, "num_parts %d < 0", num_parts);
  int64_t lo = 0, hi = 0;
  rc = blastp_shard_range(offsets, nseq, shard_index, num_shards, &lo, &hi);
  if (rc) return rc;
  DeviceGuard g(q->device);
  if (g.err != cudaSuccess) return fail(BLASTP_E_CUDA, "cudaSetDevice(%d): %s", q->device, cudaGetErrorString(g.err));
  cudaStream_t s = static_cast<cudaStream_t>(cuda_stream);
  auto *count = reinterpret_cast<unsigned long long *>(d_count);
  CUDA_TRY(cudaMemsetAsync(count, 0, sizeof(unsigned long long), s));
  const int64_t total = offsets[hi] - offsets[lo];
  if (total < 0) return fail(BLASTP_E_INVALID_ARG, "offsets decrease");
  const std::vector<int64_t> cut = part_cuts(offsets, lo, hi, num_parts);
  cudaStream_t cs = nullptr;  // copy + pack stream
  CUDA_TRY(cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking));
  // one arena for every part's packed buffers + shared staging buffers
  const int sms = num_sms(q->device);
  size_t total_bytes = 0;
  int64_t max_n = 0, max_res = 0;
  for (size_t k = 0; k + 1 < cut.size(); ++k) {
    const int64_t n = cut[k + 1] - cut[k], r = offsets[cut[k + 1]] - offsets[cut[k]];
    if (r < 0) {
      cudaStreamDestroy(cs);
      return fail(BLASTP_E_INVALID_ARG, "offsets decrease");
    }
    total_bytes += arena_bytes(n, r, sms);
    max_n = std::max(max_n, n);
    max_res = std::max(max_res, r);
  }
  const auto al = [](size_t b) { return (b + 255) & ~size_t(255); };
  total_bytes += al(size_t(std::max<int64_t>(max_res, 1))) + al(8 * size_t(max_n + 1)) + al(4);
  Arena arena;
  if (pool_malloc_async(reinterpret_cast<void **>(&arena.base), total_bytes, cs) != cudaSuccess) {
    cudaGetLastError();
    cudaStreamDestroy(cs);
    return fail(BLASTP_E_NOMEM, "device arena of %zu bytes for the host-db search", total_bytes);
  }
  arena.cap = total_bytes;
  PackStaging staging;
  staging.ascii = static_cast<uint8_t *>(arena.take(size_t(std::max<int64_t>(max_res, 1))));
  staging.off = static_cast<int64_t *>(arena.take(8 * size_t(max_n + 1)));
  staging.err = static_cast<int *>(arena.take(4));
  std::vector<blastp_db *> parts;
  // BLASTP_DEBUG_PIPE=1: per-part host timestamps and search event times on stderr
  const bool dbg = std::getenv("BLASTP_DEBUG_PIPE") != nullptr;
  std::vector<cudaEvent_t> ev;
  const auto t0 = std::chrono::steady_clock::now();
  auto ms = [&]() {
    return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  };
  auto mark = [&]() {
    if (!dbg) return;
    cudaEvent_t e;
    cudaEventCreate(&e);
    cudaEventRecord(e, s);
    ev.push_back(e);
  };
  mark();
  // Consecutive parts are searched on two alternating streams: part k+1's
  // search kernel fills the SMs that part k's launch leaves idle in its
  // tail (the CTAs of one search are resident one per SM and retire
  // unevenly).  Parts have separate counters; they share only the HSP
  // output counter, which is atomic.  BLASTP_PIPE_STREAMS=1: one stream.
  int nstreams = 2;
  if (const char *v = std::getenv("BLASTP_PIPE_STREAMS")) nstreams = std::atoi(v) == 1 ? 1 : 2;
  cudaStream_t s2 = s;
  cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
  if (nstreams == 2) {
    if (cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking) != cudaSuccess ||
        cudaEventCreateWithFlags(&ev_fork, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&ev_join, cudaEventDisableTiming) != cudaSuccess) {
      cudaGetLastError();
      if (s2 != s) cudaStreamDestroy(s2);
      cudaFreeAsync(arena.base, cs);
      cudaStreamDestroy(cs);
      return fail(BLASTP_E_CUDA, "could not create the second search stream");
    }
    cudaEventRecord(ev_fork, s);  // after the count reset
    cudaStreamWaitEvent(s2, ev_fork, 0);
  }
  rc = BLASTP_OK;
  for (size_t k = 0; k + 1 < cut.size() && rc == BLASTP_OK; ++k) {
    // the host blocks here for part k's copy while part k-1 is searched
    blastp_db *d = nullptr;
    const double a = ms();
    rc = pack_range(residues_ascii, offsets, cut[k], cut[k + 1], q->device, cs, &d, &arena,
                    &staging);
    if (rc) break;
    const double b = ms();
    parts.push_back(d);
    rc = enqueue_search(q, d, p, (k & 1) ? s2 : s, d_out, capacity, count, nullptr, nullptr,
                        nullptr, false);
    mark();
    if (dbg)
      fprintf(stderr, "[pipe] part %zu: %lld residues, pack %.3f..%.3f ms, search enqueued %.3f ms\n",
              k, static_cast<long long>(offsets[cut[k + 1]] - offsets[cut[k]]), a, b, ms());
  }
  if (s2 != s) {  // join: s waits for the searches on s2
    cudaEventRecord(ev_join, s2);
    cudaStreamWaitEvent(s, ev_join, 0);
    cudaEventDestroy(ev_fork);
    cudaEventDestroy(ev_join);
    cudaStreamDestroy(s2);
  }
  for (blastp_db *d : parts) db_free_async(d, s);
  // the searches on s read the arena: free it in their stream order (and
  // after the copy stream's last use of the staging buffers)
  {
    cudaEvent_t done_copy;
    if (cudaEventCreateWithFlags(&done_copy, cudaEventDisableTiming) == cudaSuccess) {
      cudaEventRecord(done_copy, cs);
      cudaStreamWaitEvent(s, done_copy, 0);
      cudaEventDestroy(done_copy);
    }
  }
  cudaFreeAsync(arena.base, s);
  cudaStreamDestroy(cs);
  if (dbg && !ev.empty()) {
    cudaEventSynchronize(ev.back());
    for (size_t k = 1; k < ev.size(); ++k) {
      float t = 0, u = 0;
      cudaEventElapsedTime(&t, ev[0], ev[k - 1]);
      cudaEventElapsedTime(&u, ev[0], ev[k]);
      fprintf(stderr, "[pipe] part %zu: search on device %.3f..%.3f ms (from the first mark)\n",
              k - 1, t, u);
    }
    for (cudaEvent_t e : ev) cudaEventDestroy(e);
  }
  return rc;
}

// ------------------------------------------------- formatted host database
// A shard packed once (the makeblastdb step of a BLAST installation) and kept
// in pinned host memory as ready-to-copy parts: each part's code stream,
// subject starts, chunk plan and long-item plan are the device buffers of a
// blastp_pack_db of that part, copied back.  A search then only copies them
// (copy engine, no kernel and no host synchronisation per part) and searches.
struct HostPart {
  int64_t nseq = 0, residues = 0, subject_base = 0, stream_len = 0;
  int32_t nchunks = 0, nlong = 0, nsegs = 0, seg_len = kSegLen, seg_cap = kSegCap;
  size_t off_stream = 0, off_sstart = 0, off_chunks = 0, off_items = 0, off_seg_item = 0;
};
struct blastp_host_db {
  int device = 0;
  int64_t nseq = 0, residues = 0, subject_base = 0;
  std::vector<HostPart> parts;
  uint8_t *buf = nullptr;  // pinned
  size_t bytes = 0;
};

static size_t al256(size_t b) { return (b + 255) & ~size_t(255); }

int blastp_format_host_db(const char *residues_ascii, const int64_t *offsets, int64_t nseq,
                          int32_t shard_index, int32_t num_shards, int32_t num_parts,
                          int device, void *cuda_stream, blastp_host_db **out) {
  if (!out) return fail(BLASTP_E_INVALID_ARG, "out is NULL");
  *out = nullptr;
  if (!offsets || nseq < 0) return fail(BLASTP_E_INVALID_ARG, "offsets NULL or nseq < 0");
  if (num_parts < 0) return fail(BLASTP_E_INVALID_ARG, "num_parts %d < 0", num_parts);
  int64_t lo = 0, hi = 0;
  int rc = blastp_shard_range(offsets, nseq, shard_index, num_shards, &lo, &hi);
  if (rc) return rc;
  if (offsets[hi] - offsets[lo] < 0) return fail(BLASTP_E_INVALID_ARG, "offsets decrease");
  DeviceGuard g(device);
  if (g.err != cudaSuccess) return fail(BLASTP_E_CUDA, "cudaSetDevice(%d): %s", device, cudaGetErrorString(g.err));
  cudaStream_t s = static_cast<cudaStream_t>(cuda_stream);
  // growth 1.25x (part_cuts' default): a part's copy (~52 GB/s from pinned
  // memory) must not take longer than the previous part's search (~41 G
  // residues/s at q1054): config 3 e2e 30.4 ms vs 31.7 at 1.4x
  // (profiles/r02/pipe_e2e_sweep.txt; r01: profiles/r01/fmt_sweep_v2.txt)
  const std::vector<int64_t> cut = part_cuts(offsets, lo, hi, num_parts);
  auto *h = new (std::nothrow) blastp_host_db;
  if (!h) return fail(BLASTP_E_NOMEM, "host allocation failed");
  h->device = device;
  h->nseq = hi - lo;
  h->residues = offsets[hi] - offsets[lo];
  h->subject_base = lo;
  std::vector<blastp_db *> dbs;
  auto cleanup = [&](int code) {
    for (blastp_db *d : dbs) blastp_db_free(d);
    if (code != BLASTP_OK) blastp_host_db_free(h);
    return code;
  };
  // pack every part on the device and lay out the host image; then copy
  // each part back
  size_t bytes = 0;
  for (size_t k = 0; k + 1 < cut.size(); ++k) {
    blastp_db *d = nullptr;
    rc = pack_range(residues_ascii, offsets, cut[k], cut[k + 1], device, s, &d);
    if (rc) return cleanup(rc);
    HostPart hp;
    hp.nseq = d->nseq;
    hp.residues = d->residues;
    hp.subject_base = d->subject_base;
    hp.stream_len = d->stream_len;
    hp.nchunks = d->nchunks;
    hp.nlong = d->nlong;
    hp.nsegs = d->nsegs;
    hp.seg_len = d->seg_len;
    hp.seg_cap = d->seg_cap;
    hp.off_stream = bytes;
    bytes += al256(size_t(hp.stream_len));
    hp.off_sstart = bytes;
    bytes += al256(sizeof(int64_t) * size_t(std::max<int64_t>(hp.nseq, 1)));
    hp.off_chunks = bytes;
    bytes += al256(sizeof(Chunk) * size_t(std::max(hp.nchunks, 1)));
    hp.off_items = bytes;
    bytes += al256(sizeof(LongItem) * size_t(std::max(hp.nlong, 1)));
    hp.off_seg_item = bytes;
    bytes += al256(sizeof(int32_t) * size_t(std::max(hp.nsegs, 1)));
    h->parts.push_back(hp);
    dbs.push_back(d);  // kept until the host image (sized by all parts) exists
  }
  if (cudaMallocHost(reinterpret_cast<void **>(&h->buf), std::max<size_t>(bytes, 1)) != cudaSuccess) {
    cudaGetLastError();
    return cleanup(fail(BLASTP_E_NOMEM, "pinned host image of %zu bytes", bytes));
  }
  h->bytes = bytes;
  cudaError_t e = cudaSuccess;
  for (size_t k = 0; k < dbs.size() && e == cudaSuccess; ++k) {
    const blastp_db *d = dbs[k];
    const HostPart &hp = h->parts[k];
    e = cudaMemcpyAsync(h->buf + hp.off_stream, d->stream, size_t(hp.stream_len),
                        cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess && hp.nseq > 0)
      e = cudaMemcpyAsync(h->buf + hp.off_sstart, d->sstart, sizeof(int64_t) * size_t(hp.nseq),
                          cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess && hp.nchunks > 0)
      e = cudaMemcpyAsync(h->buf + hp.off_chunks, d->chunks, sizeof(Chunk) * size_t(hp.nchunks),
                          cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess && hp.nlong > 0)
      e = cudaMemcpyAsync(h->buf + hp.off_items, d->items, sizeof(LongItem) * size_t(hp.nlong),
                          cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess && hp.nsegs > 0)
      e = cudaMemcpyAsync(h->buf + hp.off_seg_item, d->seg_item,
                          sizeof(int32_t) * size_t(hp.nsegs), cudaMemcpyDeviceToHost, s);
  }
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess)
    return cleanup(fail(BLASTP_E_CUDA, "copying the formatted parts back: %s", cudaGetErrorString(e)));
  *out = h;
  return cleanup(BLASTP_OK);
}

int blastp_host_db_info(const blastp_host_db *h, int64_t *nseq, int64_t *residues,
                        int64_t *subject_base, int32_t *num_parts, int64_t *host_bytes) {
  if (!h) return fail(BLASTP_E_INVALID_ARG, "host db is NULL");
  if (nseq) *nseq = h->nseq;
  if (residues) *residues = h->residues;
  if (subject_base) *subject_base = h->subject_base;
  if (num_parts) *num_parts = static_cast<int32_t>(h->parts.size());
  if (host_bytes) *host_bytes = static_cast<int64_t>(h->bytes);
  return BLASTP_OK;
}

void blastp_host_db_free(blastp_host_db *h) {
  if (!h) return;
  if (h->buf) cudaFreeHost(h->buf);
  delete h;
}

int blastp_search_formatted_db(const blastp_query_table *q, const blastp_host_db *h,
                               const blastp_params *p, void *cuda_stream, blastp_hsp *d_out,
                               int64_t capacity, int64_t *d_count) {
  if (!q || !h) return fail(BLASTP_E_INVALID_ARG, "table or host db is NULL");
  int rc = validate_params(p);
  if (rc) return rc;
  if (p->threshold != q->p.threshold || p->word_len != q->p.word_len)
    return fail(BLASTP_E_INVALID_ARG, "threshold/word_len differ from the table's (%d/%d)",
                q->p.threshold, q->p.word_len);
  if (q->device != h->device)
    return fail(BLASTP_E_INVALID_ARG, "table on device %d, host db formatted for device %d",
                q->device, h->device);
  if (!d_count || capacity < 0 || (capacity > 0 && !d_out))
    return fail(BLASTP_E_INVALID_ARG, "bad output buffer");
  DeviceGuard g(q->device);
  if (g.err != cudaSuccess) return fail(BLASTP_E_CUDA, "cudaSetDevice(%d): %s", q->device, cudaGetErrorString(g.err));
  cudaStream_t s = static_cast<cudaStream_t>(cuda_stream);
  auto *count = reinterpret_cast<unsigned long long *>(d_count);
  CUDA_TRY(cudaMemsetAsync(count, 0, sizeof(unsigned long long), s));
  // Device memory: a ring of part slots (BLASTP_PIPE_SLOTS, default 3, at
  // most one per part), each the largest part's image plus its scratch
  // (counters, segment lists / counts / publication flags); part k goes to
  // slot k mod nslots once the search of part k - nslots has released it.
  // The part images are position-independent (offsets within the part).
  const size_t nparts = h->parts.size();
  auto part_bytes = [&](size_t k) {
    const size_t end = k + 1 < nparts ? h->parts[k + 1].off_stream : h->bytes;
    return end - h->parts[k].off_stream;
  };
  size_t slot_img = 0, slot_bytes = 0;
  for (size_t k = 0; k < nparts; ++k) slot_img = std::max(slot_img, al256(part_bytes(k)));
  slot_bytes = slot_img;
  {
    size_t scr = 0;
    for (size_t k = 0; k < nparts; ++k) {
      const HostPart &hp = h->parts[k];
      const size_t ns = size_t(std::max(hp.nsegs, 1));
      scr = std::max(scr, al256(64) + al256(4 * ns) + al256(4 * ns) +
                              al256(4 * ns * size_t(hp.seg_cap)));
    }
    slot_bytes += scr;
  }
  size_t nslots = 3;
  if (const char *v = std::getenv("BLASTP_PIPE_SLOTS")) nslots = size_t(std::max(1, std::atoi(v)));
  nslots = std::max<size_t>(1, std::min(nslots, nparts));
  cudaStream_t cs = nullptr, s2 = nullptr;
  CUDA_TRY(cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking));
  if (cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking) != cudaSuccess) {
    cudaGetLastError();
    cudaStreamDestroy(cs);
    return fail(BLASTP_E_CUDA, "could not create the second search stream");
  }
  const size_t bytes = std::max<size_t>(nslots * slot_bytes, 256);
  uint8_t *dev = nullptr;
  // the slots are allocated in s's order; the copies on cs wait for that
  if (pool_malloc_async(reinterpret_cast<void **>(&dev), bytes, s) != cudaSuccess) {
    cudaGetLastError();
    cudaStreamDestroy(cs);
    cudaStreamDestroy(s2);
    return fail(BLASTP_E_NOMEM, "%zu part slots of %zu bytes for the formatted search", nslots,
                slot_bytes);
  }
  std::vector<cudaEvent_t> evs;
  auto event = [&]() {
    cudaEvent_t e = nullptr;
    if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) == cudaSuccess) evs.push_back(e);
    return e;
  };
  cudaEvent_t ev_start = event();
  cudaEventRecord(ev_start, s);  // arena allocated, count reset
  cudaStreamWaitEvent(cs, ev_start, 0);
  cudaStreamWaitEvent(s2, ev_start, 0);
  std::vector<blastp_db> dbs(nparts);
  std::vector<cudaEvent_t> done(nparts, nullptr);  // part k's search released its slot
  rc = BLASTP_OK;
  for (size_t k = 0; k < nparts && rc == BLASTP_OK; ++k) {
    const HostPart &hp = h->parts[k];
    blastp_db &d = dbs[k];
    uint8_t *slot = dev + (k % nslots) * slot_bytes;
    auto at = [&](size_t off) { return slot + (off - hp.off_stream); };
    d.device = h->device;
    d.sms = num_sms(h->device);
    d.nseq = hp.nseq;
    d.residues = hp.residues;
    d.subject_base = hp.subject_base;
    d.stream_len = hp.stream_len;
    d.nchunks = hp.nchunks;
    d.nlong = hp.nlong;
    d.nsegs = hp.nsegs;
    d.seg_len = hp.seg_len;
    d.seg_cap = hp.seg_cap;
    d.carved = true;
    d.stream = slot;
    d.sstart = reinterpret_cast<int64_t *>(at(hp.off_sstart));
    d.chunks = reinterpret_cast<Chunk *>(at(hp.off_chunks));
    d.items = reinterpret_cast<LongItem *>(at(hp.off_items));
    d.seg_item = reinterpret_cast<int32_t *>(at(hp.off_seg_item));
    const size_t ns = size_t(std::max(hp.nsegs, 1));
    uint8_t *sc = slot + slot_img;
    d.counters = reinterpret_cast<unsigned long long *>(sc);
    sc += al256(64);
    d.seg_count = reinterpret_cast<int32_t *>(sc);
    sc += al256(4 * ns);
    d.seg_done = reinterpret_cast<unsigned *>(sc);
    sc += al256(4 * ns);
    d.seg_list = reinterpret_cast<uint32_t *>(sc);
    // copy engine only: the part's image in one copy (its buffers are
    // contiguous in the image), after the slot's previous part was searched
    cudaError_t e = cudaSuccess;
    if (k >= nslots) e = cudaStreamWaitEvent(cs, done[k - nslots], 0);
    if (e == cudaSuccess)
      e = cudaMemcpyAsync(slot, h->buf + hp.off_stream, part_bytes(k), cudaMemcpyHostToDevice, cs);
    cudaEvent_t ready = event();
    if (e == cudaSuccess) e = cudaEventRecord(ready, cs);
    cudaStream_t ss = (k & 1) ? s2 : s;
    if (e == cudaSuccess) e = cudaStreamWaitEvent(ss, ready, 0);
    // per-part scratch reset (segment epochs start at 0; searches bump seq)
    if (e == cudaSuccess) e = cudaMemsetAsync(d.seg_done, 0, 4 * ns, ss);
    if (e == cudaSuccess) e = cudaMemsetAsync(d.counters, 0, 64, ss);
    if (e != cudaSuccess) {
      rc = fail(BLASTP_E_CUDA, "enqueueing part %zu: %s", k, cudaGetErrorString(e));
      break;
    }
    rc = enqueue_search(q, &d, p, ss, d_out, capacity, count, nullptr, nullptr, nullptr, false);
    done[k] = event();
    if (rc == BLASTP_OK && (!done[k] || cudaEventRecord(done[k], ss) != cudaSuccess))
      rc = fail(BLASTP_E_CUDA, "recording the end of part %zu's search", k);
  }
  // join s2 into s, then release the arena in s's order
  cudaEvent_t ev_join = event();
  cudaEventRecord(ev_join, s2);
  cudaStreamWaitEvent(s, ev_join, 0);
  cudaEvent_t ev_copy = event();
  cudaEventRecord(ev_copy, cs);
  cudaStreamWaitEvent(s, ev_copy, 0);
  cudaFreeAsync(dev, s);
  for (cudaEvent_t e : evs) cudaEventDestroy(e);
  cudaStreamDestroy(cs);
  cudaStreamDestroy(s2);
  for (blastp_db &d : dbs) d.carved = true;  // nothing owned: the arena holds it all
  return rc;
}

int blastp_sort_hsps_device(blastp_hsp *d_hsps, int64_t n, void *cuda_stream) {
  if (n < 0 || (n > 0 && !d_hsps)) return fail(BLASTP_E_INVALID_ARG, "bad HSP buffer");
  const cudaError_t e = sort_hsps(d_hsps, n, static_cast<cudaStream_t>(cuda_stream));
  if (e == cudaErrorMemoryAllocation) return fail(BLASTP_E_NOMEM, "sort scratch");
  CUDA_TRY(e);
  return BLASTP_OK;
}

int blastp_dedup_covered_device(blastp_hsp *d_rec, int64_t n, int32_t cutoff, int64_t *d_n_out,
                                void *cuda_stream) {
  if (n < 0 || (n > 0 && !d_rec) || !d_n_out) return fail(BLASTP_E_INVALID_ARG, "bad buffers");
  const cudaError_t e = dedup_covered(d_rec, n, cutoff, d_n_out, static_cast<cudaStream_t>(cuda_stream));
  if (e == cudaErrorMemoryAllocation) return fail(BLASTP_E_NOMEM, "de-duplication scratch");
  CUDA_TRY(e);
  return BLASTP_OK;
}

int blastp_unique_hsps_device(blastp_hsp *d_hsps, int64_t n, int64_t *d_n_out,
                              void *cuda_stream) {
  if (n < 0 || (n > 0 && !d_hsps) || !d_n_out)
    return fail(BLASTP_E_INVALID_ARG, "bad HSP buffer");
  const cudaError_t e = unique_hsps(d_hsps, n, d_n_out, static_cast<cudaStream_t>(cuda_stream));
  if (e == cudaErrorMemoryAllocation) return fail(BLASTP_E_NOMEM, "unique scratch");
  CUDA_TRY(e);
  return BLASTP_OK;
}

// The search into the db's device buffer (grown and re-run on overflow), then
// the canonical order (or Alg. 4's de-duplication, R17); *n = the HSP count.
// Synchronises s.
static int search_sorted_device(const blastp_query_table *q, const blastp_db *db,
                                const blastp_params *p, cudaStream_t s, int64_t *n_out) {
  auto *mdb = const_cast<blastp_db *>(db);
  if (mdb->out_cap == 0) {
    const int64_t want = std::max<int64_t>(4096, (db->residues / 1000 + 1) * int64_t(q->q.size()));
    if (cudaMalloc(&mdb->out, sizeof(blastp_hsp) * static_cast<size_t>(want)) != cudaSuccess)
      return fail(BLASTP_E_NOMEM, "device HSP buffer");
    mdb->out_cap = want;
  }
  unsigned long long h_count = 0;
  for (int attempt = 0; attempt < 2; ++attempt) {
    const int rc = enqueue_search(q, db, p, s, mdb->out, mdb->out_cap, mdb->counters, nullptr,
                                  nullptr, nullptr);
    if (rc) return rc;
    CUDA_TRY(cudaMemcpyAsync(&h_count, mdb->counters, sizeof(h_count), cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaStreamSynchronize(s));
    if (static_cast<int64_t>(h_count) <= mdb->out_cap) break;
    cudaFree(mdb->out);
    mdb->out = nullptr;
    mdb->out_cap = 0;
    const int64_t want = static_cast<int64_t>(h_count) + static_cast<int64_t>(h_count) / 4 + 1024;
    if (cudaMalloc(&mdb->out, sizeof(blastp_hsp) * static_cast<size_t>(want)) != cudaSuccess)
      return fail(BLASTP_E_NOMEM, "device HSP buffer (%lld)", static_cast<long long>(want));
    mdb->out_cap = want;
  }
  int64_t n = static_cast<int64_t>(h_count);
  if (p->ext_mode == BLASTP_EXT_HIT_DEDUP) {
    // Alg. 4's de-duplication step (R17): every extension's seed record ->
    // the coverage chain per diagonal -> canonical HSPs (synchronises s)
    const cudaError_t e = dedup_covered(mdb->out, n, p->cutoff,
                                        reinterpret_cast<int64_t *>(mdb->counters + 2), s);
    if (e == cudaErrorMemoryAllocation) return fail(BLASTP_E_NOMEM, "de-duplication scratch");
    CUDA_TRY(e);
    CUDA_TRY(cudaMemcpyAsync(&n, mdb->counters + 2, sizeof(n), cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaStreamSynchronize(s));
  } else {
    CUDA_TRY(sort_hsps(mdb->out, n, s));
  }
  *n_out = n;
  return BLASTP_OK;
}

int blastp_search_ungapped(const blastp_query_table *q, const blastp_db *db,
                           const blastp_params *p, void *cuda_stream, blastp_hsp **out_host,
                           int64_t *out_count) {
  if (!out_host || !out_count) return fail(BLASTP_E_INVALID_ARG, "output pointers are NULL");
  *out_host = nullptr;
  *out_count = 0;
  int rc = check_pair(q, db, p);
  if (rc) return rc;
  DeviceGuard g(db->device);
  cudaStream_t s = static_cast<cudaStream_t>(cuda_stream);
  int64_t n = 0;
  if ((rc = search_sorted_device(q, db, p, s, &n))) return rc;
  auto *h = static_cast<blastp_hsp *>(malloc(sizeof(blastp_hsp) * static_cast<size_t>(std::max<int64_t>(n, 1))));
  if (!h) return fail(BLASTP_E_NOMEM, "host HSP array");
  if (n > 0) CUDA_TRY(cudaMemcpyAsync(h, db->out, sizeof(blastp_hsp) * static_cast<size_t>(n),
                                      cudaMemcpyDeviceToHost, s));
  CUDA_TRY(cudaStreamSynchronize(s));
  *out_host = h;
  *out_count = n;
  return BLASTP_OK;
}

// ------------------------------------------------------------ gapped stage

void blastp_gapped_params_default(blastp_gapped_params *gp) {
  if (!gp) return;
  gp->gap_open = 11;
  gp->gap_extend = 1;
  gp->xdrop = 38;
  gp->cutoff = 41;
}

void blastp_gapped_free(blastp_gapped *g) { free(g); }

static int validate_gapped(const blastp_gapped_params *gp) {
  if (!gp) return fail(BLASTP_E_INVALID_ARG, "gapped params are NULL");
  if (gp->gap_open < 0 || gp->gap_open > 1000)
    return fail(BLASTP_E_INVALID_ARG, "gap_open %d outside [0, 1000]", gp->gap_open);
  if (gp->gap_extend < 1 || gp->gap_extend > 1000)
    return fail(BLASTP_E_INVALID_ARG, "gap_extend %d outside [1, 1000]", gp->gap_extend);
  if (gp->xdrop < 0 || gp->xdrop > 100000)
    return fail(BLASTP_E_INVALID_ARG, "xdrop %d outside [0, 100000]", gp->xdrop);
  return BLASTP_OK;
}

// The gapped stage over a device list of this shard (synchronous on s).
static int gapped_device(const blastp_query_table *q, const blastp_db *db, const blastp_hsp *d_hsps,
                         int64_t n, const blastp_gapped_params *gp, cudaStream_t s,
                         blastp_gapped *d_out, int64_t capacity, int64_t *count) {
  *count = 0;
  if (n == 0) return BLASTP_OK;
  if (n > (int64_t(1) << 30) - 1)
    return fail(BLASTP_E_INVALID_ARG, "%lld HSPs in one gapped call (at most 2^30 - 1)",
                static_cast<long long>(n));
  const int32_t nq = static_cast<int32_t>(q->q.size());
  std::vector<const uint8_t *> qp(static_cast<size_t>(nq));
  std::vector<int32_t> ql(static_cast<size_t>(nq));
  for (int32_t k = 0; k < nq; ++k) {
    qp[k] = q->q[k].qcodes;
    ql[k] = q->q[k].lq;
  }
  if (db->max_len < 0) {  // once per shard (a pass over the host copy of the subject starts)
    int64_t maxlen = 0;
    const std::vector<int64_t> &st = host_sstart(db);
    for (int64_t i = 0; i < db->nseq; ++i) {
      const int64_t en =
          i + 1 < db->nseq ? st[i + 1] - 1 : kStreamPadFront + db->residues + db->nseq - 1;
      maxlen = std::max(maxlen, en - st[i]);
    }
    const_cast<blastp_db *>(db)->max_len = maxlen;
  }
  const int64_t maxlen = db->max_len;
  const uint8_t **d_qp = nullptr;
  int32_t *d_ql = nullptr;
  if (pool_malloc_async(&d_qp, sizeof(void *) * static_cast<size_t>(nq), s) != cudaSuccess ||
      pool_malloc_async(&d_ql, sizeof(int32_t) * static_cast<size_t>(nq), s) != cudaSuccess) {
    if (d_qp) cudaFreeAsync(d_qp, s);
    return fail(BLASTP_E_NOMEM, "gapped query arrays");
  }
  CUDA_TRY(cudaMemcpyAsync(d_qp, qp.data(), sizeof(void *) * qp.size(), cudaMemcpyHostToDevice, s));
  CUDA_TRY(cudaMemcpyAsync(d_ql, ql.data(), sizeof(int32_t) * ql.size(), cudaMemcpyHostToDevice, s));
  GappedArgs a{};
  a.hsps = d_hsps;
  a.n = n;
  a.qcodes = d_qp;
  a.qlens = d_ql;
  a.nq = nq;
  a.stream = db->stream;
  a.sstart = db->sstart;
  a.nseq = db->nseq;
  a.subject_base = db->subject_base;
  a.stream_end = kStreamPadFront + db->residues + db->nseq - 1;
  a.max_subject_len = maxlen;
  a.gap_open = gp->gap_open;
  a.gap_extend = gp->gap_extend;
  a.xdrop = gp->xdrop;
  a.cutoff = gp->cutoff;
  int err = 0;
  const cudaError_t e = launch_gapped(a, db->sms, d_out, capacity, count, &err, s);
  cudaFreeAsync(d_qp, s);
  cudaFreeAsync(d_ql, s);
  if (e == cudaErrorMemoryAllocation) return fail(BLASTP_E_NOMEM, "gapped scratch");
  CUDA_TRY(e);
  if (err & 1)
    return fail(BLASTP_E_INVALID_ARG, "HSP list: an id outside the table / shard, or pairs not "
                "in canonical order");
  if (err & 2) return fail(BLASTP_E_INVALID_ARG, "HSP list: a seed outside its sequences");
  if (*count > capacity)
    return fail(BLASTP_E_CAPACITY, "%lld gapped alignments, capacity %lld",
                static_cast<long long>(*count), static_cast<long long>(capacity));
  return BLASTP_OK;
}

int blastp_gapped_extend_device(const blastp_query_table *q, const blastp_db *db,
                                const blastp_hsp *d_hsps, int64_t n,
                                const blastp_gapped_params *gp, void *cuda_stream,
                                blastp_gapped *d_out, int64_t capacity, int64_t *out_count) {
  if (!q || !db || !out_count || n < 0 || (n > 0 && !d_hsps) || capacity < 0 ||
      (capacity > 0 && !d_out))
    return fail(BLASTP_E_INVALID_ARG, "bad arguments");
  *out_count = 0;
  int rc = validate_gapped(gp);
  if (rc) return rc;
  if (q->device != db->device)
    return fail(BLASTP_E_INVALID_ARG, "table on device %d, db on device %d", q->device, db->device);
  DeviceGuard g(db->device);
  return gapped_device(q, db, d_hsps, n, gp, static_cast<cudaStream_t>(cuda_stream), d_out,
                       capacity, out_count);
}

// Fig. 12's overlap on one GPU: the search of launch unit
// u + 1 (a query group or a lone query) runs on stream s while the gapped
// stage of unit u runs on a second stream; two unit buffers alternate.
// Results are gathered on the host and put in canonical order.  Synchronous.
static int search_gapped_pipelined(const blastp_query_table *q, const blastp_db *db,
                                   const blastp_params *p, const blastp_gapped_params *gp,
                                   cudaStream_t s, std::vector<blastp_gapped> *gout,
                                   std::vector<blastp_hsp> *uout, bool want_ungapped) {
  std::vector<const QueryDev *> list;
  std::vector<int32_t> ids;
  launch_units(q, p, false, &list, &ids);
  const size_t U = list.size();
  int32_t max_members = 1;
  for (const QueryDev *u : list) max_members = std::max(max_members, std::max(u->nsub, 1));
  int64_t cap = std::max<int64_t>(4096, (db->residues / 1000 + 1) * max_members);
  if (const char *v = std::getenv("BLASTP_PIPE_CAP"))  // tests: force the overflow re-run
    cap = std::max<int64_t>(1, std::atoll(v));
  cudaStream_t s2 = nullptr;
  CUDA_TRY(cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking));
  blastp_hsp *buf[2] = {nullptr, nullptr};
  int64_t bcap[2] = {0, 0};
  unsigned long long *cnt = nullptr;
  blastp_gapped *gbuf = nullptr;
  int64_t gcap = 0;
  cudaEvent_t ev[2] = {nullptr, nullptr};
  int rc = BLASTP_OK;
  auto cleanup = [&]() {
    cudaStreamSynchronize(s);
    cudaStreamSynchronize(s2);
    for (int k = 0; k < 2; ++k) {
      if (buf[k]) cudaFree(buf[k]);
      if (ev[k]) cudaEventDestroy(ev[k]);
    }
    if (cnt) cudaFree(cnt);
    if (gbuf) cudaFree(gbuf);
    cudaStreamDestroy(s2);
  };
  auto grow = [&](int k, int64_t want) -> bool {
    if (bcap[k] >= want) return true;
    if (buf[k]) cudaFree(buf[k]);
    buf[k] = nullptr;
    bcap[k] = 0;
    if (cudaMalloc(&buf[k], sizeof(blastp_hsp) * static_cast<size_t>(want)) != cudaSuccess) return false;
    bcap[k] = want;
    return true;
  };
  if (!grow(0, cap) || !grow(1, cap) ||
      cudaMalloc(&cnt, 2 * sizeof(unsigned long long)) != cudaSuccess ||
      cudaEventCreateWithFlags(&ev[0], cudaEventDisableTiming) != cudaSuccess ||
      cudaEventCreateWithFlags(&ev[1], cudaEventDisableTiming) != cudaSuccess) {
    cleanup();
    return fail(BLASTP_E_NOMEM, "pipeline buffers");
  }
  auto enqueue_unit = [&](size_t u, cudaStream_t st) -> int {
    const int k = int(u & 1);
    int r = enqueue_search(q, db, p, st, buf[k], bcap[k], cnt + k, nullptr, nullptr, nullptr,
                           true, false, u, u + 1);
    if (!r && cudaEventRecord(ev[k], st) != cudaSuccess) r = fail(BLASTP_E_CUDA, "event record");
    return r;
  };
  rc = enqueue_unit(0, s);
  for (size_t u = 0; u < U && rc == BLASTP_OK; ++u) {
    const int k = int(u & 1);
    // the next unit's search goes ahead on s while this one is extended on s2
    if (u + 1 < U && (rc = enqueue_unit(u + 1, s))) break;
    unsigned long long n = 0;
    cudaError_t e = cudaStreamWaitEvent(s2, ev[k], 0);
    if (e == cudaSuccess) e = cudaMemcpyAsync(&n, cnt + k, sizeof(n), cudaMemcpyDeviceToHost, s2);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s2);
    if (e != cudaSuccess) {
      rc = fail(BLASTP_E_CUDA, "pipeline unit %zu: %s", u, cudaGetErrorString(e));
      break;
    }
    if (static_cast<int64_t>(n) > bcap[k]) {
      // overflow: drain s (the next unit's search shares the db's chunk
      // cursor), grow and re-run this unit on s2
      if ((e = cudaStreamSynchronize(s)) != cudaSuccess) {
        rc = fail(BLASTP_E_CUDA, "pipeline drain: %s", cudaGetErrorString(e));
        break;
      }
      if (!grow(k, static_cast<int64_t>(n) + static_cast<int64_t>(n) / 4 + 1024)) {
        rc = fail(BLASTP_E_NOMEM, "pipeline unit buffer (%llu HSPs)", n);
        break;
      }
      if ((rc = enqueue_search(q, db, p, s2, buf[k], bcap[k], cnt + k, nullptr, nullptr, nullptr,
                               true, false, u, u + 1)))
        break;
      e = cudaMemcpyAsync(&n, cnt + k, sizeof(n), cudaMemcpyDeviceToHost, s2);
      if (e == cudaSuccess) e = cudaStreamSynchronize(s2);
      if (e != cudaSuccess) {
        rc = fail(BLASTP_E_CUDA, "pipeline re-run: %s", cudaGetErrorString(e));
        break;
      }
    }
    int64_t m = static_cast<int64_t>(n);
    if (p->ext_mode == BLASTP_EXT_HIT_DEDUP) {
      e = dedup_covered(buf[k], m, p->cutoff, reinterpret_cast<int64_t *>(cnt + k), s2);
      if (e == cudaSuccess) e = cudaMemcpyAsync(&m, cnt + k, sizeof(m), cudaMemcpyDeviceToHost, s2);
      if (e == cudaSuccess) e = cudaStreamSynchronize(s2);
    } else {
      e = sort_hsps(buf[k], m, s2);
    }
    if (e != cudaSuccess) {
      rc = e == cudaErrorMemoryAllocation ? fail(BLASTP_E_NOMEM, "sort scratch")
                                          : fail(BLASTP_E_CUDA, "sort: %s", cudaGetErrorString(e));
      break;
    }
    if (gcap < std::max<int64_t>(m, 1)) {
      if (gbuf) cudaFree(gbuf);
      gbuf = nullptr;
      gcap = 0;
      if (cudaMalloc(&gbuf, sizeof(blastp_gapped) * static_cast<size_t>(std::max<int64_t>(m, 1))) != cudaSuccess) {
        rc = fail(BLASTP_E_NOMEM, "gapped output");
        break;
      }
      gcap = std::max<int64_t>(m, 1);
    }
    int64_t g = 0;
    if ((rc = gapped_device(q, db, buf[k], m, gp, s2, gbuf, gcap, &g))) break;
    const size_t g0 = gout->size(), u0 = uout->size();
    gout->resize(g0 + static_cast<size_t>(g));
    if (want_ungapped) uout->resize(u0 + static_cast<size_t>(m));
    e = cudaSuccess;
    if (g > 0) e = cudaMemcpyAsync(gout->data() + g0, gbuf, sizeof(blastp_gapped) * size_t(g), cudaMemcpyDeviceToHost, s2);
    if (e == cudaSuccess && want_ungapped && m > 0)
      e = cudaMemcpyAsync(uout->data() + u0, buf[k], sizeof(blastp_hsp) * size_t(m), cudaMemcpyDeviceToHost, s2);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s2);
    if (e != cudaSuccess) {
      rc = fail(BLASTP_E_CUDA, "pipeline results: %s", cudaGetErrorString(e));
      break;
    }
  }
  cleanup();
  if (rc) return rc;
  // units partition the queries and each unit's list is canonical: a stable
  // counting sort by query id gives the canonical order of the whole
  const size_t nq = q->q.size();
  auto by_query = [nq](auto &v) {
    using T = typename std::decay<decltype(v)>::type::value_type;
    std::vector<size_t> start(nq + 1, 0);
    for (const T &r : v) ++start[static_cast<size_t>(r.query_id) + 1];
    for (size_t i = 0; i < nq; ++i) start[i + 1] += start[i];
    std::vector<T> out(v.size());
    for (const T &r : v) out[start[static_cast<size_t>(r.query_id)]++] = r;
    v.swap(out);
  };
  by_query(*gout);
  if (want_ungapped) by_query(*uout);
  return BLASTP_OK;
}

int blastp_search_gapped(const blastp_query_table *q, const blastp_db *db,
                         const blastp_params *p, const blastp_gapped_params *gp,
                         void *cuda_stream, blastp_gapped **out_host, int64_t *out_count,
                         blastp_hsp **ungapped_host, int64_t *ungapped_count) {
  if (!out_host || !out_count) return fail(BLASTP_E_INVALID_ARG, "output pointers are NULL");
  *out_host = nullptr;
  *out_count = 0;
  if (ungapped_host) *ungapped_host = nullptr;
  if (ungapped_count) *ungapped_count = 0;
  int rc = check_pair(q, db, p);
  if (rc) return rc;
  if ((rc = validate_gapped(gp))) return rc;
  DeviceGuard g(db->device);
  cudaStream_t s = static_cast<cudaStream_t>(cuda_stream);
  std::vector<const QueryDev *> list;
  std::vector<int32_t> ids;
  launch_units(q, p, false, &list, &ids);
  // BLASTP_GAPPED_PIPE=1: Fig. 12's overlap across launch units (measured
  // slower on one B200 -- both stages fill every SM, DESIGN.md 5.11 -- so the
  // default runs the two stages one after the other)
  const char *pipe = std::getenv("BLASTP_GAPPED_PIPE");
  if (list.size() > 1 && db->nchunks > 0 && pipe && std::atoi(pipe) == 1) {
    std::vector<blastp_gapped> gv;
    std::vector<blastp_hsp> uv;
    if ((rc = search_gapped_pipelined(q, db, p, gp, s, &gv, &uv, ungapped_host != nullptr))) return rc;
    auto *h = static_cast<blastp_gapped *>(malloc(sizeof(blastp_gapped) * std::max<size_t>(gv.size(), 1)));
    blastp_hsp *u = nullptr;
    if (ungapped_host) u = static_cast<blastp_hsp *>(malloc(sizeof(blastp_hsp) * std::max<size_t>(uv.size(), 1)));
    if (!h || (ungapped_host && !u)) {
      free(h);
      free(u);
      return fail(BLASTP_E_NOMEM, "host result arrays");
    }
    std::copy(gv.begin(), gv.end(), h);
    if (u) std::copy(uv.begin(), uv.end(), u);
    *out_host = h;
    *out_count = static_cast<int64_t>(gv.size());
    if (ungapped_host) *ungapped_host = u;
    if (ungapped_count) *ungapped_count = static_cast<int64_t>(uv.size());
    return BLASTP_OK;
  }
  int64_t n = 0;
  if ((rc = search_sorted_device(q, db, p, s, &n))) return rc;
  blastp_gapped *d_out = nullptr;
  if (pool_malloc_async(&d_out, sizeof(blastp_gapped) * static_cast<size_t>(std::max<int64_t>(n, 1)), s) !=
      cudaSuccess)
    return fail(BLASTP_E_NOMEM, "gapped output");
  int64_t m = 0;
  rc = gapped_device(q, db, db->out, n, gp, s, d_out, n, &m);  // one alignment per HSP at most
  blastp_gapped *h = nullptr;
  blastp_hsp *u = nullptr;
  if (!rc) {
    h = static_cast<blastp_gapped *>(malloc(sizeof(blastp_gapped) * static_cast<size_t>(std::max<int64_t>(m, 1))));
    if (ungapped_host)
      u = static_cast<blastp_hsp *>(malloc(sizeof(blastp_hsp) * static_cast<size_t>(std::max<int64_t>(n, 1))));
    if (!h || (ungapped_host && !u)) rc = fail(BLASTP_E_NOMEM, "host result arrays");
  }
  cudaError_t e = cudaSuccess;
  if (!rc && m > 0)
    e = cudaMemcpyAsync(h, d_out, sizeof(blastp_gapped) * static_cast<size_t>(m), cudaMemcpyDeviceToHost, s);
  if (!rc && e == cudaSuccess && u && n > 0)
    e = cudaMemcpyAsync(u, db->out, sizeof(blastp_hsp) * static_cast<size_t>(n), cudaMemcpyDeviceToHost, s);
  cudaFreeAsync(d_out, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (!rc && e != cudaSuccess) rc = fail(BLASTP_E_CUDA, "gapped result copy: %s", cudaGetErrorString(e));
  if (rc) {
    free(h);
    free(u);
    return rc;
  }
  *out_host = h;
  *out_count = m;
  if (ungapped_host) *ungapped_host = u;
  if (ungapped_count) *ungapped_count = n;
  return BLASTP_OK;
}

// ------------------------------------------------------------------- debug

static int debug_run(const blastp_query_table *q, const blastp_db *db, const blastp_params *p,
                     void *cuda_stream, blastp_hit *hits, int64_t hits_cap, int64_t *n_hits,
                     blastp_hit *passing, int64_t passing_cap, int64_t *n_passing,
                     blastp_hsp *exts, int64_t exts_cap, int64_t *n_exts, int64_t *stats_out,
                     int32_t nstats) {
  int rc = check_pair(q, db, p);
  if (rc) return rc;
  if (hits_cap < 0 || passing_cap < 0 || exts_cap < 0 || (hits_cap && !hits) ||
      (passing_cap && !passing) || (exts_cap && !exts))
    return fail(BLASTP_E_INVALID_ARG, "bad trace buffers");
  DeviceGuard g(db->device);
  cudaStream_t s = static_cast<cudaStream_t>(cuda_stream);
  const int64_t caps[3] = {hits_cap, passing_cap, exts_cap};
  TraceRec *tr[3] = {nullptr, nullptr, nullptr};
  unsigned long long *tcount = nullptr, *hcount = nullptr;
  blastp_hsp *dout = nullptr;
  auto cleanup = [&](int code) {
    for (auto *t : tr) cudaFree(t);
    cudaFree(tcount);
    cudaFree(hcount);
    cudaFree(dout);
    return code;
  };
  for (int k = 0; k < 3; ++k)
    if (cudaMalloc(&tr[k], sizeof(TraceRec) * static_cast<size_t>(std::max<int64_t>(caps[k], 1))) != cudaSuccess)
      return cleanup(fail(BLASTP_E_NOMEM, "trace buffers"));
  if (cudaMalloc(&tcount, (3 + kNumStats) * sizeof(unsigned long long)) != cudaSuccess ||
      cudaMalloc(&hcount, sizeof(unsigned long long)) != cudaSuccess ||
      cudaMalloc(&dout, sizeof(blastp_hsp)) != cudaSuccess)
    return cleanup(fail(BLASTP_E_NOMEM, "trace counters"));
  rc = enqueue_search(q, db, p, s, dout, 0, hcount, tr, caps, tcount);
  if (rc) return cleanup(rc);
  unsigned long long cnt[3 + kNumStats] = {};
  if (cudaMemcpyAsync(cnt, tcount, sizeof(cnt), cudaMemcpyDeviceToHost, s) != cudaSuccess ||
      cudaStreamSynchronize(s) != cudaSuccess)
    return cleanup(fail(BLASTP_E_CUDA, "trace readback: %s", cudaGetErrorString(cudaGetLastError())));
  if (stats_out) {
    for (int i = 0; i < nstats; ++i)
      stats_out[i] = i < kNumStats ? static_cast<int64_t>(cnt[3 + i]) : 0;
    return cleanup(BLASTP_OK);
  }
  int64_t *outs[3] = {n_hits, n_passing, n_exts};
  bool over = false;
  std::vector<TraceRec> buf;
  for (int k = 0; k < 3; ++k) {
    if (outs[k]) *outs[k] = static_cast<int64_t>(cnt[k]);
    const int64_t m = std::min<int64_t>(static_cast<int64_t>(cnt[k]), caps[k]);
    if (static_cast<int64_t>(cnt[k]) > caps[k]) over = true;
    if (m <= 0) continue;
    buf.resize(static_cast<size_t>(m));
    if (cudaMemcpy(buf.data(), tr[k], sizeof(TraceRec) * static_cast<size_t>(m),
                   cudaMemcpyDeviceToHost) != cudaSuccess)
      return cleanup(fail(BLASTP_E_CUDA, "trace copy"));
    for (int64_t i = 0; i < m; ++i) {
      const TraceRec &r = buf[static_cast<size_t>(i)];
      const std::vector<int64_t> &hs = host_sstart(db);
      const auto it = std::upper_bound(hs.begin(), hs.end(), r.sp);
      const int64_t subj = (it - hs.begin()) - 1;
      const int32_t sl = static_cast<int32_t>(r.sp - hs[static_cast<size_t>(subj)]);
      const int32_t sid = static_cast<int32_t>(db->subject_base + subj);
      if (k < 2) {
        blastp_hit h{r.query_id, sid, r.q, sl};
        (k == 0 ? hits : passing)[i] = h;
      } else {
        blastp_hsp h;
        h.query_id = r.query_id;
        h.subject_id = sid;
        h.q_start = r.q - r.llen;
        h.s_start = sl - r.llen;
        h.diagonal = h.s_start - h.q_start;
        h.length = r.llen + p->word_len + r.rlen;
        h.score = r.score;
        exts[i] = h;
      }
    }
  }
  return cleanup(over ? fail(BLASTP_E_CAPACITY, "trace capacity exceeded") : BLASTP_OK);
}

int blastp_debug_trace(const blastp_query_table *q, const blastp_db *db, const blastp_params *p,
                       void *cuda_stream, blastp_hit *hits, int64_t hits_cap, int64_t *n_hits,
                       blastp_hit *passing, int64_t passing_cap, int64_t *n_passing,
                       blastp_hsp *exts, int64_t exts_cap, int64_t *n_exts) {
  return debug_run(q, db, p, cuda_stream, hits, hits_cap, n_hits, passing, passing_cap, n_passing,
                   exts, exts_cap, n_exts, nullptr, 0);
}

int blastp_debug_stats(const blastp_query_table *q, const blastp_db *db, const blastp_params *p,
                       void *cuda_stream, int64_t *stats, int32_t nstats) {
  if (!stats || nstats < 1) return fail(BLASTP_E_INVALID_ARG, "stats buffer");
  return debug_run(q, db, p, cuda_stream, nullptr, 0, nullptr, nullptr, 0, nullptr, nullptr, 0,
                   nullptr, stats, nstats);
}

int blastp_trim_memory(int device) {
  DeviceGuard g(device);
  if (g.err != cudaSuccess) return fail(BLASTP_E_CUDA, "cudaSetDevice(%d): %s", device, cudaGetErrorString(g.err));
  CUDA_TRY(pool_trim(device));
  return BLASTP_OK;
}

int blastp_debug_alu_peak(int device, double *lane_ops_per_s) {
  if (!lane_ops_per_s) return fail(BLASTP_E_INVALID_ARG, "output is NULL");
  DeviceGuard g(device);
  if (g.err != cudaSuccess) return fail(BLASTP_E_CUDA, "cudaSetDevice(%d): %s", device, cudaGetErrorString(g.err));
  CUDA_TRY(measure_alu_peak(lane_ops_per_s));
  return BLASTP_OK;
}

int blastp_debug_hits(const blastp_query_table *q, const blastp_db *db, const blastp_params *p,
                      void *cuda_stream, blastp_hit *hits, int64_t cap, int64_t *n) {
  return blastp_debug_trace(q, db, p, cuda_stream, hits, cap, n, nullptr, 0, nullptr, nullptr, 0,
                            nullptr);
}

int blastp_debug_passing(const blastp_query_table *q, const blastp_db *db,
                         const blastp_params *p, void *cuda_stream, blastp_hit *passing,
                         int64_t cap, int64_t *n) {
  return blastp_debug_trace(q, db, p, cuda_stream, nullptr, 0, nullptr, passing, cap, n, nullptr,
                            0, nullptr);
}

}  // extern "C"
