// pack.cu -- GPU side of blastp_pack_db: ASCII residues -> sentinel-separated
// 1-byte code stream (R1), the coalesced residue-major layout the hit
// detector scans (consecutive lanes read consecutive positions).
#include <cuda_runtime.h>

#include "common.cuh"

namespace blastp {

namespace {

__constant__ uint8_t c_encode[256];

// One warp per subject (grid-stride): lanes copy consecutive bytes, so every
// load and store instruction of a warp touches one or two 32-byte sectors.
// The encode table is staged in shared memory: lanes look up different
// letters, which a __constant__ table would serialise (one address per
// cycle); four bytes per lane are in flight per iteration.
// Every byte of the stream is written here (no separate memset, which as a
// kernel would queue behind a running search and hold up the copies of a
// pipelined blastp_search_host_db): the front pad, each subject followed by
// its sentinel, and the back pad up to stream_len.
__global__ void pack_kernel(const uint8_t *__restrict__ ascii, const int64_t *__restrict__ off,
                            int64_t n, const int64_t *__restrict__ sstart,
                            uint8_t *__restrict__ stream, int64_t stream_len, int *err) {
  __shared__ uint8_t lut[256];
  for (int i = threadIdx.x; i < 256; i += blockDim.x) lut[i] = c_encode[i];
  __syncthreads();
  const int lane = threadIdx.x & 31;
  const int64_t gtid = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  const int64_t nthreads = int64_t(gridDim.x) * blockDim.x;
  const int64_t warps = nthreads >> 5;
  const int64_t base = off[0];
  // pads: [0, kStreamPadFront) and [pad + residues + n, stream_len)
  const int64_t tail = kStreamPadFront + (off[n] - base) + n;
  for (int64_t j = gtid; j < kStreamPadFront; j += nthreads) stream[j] = uint8_t(kSentinel);
  for (int64_t j = tail + gtid; j < stream_len; j += nthreads) stream[j] = uint8_t(kSentinel);
  for (int64_t i = gtid >> 5; i < n; i += warps) {
    const int64_t a = off[i] - base, len = off[i + 1] - off[i];
    uint8_t *dst = stream + sstart[i];
    const uint8_t *src = ascii + a;
    int bad = 0;
    int64_t j = lane;
    for (; j + 96 < len; j += 128) {
      const uint8_t c0 = __ldg(src + j), c1 = __ldg(src + j + 32), c2 = __ldg(src + j + 64),
                    c3 = __ldg(src + j + 96);
      const uint8_t e0 = lut[c0], e1 = lut[c1], e2 = lut[c2], e3 = lut[c3];
      bad |= (e0 == 0xFF) | (e1 == 0xFF) | (e2 == 0xFF) | (e3 == 0xFF);
      dst[j] = e0;
      dst[j + 32] = e1;
      dst[j + 64] = e2;
      dst[j + 96] = e3;
    }
    for (; j < len; j += 32) {
      const uint8_t c = lut[__ldg(src + j)];
      bad |= (c == 0xFF);
      dst[j] = c;
    }
    if (lane == 0 && len >= 0) dst[len] = uint8_t(kSentinel);
    if (__any_sync(0xffffffffu, bad) && lane == 0) atomicOr(err, 1);
  }
}

// Stream layout: subject i starts at pad + (off[i] - off[0]) + i (one sentinel
// after each subject).  Also validates the lengths (err bit 2: negative,
// bit 4: longer than BLASTP_MAX_SUBJECT_LEN).
__global__ void layout_kernel(const int64_t *__restrict__ off, int64_t n, int64_t *sstart,
                              int *err) {
  const int64_t base = off[0];
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n;
       i += int64_t(gridDim.x) * blockDim.x) {
    const int64_t o = off[i], L = off[i + 1] - o;
    sstart[i] = kStreamPadFront + (o - base) + i;
    if (L < 0) atomicOr(err, 2);
    if (L > BLASTP_MAX_SUBJECT_LEN) atomicOr(err, 4);
  }
}

// Chunk k = the subjects whose first residue lies in [target(k),
// target(k+1)) of the shard's residues (ChunkPlan; binary search over the
// offsets); empty chunks have start == end and are skipped by the kernels.
__global__ void chunk_kernel(const int64_t *__restrict__ off, int64_t n,
                             const int64_t *__restrict__ sstart, ChunkPlan plan,
                             Chunk *chunks, Chunk *long_chunks, int *nlong) {
  const int64_t base = off[0];
  const int64_t nchunks = plan.nchunks;
  auto first_at = [&](int64_t k) -> int64_t {
    if (k >= nchunks) return n;
    const int64_t target = chunk_target(plan, k);
    int64_t lo = 0, hi = n;
    while (lo < hi) {
      const int64_t m = (lo + hi) >> 1;
      if (off[m] - base >= target) hi = m; else lo = m + 1;
    }
    return lo;
  };
  for (int64_t k = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; k < nchunks;
       k += int64_t(gridDim.x) * blockDim.x) {
    const int64_t f = first_at(k), l = first_at(k + 1);
    Chunk c;
    c.first_subj = f;
    c.last_subj = l > f ? l : f;
    if (l > f) {
      c.start = sstart[f];
      c.end = sstart[l - 1] + (off[l] - off[l - 1]);
    } else {
      c.start = c.end = 0;
    }
    // chunks much longer than C (long subjects) are scheduled first, so the
    // single warp walking one never becomes the tail of the launch
    if (c.end - c.start > 2 * (chunk_target(plan, k + 1) - chunk_target(plan, k))) {
      long_chunks[atomicAdd(nlong, 1)] = c;
      c.start = c.end = 0;
    }
    chunks[k] = c;
  }
}

}  // namespace

cudaError_t launch_layout(const int64_t *off, int64_t n, const ChunkPlan &plan, int64_t *sstart,
                          Chunk *chunks, Chunk *long_chunks, int *nlong, int *err,
                          cudaStream_t s) {
  const int64_t nchunks = plan.nchunks;
  if (n > 0) {
    const int64_t blocks = (n + 255) / 256 > 4096 ? 4096 : (n + 255) / 256;
    layout_kernel<<<unsigned(blocks), 256, 0, s>>>(off, n, sstart, err);
  }
  if (nchunks > 0) {
    const int64_t blocks = (nchunks + 255) / 256 > 4096 ? 4096 : (nchunks + 255) / 256;
    chunk_kernel<<<unsigned(blocks), 256, 0, s>>>(off, n, sstart, plan, chunks, long_chunks,
                                                  nlong);
  }
  return cudaGetLastError();
}

// Once per device: cudaMemcpyToSymbol is synchronous on the legacy default
// stream, so calling it per pack would wait for searches running there (it
// serialised the pipelined blastp_search_host_db).
void upload_encode_table() {
  static unsigned long long ready = 0;  // one bit per device
  int dev = 0;
  cudaGetDevice(&dev);
  if (ready >> dev & 1ull) return;
  uint8_t lut[256];
  for (int i = 0; i < 256; ++i) lut[i] = 0xFF;
  for (int k = 0; k < kNumLetters; ++k) {
    const unsigned char c = static_cast<unsigned char>(kAlphabet[k]);
    lut[c] = uint8_t(k);
    if (c >= 'A' && c <= 'Z') lut[c - 'A' + 'a'] = uint8_t(k);
  }
  const uint8_t x = 22;  // 'X'
  for (const char c : {'U', 'O', 'J', 'u', 'o', 'j'}) lut[static_cast<unsigned char>(c)] = x;
  if (cudaMemcpyToSymbol(c_encode, lut, sizeof(lut)) == cudaSuccess) ready |= 1ull << dev;
}

cudaError_t launch_pack(const uint8_t *ascii, const int64_t *off, int64_t n, const int64_t *sstart,
                        uint8_t *stream, int64_t stream_len, int *err, cudaStream_t s) {
  if (n <= 0) return cudaMemsetAsync(stream, kSentinel, static_cast<size_t>(stream_len), s);
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const int threads = 256;
  int64_t blocks = (n * 32 + threads - 1) / threads;
  const int64_t cap = int64_t(sms) * 16;
  if (blocks > cap) blocks = cap;
  pack_kernel<<<unsigned(blocks), threads, 0, s>>>(ascii, off, n, sstart, stream, stream_len, err);
  return cudaGetLastError();
}

}  // namespace blastp
