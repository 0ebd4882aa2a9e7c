// table.cu -- query lookup table (R3) built on the GPU: for every word v of
// the 24^3 words and every query position q, v neighbours the query word at
// q iff sum_i BLOSUM62[query[q+i]][v_i] >= T (the
// function of the paper's DFA).  CSR layout as the search kernels read it:
// woff[v] .. woff[v+1] index qpos[], which lists q in ascending order.
//
// Thread per word: it walks the query once to count (pass 1) and once to
// write its positions (pass 2); in between, an inclusive scan of the counts
// gives the offsets.  The query codes are read warp-uniformly (broadcast)
// and the matrix is staged transposed, BT[query letter][word letter], so the
// lanes of a warp (consecutive words: same first letter, one or two second
// letters, different third letters) hit distinct banks or broadcast.
#include <cub/device/device_scan.cuh>
#include <cuda_runtime.h>

#include "common.cuh"

namespace blastp {

namespace {

constexpr int kTableThreads = 128;

struct Matrix {  // BLOSUM62 (R2) by value as a kernel parameter
  int8_t m[kNumLetters * kNumLetters];
};

Matrix blosum62_param() {
  Matrix M;
  for (int a = 0; a < kNumLetters; ++a)
    for (int b = 0; b < kNumLetters; ++b) M.m[a * kNumLetters + b] = kBlosum62[a][b];
  return M;
}

template <bool kFill>
__global__ void __launch_bounds__(kTableThreads)
    table_kernel(const Matrix B, const uint8_t *__restrict__ qcodes, int lq, int T,
                 uint32_t *__restrict__ woff, uint16_t *__restrict__ qpos) {
  // rows for every 5-bit query code: the sentinels between the members of a
  // query group score -1000 against everything (no word touching one)
  __shared__ int bt[32 * 32];
  for (int i = threadIdx.x; i < 32 * 32; i += blockDim.x) {
    const int a = i >> 5, x = i & 31;
    bt[i] = (a < kNumLetters && x < kNumLetters) ? int(B.m[a * kNumLetters + x]) : -1000;
  }
  __syncthreads();
  const int w = blockIdx.x * blockDim.x + threadIdx.x;
  if (w >= kWords) return;
  const int x = w / (kNumLetters * kNumLetters), y = (w / kNumLetters) % kNumLetters,
            z = w % kNumLetters;
  uint32_t k = 0;
  uint32_t base = 0;
  if (kFill) base = woff[w];
  int a0 = __ldg(qcodes), a1 = __ldg(qcodes + 1);
  for (int q = 0; q + 3 <= lq; ++q) {
    const int a2 = __ldg(qcodes + q + 2);
    const int sc = bt[a0 * 32 + x] + bt[a1 * 32 + y] + bt[a2 * 32 + z];
    if (sc >= T) {
      if (kFill) qpos[base + k] = uint16_t(q);
      ++k;
    }
    a0 = a1;
    a1 = a2;
  }
  if (!kFill) woff[w + 1] = k;  // counts; scanned in place into offsets
}

// Radix-32 view of the CSR table for the block kernel (search_block.cu):
// entry (r0 << 10 | r1 << 5 | r2) = (woff[w], count of w) for the word w of
// letters r0 r1 r2 < 24, (0, 0) for any code with a sentinel or unused letter
// -- a word touching a subject boundary neighbours nothing (R4), and the
// kernel needs no letter check; one 8-byte load per subject position.
__global__ void radix32_kernel(const uint32_t *__restrict__ woff, uint2 *__restrict__ wtab) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= 32 * 32 * 32) return;
  const int r0 = c >> 10, r1 = (c >> 5) & 31, r2 = c & 31;
  uint2 v = make_uint2(0u, 0u);
  if (r0 < kNumLetters && r1 < kNumLetters && r2 < kNumLetters) {
    const int w = (r0 * kNumLetters + r1) * kNumLetters + r2;
    v.x = woff[w];
    v.y = woff[w + 1] - woff[w];
  }
  wtab[c] = v;
}

}  // namespace

cudaError_t launch_table_radix32(const uint32_t *woff, uint2 *wtab, cudaStream_t s) {
  radix32_kernel<<<(32 * 32 * 32) / 256, 256, 0, s>>>(woff, wtab);
  return cudaGetLastError();
}

// Builds woff (device, kWords + 1) and returns the entry count on the host;
// then qpos must be allocated with max(total, 1) entries and filled by
// launch_table_fill.  Synchronises `s` once (to read the total).
cudaError_t launch_table_count(const uint8_t *qcodes, int lq, int T, uint32_t *woff,
                               int64_t *total, cudaStream_t s) {
  cudaError_t e = cudaMemsetAsync(woff, 0, sizeof(uint32_t), s);
  if (e != cudaSuccess) return e;
  const int blocks = (kWords + kTableThreads - 1) / kTableThreads;
  table_kernel<false><<<blocks, kTableThreads, 0, s>>>(blosum62_param(), qcodes, lq, T, woff,
                                                        nullptr);
  if ((e = cudaGetLastError()) != cudaSuccess) return e;
  size_t temp_bytes = 0;
  e = cub::DeviceScan::InclusiveSum(nullptr, temp_bytes, woff + 1, woff + 1, kWords, s);
  if (e != cudaSuccess) return e;
  void *temp = nullptr;
  if ((e = pool_malloc_async(&temp, temp_bytes, s)) != cudaSuccess) return e;
  e = cub::DeviceScan::InclusiveSum(temp, temp_bytes, woff + 1, woff + 1, kWords, s);
  cudaFreeAsync(temp, s);
  if (e != cudaSuccess) return e;
  uint32_t h = 0;
  if ((e = cudaMemcpyAsync(&h, woff + kWords, sizeof(h), cudaMemcpyDeviceToHost, s)) != cudaSuccess)
    return e;
  if ((e = cudaStreamSynchronize(s)) != cudaSuccess) return e;
  *total = int64_t(h);
  return cudaSuccess;
}

cudaError_t launch_table_fill(const uint8_t *qcodes, int lq, int T, const uint32_t *woff,
                              uint16_t *qpos, cudaStream_t s) {
  const int blocks = (kWords + kTableThreads - 1) / kTableThreads;
  table_kernel<true><<<blocks, kTableThreads, 0, s>>>(blosum62_param(), qcodes, lq, T,
                                                      const_cast<uint32_t *>(woff), qpos);
  return cudaGetLastError();
}

}  // namespace blastp
