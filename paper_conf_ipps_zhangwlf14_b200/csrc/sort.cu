// sort.cu -- canonical order of HSP lists on the GPU (R11): lexicographic on
// (query_id, subject_id, diagonal, q_start, s_start, length, score).
// s_start = q_start + diagonal and the score is a function of the segment,
// so five stable LSD passes (length, q_start, diagonal, subject_id,
// query_id) give the full 7-field order.  The first four fields alone are
// not unique: a later seed of a diagonal lies beyond the previous HSP's end,
// but its left extension may reach back to the same start (and ext_mode HIT
// returns one extension per seed, R14).  Output formatting only -- not part
// of the timed hot path.
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_select.cuh>
#include <cuda_runtime.h>

#include "common.cuh"

// record equality (all 7 fields) for cub::DeviceSelect::Unique
__host__ __device__ inline bool operator==(const blastp_hsp &a, const blastp_hsp &b) {
  return a.query_id == b.query_id && a.subject_id == b.subject_id && a.diagonal == b.diagonal &&
         a.q_start == b.q_start && a.s_start == b.s_start && a.length == b.length &&
         a.score == b.score;
}

namespace blastp {

namespace {

__global__ void iota_kernel(uint32_t *idx, int64_t n) {
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n;
       i += int64_t(gridDim.x) * blockDim.x)
    idx[i] = uint32_t(i);
}

// order-preserving u32 key of field f (signed -> flip sign bit)
__global__ void key_kernel(const blastp_hsp *h, const uint32_t *idx, uint32_t *key, int64_t n,
                           int f) {
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n;
       i += int64_t(gridDim.x) * blockDim.x) {
    const int32_t *r = reinterpret_cast<const int32_t *>(h + idx[i]);
    key[i] = uint32_t(r[f]) ^ 0x80000000u;
  }
}

__global__ void gather_kernel(const blastp_hsp *src, const uint32_t *idx, blastp_hsp *dst,
                              int64_t n) {
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n;
       i += int64_t(gridDim.x) * blockDim.x)
    dst[i] = src[idx[i]];
}

}  // namespace

cudaError_t sort_hsps(blastp_hsp *d, int64_t n, cudaStream_t s) {
  if (n <= 1) return cudaSuccess;
  if (n > int64_t(0x7fffffff)) return cudaErrorInvalidValue;
  const int ni = int(n);
  uint32_t *idx = nullptr, *idx2 = nullptr, *key = nullptr, *key2 = nullptr;
  blastp_hsp *tmp = nullptr;
  void *temp = nullptr;
  size_t temp_bytes = 0;
  cudaError_t e = cub::DeviceRadixSort::SortPairs(nullptr, temp_bytes, key, key2, idx, idx2, ni,
                                                  0, 32, s);
  if (e != cudaSuccess) return e;
  const size_t bytes = size_t(n) * sizeof(uint32_t);
  if ((e = cudaMallocAsync(&idx, bytes, s)) != cudaSuccess) return e;
  cudaMallocAsync(&idx2, bytes, s);
  cudaMallocAsync(&key, bytes, s);
  cudaMallocAsync(&key2, bytes, s);
  cudaMallocAsync(&tmp, size_t(n) * sizeof(blastp_hsp), s);
  e = cudaMallocAsync(&temp, temp_bytes, s);
  if (e == cudaSuccess) {
    const int blocks = int((n + 255) / 256 > 4096 ? 4096 : (n + 255) / 256);
    iota_kernel<<<blocks, 256, 0, s>>>(idx, n);
    const int fields[5] = {5, 3, 2, 1, 0};  // length, q_start, diagonal, subject_id, query_id
    for (int f : fields) {
      key_kernel<<<blocks, 256, 0, s>>>(d, idx, key, n, f);
      e = cub::DeviceRadixSort::SortPairs(temp, temp_bytes, key, key2, idx, idx2, ni, 0, 32, s);
      if (e != cudaSuccess) break;
      uint32_t *t = idx; idx = idx2; idx2 = t;
    }
    if (e == cudaSuccess) {
      gather_kernel<<<blocks, 256, 0, s>>>(d, idx, tmp, n);
      e = cudaMemcpyAsync(d, tmp, size_t(n) * sizeof(blastp_hsp), cudaMemcpyDeviceToDevice, s);
    }
  }
  cudaFreeAsync(idx, s);
  cudaFreeAsync(idx2, s);
  cudaFreeAsync(key, s);
  cudaFreeAsync(key2, s);
  cudaFreeAsync(tmp, s);
  cudaFreeAsync(temp, s);
  if (e != cudaSuccess) return e;
  return cudaGetLastError();
}

// Adjacent duplicates of a sorted list collapse to one (cub::DeviceSelect::Unique
// into a temporary, then copied back); the count lands in *d_n_out (device).
cudaError_t unique_hsps(blastp_hsp *d, int64_t n, int64_t *d_n_out, cudaStream_t s) {
  if (n <= 0) return cudaMemsetAsync(d_n_out, 0, sizeof(int64_t), s);
  if (n > int64_t(0x7fffffff)) return cudaErrorInvalidValue;
  blastp_hsp *tmp = nullptr;
  void *temp = nullptr;
  size_t temp_bytes = 0;
  cudaError_t e = cub::DeviceSelect::Unique(nullptr, temp_bytes, d, tmp, d_n_out, n, s);
  if (e != cudaSuccess) return e;
  if ((e = cudaMallocAsync(&tmp, size_t(n) * sizeof(blastp_hsp), s)) != cudaSuccess) return e;
  if ((e = cudaMallocAsync(&temp, temp_bytes, s)) == cudaSuccess) {
    e = cub::DeviceSelect::Unique(temp, temp_bytes, d, tmp, d_n_out, n, s);
    if (e == cudaSuccess)
      e = cudaMemcpyAsync(d, tmp, size_t(n) * sizeof(blastp_hsp), cudaMemcpyDeviceToDevice, s);
  }
  cudaFreeAsync(tmp, s);
  cudaFreeAsync(temp, s);
  if (e != cudaSuccess) return e;
  return cudaGetLastError();
}

}  // namespace blastp
