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
  // every allocation checked: a failed one frees the others and returns
  // cudaErrorMemoryAllocation (the C-ABI maps it to BLASTP_E_NOMEM)
  if ((e = pool_malloc_async(&idx, bytes, s)) == cudaSuccess &&
      (e = pool_malloc_async(&idx2, bytes, s)) == cudaSuccess &&
      (e = pool_malloc_async(&key, bytes, s)) == cudaSuccess &&
      (e = pool_malloc_async(&key2, bytes, s)) == cudaSuccess &&
      (e = pool_malloc_async(&tmp, size_t(n) * sizeof(blastp_hsp), s)) == cudaSuccess &&
      (e = pool_malloc_async(&temp, temp_bytes, s)) == cudaSuccess) {
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
  for (void *ptr : {static_cast<void *>(idx), static_cast<void *>(idx2), static_cast<void *>(key),
                    static_cast<void *>(key2), static_cast<void *>(tmp), temp})
    if (ptr) cudaFreeAsync(ptr, s);
  if (e != cudaSuccess) {
    cudaGetLastError();  // clear a sticky allocation error
    return e;
  }
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
  if ((e = pool_malloc_async(&tmp, size_t(n) * sizeof(blastp_hsp), s)) == cudaSuccess &&
      (e = pool_malloc_async(&temp, temp_bytes, s)) == cudaSuccess) {
    e = cub::DeviceSelect::Unique(temp, temp_bytes, d, tmp, d_n_out, n, s);
    if (e == cudaSuccess)
      e = cudaMemcpyAsync(d, tmp, size_t(n) * sizeof(blastp_hsp), cudaMemcpyDeviceToDevice, s);
  }
  if (tmp) cudaFreeAsync(tmp, s);
  if (temp) cudaFreeAsync(temp, s);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return e;
  }
  return cudaGetLastError();
}

namespace {

// One thread per sorted seed record; the first record of each (query,
// subject, diagonal) run walks the run in seed order with Alg. 3's ext_reach
// chain (L19-23, R10) and appends the kept records with score >= cutoff as
// canonical HSPs.  Runs are short (a few extensions per diagonal).
__global__ void covered_walk_kernel(const blastp_hsp *rec, int64_t n, int32_t cutoff,
                                    blastp_hsp *out, unsigned long long *count) {
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n;
       i += int64_t(gridDim.x) * blockDim.x) {
    const blastp_hsp &r = rec[i];
    if (i > 0) {
      const blastp_hsp &p = rec[i - 1];
      if (p.query_id == r.query_id && p.subject_id == r.subject_id && p.diagonal == r.diagonal)
        continue;  // not the first record of its diagonal
    }
    int64_t reach = INT64_MIN;
    for (int64_t j = i; j < n; ++j) {
      const blastp_hsp &x = rec[j];
      if (x.query_id != r.query_id || x.subject_id != r.subject_id || x.diagonal != r.diagonal)
        break;
      const int64_t seed_s = int64_t(x.diagonal) + x.q_start;
      if (seed_s <= reach) continue;  // covered by the last kept extension (Alg. 3 L19)
      const int32_t q_start = x.q_start - x.s_start;  // s_start holds llen
      reach = int64_t(x.diagonal) + q_start + x.length - 1;  // its subject end
      if (x.score >= cutoff) {
        blastp_hsp h = x;
        h.q_start = q_start;
        h.s_start = q_start + x.diagonal;
        out[atomicAdd(count, 1ull)] = h;
      }
    }
  }
}

}  // namespace

cudaError_t dedup_covered(blastp_hsp *d, int64_t n, int32_t cutoff, int64_t *d_n_out,
                          cudaStream_t s) {
  cudaError_t e = cudaMemsetAsync(d_n_out, 0, sizeof(int64_t), s);
  if (e != cudaSuccess || n <= 0) return e;
  // (query, subject, diagonal, q_seed, ...) lexicographic = seed order per diagonal
  if ((e = sort_hsps(d, n, s)) != cudaSuccess) return e;
  blastp_hsp *tmp = nullptr;
  if ((e = pool_malloc_async(&tmp, size_t(n) * sizeof(blastp_hsp), s)) != cudaSuccess) {
    cudaGetLastError();
    return e;
  }
  const int blocks = int((n + 255) / 256 > 4096 ? 4096 : (n + 255) / 256);
  covered_walk_kernel<<<blocks, 256, 0, s>>>(d, n, cutoff, tmp,
                                             reinterpret_cast<unsigned long long *>(d_n_out));
  e = cudaGetLastError();
  int64_t kept = 0;
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(&kept, d_n_out, sizeof(kept), cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e == cudaSuccess && kept > 0)
    e = cudaMemcpyAsync(d, tmp, size_t(kept) * sizeof(blastp_hsp), cudaMemcpyDeviceToDevice, s);
  cudaFreeAsync(tmp, s);
  if (e == cudaSuccess) e = sort_hsps(d, kept, s);  // canonical order (R11)
  return e;
}

}  // namespace blastp
