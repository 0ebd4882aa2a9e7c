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
__global__ void pack_kernel(const uint8_t *__restrict__ ascii, const int64_t *__restrict__ off,
                            int64_t n, const int64_t *__restrict__ sstart,
                            uint8_t *__restrict__ stream, int *err) {
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t(gridDim.x) * blockDim.x) >> 5;
  const int64_t base = off[0];
  for (int64_t i = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5; i < n; i += warps) {
    const int64_t a = off[i] - base, len = off[i + 1] - off[i];
    uint8_t *dst = stream + sstart[i];
    int bad = 0;
    for (int64_t j = lane; j < len; j += 32) {
      const uint8_t c = c_encode[__ldg(ascii + a + j)];
      bad |= (c == 0xFF);
      dst[j] = c;
    }
    if (__any_sync(0xffffffffu, bad) && lane == 0) atomicOr(err, 1);
  }
}

}  // namespace

void upload_encode_table() {
  uint8_t lut[256];
  for (int i = 0; i < 256; ++i) lut[i] = 0xFF;
  for (int k = 0; k < kNumLetters; ++k) {
    const unsigned char c = static_cast<unsigned char>(kAlphabet[k]);
    lut[c] = uint8_t(k);
    if (c >= 'A' && c <= 'Z') lut[c - 'A' + 'a'] = uint8_t(k);
  }
  const uint8_t x = 22;  // 'X'
  for (const char c : {'U', 'O', 'J', 'u', 'o', 'j'}) lut[static_cast<unsigned char>(c)] = x;
  cudaMemcpyToSymbol(c_encode, lut, sizeof(lut));
}

cudaError_t launch_pack(const uint8_t *ascii, const int64_t *off, int64_t n, const int64_t *sstart,
                        uint8_t *stream, int *err, cudaStream_t s) {
  if (n <= 0) return cudaSuccess;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const int threads = 256;
  int64_t blocks = (n * 32 + threads - 1) / threads;
  const int64_t cap = int64_t(sms) * 16;
  if (blocks > cap) blocks = cap;
  pack_kernel<<<unsigned(blocks), threads, 0, s>>>(ascii, off, n, sstart, stream, err);
  return cudaGetLastError();
}

}  // namespace blastp
