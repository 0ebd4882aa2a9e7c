// micro.cu -- the on-chip roof the bench reports beside the HBM roofline:
// the device's integer-ALU throughput, measured (not a datasheet number).
//
// Every SM runs 32 warps (the search kernel's residency) of independent
// integer add / xor chains -- the instruction classes the search kernel's
// integer work compiles to -- and the result is lane instructions per second
// (one integer operation each), the unit in which SURVEY.md 8(d) states the
// method's work (ops per residue / hit / extension step).
#include <cuda_runtime.h>

#include "common.cuh"

namespace blastp {
namespace {

constexpr int kAluIters = 4096;

// 16 independent integer instructions per iteration (8 chains x {add, xor}),
// each its own volatile asm statement so ptxas keeps them one SASS
// instruction each (IADD3 / LOP3: the ALU pipe; ptxas may move adds to the
// FMA pipe as IMAD.IADD, as it does in the search kernel).
#define ALU2(x, y)                                       \
  asm volatile("add.u32 %0, %0, %1;" : "+r"(x) : "r"(y)); \
  asm volatile("xor.b32 %0, %0, %1;" : "+r"(x) : "r"(y));
__global__ void __launch_bounds__(1024) alu_peak_kernel(unsigned *out, unsigned seed) {
  unsigned a = threadIdx.x ^ seed, b = a * 3u + 1u, c = a * 5u + 7u, d = a * 9u + 3u;
  unsigned e = a + 11u, f = b ^ 0x55u, g = c + 0x1234u, h = d ^ 0xf0f0u;
  const unsigned k = seed * 2654435761u + 1u;
#pragma unroll 4
  for (int i = 0; i < kAluIters; ++i) {
    ALU2(a, k) ALU2(b, k) ALU2(c, k) ALU2(d, k) ALU2(e, k) ALU2(f, k) ALU2(g, k) ALU2(h, k)
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = a ^ b ^ c ^ d ^ e ^ f ^ g ^ h;
}
#undef ALU2

}  // namespace

// lane operations per second of integer add / logic / multiply-add work.
cudaError_t measure_alu_peak(double *lane_ops_per_s) {
  int dev = 0, sms = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e == cudaSuccess) e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  if (e != cudaSuccess) return e;
  unsigned *out = nullptr;
  if ((e = cudaMalloc(&out, sizeof(unsigned) * size_t(sms) * 1024)) != cudaSuccess) return e;
  cudaEvent_t t0, t1;
  cudaEventCreate(&t0);
  cudaEventCreate(&t1);
  alu_peak_kernel<<<sms, 1024>>>(out, 1u);  // warm-up (clocks up)
  alu_peak_kernel<<<sms, 1024>>>(out, 2u);
  cudaEventRecord(t0);
  const int reps = 20;
  for (int r = 0; r < reps; ++r) alu_peak_kernel<<<sms, 1024>>>(out, 3u + r);
  cudaEventRecord(t1);
  e = cudaEventSynchronize(t1);
  float ms = 0.f;
  if (e == cudaSuccess) e = cudaEventElapsedTime(&ms, t0, t1);
  cudaEventDestroy(t0);
  cudaEventDestroy(t1);
  cudaFree(out);
  if (e != cudaSuccess) return e;
  // 16 integer instructions per thread per iteration
  const double ops = double(reps) * sms * 1024.0 * kAluIters * 16.0;
  *lane_ops_per_s = ops / (double(ms) * 1e-3);
  return cudaSuccess;
}

}  // namespace blastp
