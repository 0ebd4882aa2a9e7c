// Microbenchmark: throughput of __match_any_sync, __reduce_or_sync, __shfl_sync
// and shared-memory loads on one B200 (all SMs, 32 warps per SM).
#include <cstdio>
#include <cuda_runtime.h>

template <int kOp>
__global__ void __launch_bounds__(1024) bench(unsigned *out, int iters, unsigned seed) {
  __shared__ unsigned sm[4096];
  for (int i = threadIdx.x; i < 4096; i += blockDim.x) sm[i] = i * 2654435761u;
  __syncthreads();
  unsigned v0 = (threadIdx.x * 2654435761u) ^ seed, v1 = v0 * 3, v2 = v0 * 5, v3 = v0 * 7;
  unsigned acc = 0;
  for (int i = 0; i < iters; ++i) {
    if (kOp == 0) {  // 4 independent MATCH.ANY per iteration
      acc += __match_any_sync(0xffffffffu, v0 & 1023) + __match_any_sync(0xffffffffu, v1 & 1023) +
             __match_any_sync(0xffffffffu, v2 & 1023) + __match_any_sync(0xffffffffu, v3 & 1023);
    } else if (kOp == 1) {
      acc += __reduce_or_sync(0xffffffffu, v0) + __reduce_or_sync(0xffffffffu, v1) +
             __reduce_or_sync(0xffffffffu, v2) + __reduce_or_sync(0xffffffffu, v3);
    } else if (kOp == 2) {
      acc += __shfl_sync(0xffffffffu, v0, v1 & 31) + __shfl_sync(0xffffffffu, v1, v2 & 31) +
             __shfl_sync(0xffffffffu, v2, v3 & 31) + __shfl_sync(0xffffffffu, v3, v0 & 31);
    } else if (kOp == 3) {
      acc += sm[v0 & 4095] + sm[v1 & 4095] + sm[v2 & 4095] + sm[v3 & 4095];
    } else {  // 4 dependent MATCH.ANY (latency)
      unsigned x = v0;
      x = __match_any_sync(0xffffffffu, x & 1023);
      x = __match_any_sync(0xffffffffu, x & 1023);
      x = __match_any_sync(0xffffffffu, x & 1023);
      x = __match_any_sync(0xffffffffu, x & 1023);
      acc += x;
      v0 = x;
    }
    v0 = v0 * 1664525u + 1013904223u; v1 = v1 * 1664525u + 1013904223u;
    v2 = v2 * 1664525u + 1013904223u; v3 = v3 * 1664525u + 1013904223u;
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

template <int kOp>
void run(const char *name, int warps_per_block) {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  unsigned *out;
  cudaMalloc(&out, sizeof(unsigned) * sms * 1024);
  const int iters = 20000;
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  bench<kOp><<<sms, warps_per_block * 32>>>(out, 100, 1);
  cudaEventRecord(a);
  bench<kOp><<<sms, warps_per_block * 32>>>(out, iters, 2);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms = 0;
  cudaEventElapsedTime(&ms, a, b);
  int clk = 0;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  const double cycles = ms * 1e-3 * clk * 1e3;
  const double ops_per_sm = double(iters) * 4 * warps_per_block;
  printf("%-28s warps/SM %2d: %.2f SM-cycles per warp-op (%.1f ms)\n", name, warps_per_block,
         cycles / ops_per_sm, ms);
  cudaFree(out);
}

int main() {
  for (int w : {1, 8, 32}) {
    run<0>("match.any (independent)", w);
    run<4>("match.any (dependent)", w);
    run<1>("redux.or", w);
    run<2>("shfl.idx", w);
    run<3>("lds (random)", w);
  }
  return 0;
}
