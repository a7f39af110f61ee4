// tools/microbench2.cu — ranking-primitive throughput on sm_100a with 16 independent items per
// thread (the onesweep shape): MATCH.ANY at several digit cardinalities, 8-ballot multisplit,
// 4-ballot (nibble) multisplit, and per-thread private smem counters (LDS+STS).
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/bin/microbench2 tools/microbench2.cu
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t hashu(uint32_t x) {
  x ^= x >> 16; x *= 0x7feb352d; x ^= x >> 15; x *= 0x846ca68b; x ^= x >> 16; return x;
}

template <int MODE>
__global__ void __launch_bounds__(256, 2) k_rank(uint32_t* out, int iters, uint32_t mask, uint32_t seed) {
  __shared__ uint32_t cnt[16 * 256];
  for (int i = threadIdx.x; i < 16 * 256; i += blockDim.x) cnt[i] = 0;
  __syncthreads();
  uint32_t acc = 0;
  const int lane = threadIdx.x & 31;
  for (int it = 0; it < iters; ++it) {
    uint32_t d[16];
#pragma unroll
    for (int i = 0; i < 16; ++i) d[i] = hashu(threadIdx.x * 977 + i * 131 + it * 7919 + seed) & mask;
    if (MODE == 0) {  // MATCH.ANY
      uint32_t p[16];
#pragma unroll
      for (int i = 0; i < 16; ++i) p[i] = __match_any_sync(0xffffffffu, d[i]);
#pragma unroll
      for (int i = 0; i < 16; ++i) acc += __popc(p[i] & ((1u << lane) - 1));
    } else if (MODE == 1 || MODE == 2) {  // ballot multisplit over 8 (MODE 1) or 4 (MODE 2) bits
      constexpr int BITS = (MODE == 1) ? 8 : 4;
      uint32_t p[16];
#pragma unroll
      for (int i = 0; i < 16; ++i) p[i] = 0xffffffffu;
#pragma unroll
      for (int b = 0; b < BITS; ++b) {
#pragma unroll
        for (int i = 0; i < 16; ++i) {
          const uint32_t bal = __ballot_sync(0xffffffffu, (d[i] >> b) & 1u);
          p[i] &= ((d[i] >> b) & 1u) ? bal : ~bal;
        }
      }
#pragma unroll
      for (int i = 0; i < 16; ++i) acc += __popc(p[i] & ((1u << lane) - 1));
    } else {  // private per-thread counters in smem, 16 bins (nibble): LDS + STS per key
#pragma unroll
      for (int i = 0; i < 16; ++i) {
        uint32_t* c = &cnt[(d[i] & 15u) * 256 + threadIdx.x];
        const uint32_t v = *c;
        *c = v + 1;
        acc += v;
      }
    }
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

int main() {
  uint32_t* out;
  cudaMalloc(&out, 148 * 2 * 256 * 4);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const int iters = 400, grid = 148 * 2, threads = 256;
  const double items = (double)grid * threads * iters * 16;  // keys ranked
  auto run = [&](const char* name, auto kern, uint32_t mask) {
    kern<<<grid, threads>>>(out, iters, mask, 1);
    cudaEventRecord(a);
    kern<<<grid, threads>>>(out, iters, mask, 2);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    const double cyc = ms * 1e-3 * 1.965e9 * 148;  // SM-cycles
    printf("%-28s %8.3f ms  %.3f SM-cycles/key  (%.0f keys/SM-cycle*1000)\n", name, ms, cyc / items,
           1000 * items / cyc);
  };
  run("match.any 256 values", k_rank<0>, 255u);
  run("match.any 16 values", k_rank<0>, 15u);
  run("match.any 4 values", k_rank<0>, 3u);
  run("match.any 1 value", k_rank<0>, 0u);
  run("ballot multisplit 8 bits", k_rank<1>, 255u);
  run("ballot multisplit 4 bits", k_rank<2>, 15u);
  run("private smem counters 4b", k_rank<3>, 15u);
  printf("err=%s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
