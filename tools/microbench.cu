// tools/microbench.cu — throughput of the ranking primitives on sm_100a (MATCH.ANY vs ballot
// multi-split vs shared atomics), to choose the onesweep ranking scheme.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/mb tools/microbench.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__global__ void k_match(uint32_t* out, int iters, uint32_t seed) {
  uint32_t x[8];
  for (int i = 0; i < 8; ++i) x[i] = (threadIdx.x * 2654435761u + i * 97 + seed) & 255u;
  uint32_t acc = 0;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      uint32_t p = __match_any_sync(0xffffffffu, x[i]);
      acc += p;
      x[i] = (x[i] + (p & 1) + 1) & 255u;
    }
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

__device__ __forceinline__ uint32_t ballot_peers(uint32_t d) {
  uint32_t peers = 0xffffffffu;
#pragma unroll
  for (int b = 0; b < 8; ++b) {
    const bool bit = (d >> b) & 1u;
    const uint32_t bal = __ballot_sync(0xffffffffu, bit);
    peers &= bit ? bal : ~bal;
  }
  return peers;
}

__global__ void k_ballot(uint32_t* out, int iters, uint32_t seed) {
  uint32_t x[8];
  for (int i = 0; i < 8; ++i) x[i] = (threadIdx.x * 2654435761u + i * 97 + seed) & 255u;
  uint32_t acc = 0;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      uint32_t p = ballot_peers(x[i]);
      acc += p;
      x[i] = (x[i] + (p & 1) + 1) & 255u;
    }
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

__global__ void k_atoms(uint32_t* out, int iters, uint32_t seed) {
  __shared__ uint32_t h[8 * 257];
  for (int i = threadIdx.x; i < 8 * 257; i += blockDim.x) h[i] = 0;
  __syncthreads();
  uint32_t x[8];
  for (int i = 0; i < 8; ++i) x[i] = (threadIdx.x * 2654435761u + i * 97 + seed) & 255u;
  uint32_t acc = 0;
  uint32_t* wh = h + (threadIdx.x >> 5) * 257;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      acc += atomicAdd(&wh[x[i]], 1u);
      x[i] = (x[i] * 5u + 1u) & 255u;
    }
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

int main() {
  uint32_t* out;
  cudaMalloc(&out, 148 * 8 * 1024 * 4);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const int iters = 2000;
  for (int blocksPerSm : {2, 4, 8}) {
    int grid = 148 * blocksPerSm, threads = 256;
    double ops = (double)grid * threads / 32 * iters * 8;  // warp-level ops
    for (int k = 0; k < 3; ++k) {
      for (int rep = 0; rep < 2; ++rep) {
        cudaEventRecord(a);
        if (k == 0) k_match<<<grid, threads>>>(out, iters, rep);
        if (k == 1) k_ballot<<<grid, threads>>>(out, iters, rep);
        if (k == 2) k_atoms<<<grid, threads>>>(out, iters, rep);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        if (rep == 1)
          printf("%-7s blocks/SM=%d  %.3f ms  %.2f warp-ops/SM/cycle(1.965GHz)  %.1f cycles/warp-op/SMSP\n",
                 k == 0 ? "match" : (k == 1 ? "ballot" : "atoms"), blocksPerSm, ms,
                 ops / 148 / (ms * 1e-3 * 1.965e9), (ms * 1e-3 * 1.965e9) * 4 / (ops / 148));
      }
    }
  }
  printf("err=%s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
