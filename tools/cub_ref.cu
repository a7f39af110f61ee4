// tools/cub_ref.cu — context measurement only (not product code): CUB DeviceRadixSort::SortKeys
// on 2^30 uint64 keys on this B200, the library baseline our hand-written onesweep is compared to.
#include <cub/device/device_radix_sort.cuh>
#include <cstdio>
#include <cstdint>
#include <vector>
__global__ void fill(uint64_t* k, uint64_t n) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t z = i * 0x9E3779B97F4A7C15ull + 12345;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull; z = (z ^ (z >> 27)) * 0x94D049BB133111EBull; z ^= z >> 31;
    double d = (double)(z >> 11) * 0x1.0p-53;  // U[0,1) like the bench
    uint64_t u = __double_as_longlong(d);
    k[i] = u | 0x8000000000000000ull;          // order-preserving key of a non-negative double
  }
}
int main(int argc, char** argv) {
  uint64_t n = argc > 1 ? strtoull(argv[1], 0, 0) : (1ull << 30);
  uint64_t *a, *b; cudaMalloc(&a, n * 8); cudaMalloc(&b, n * 8);
  fill<<<148 * 8, 256>>>(a, n);
  void* tmp = nullptr; size_t tb = 0;
  cub::DoubleBuffer<uint64_t> db(a, b);
  cub::DeviceRadixSort::SortKeys(tmp, tb, db, (int)n);
  cudaMalloc(&tmp, tb);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  for (int r = 0; r < 3; ++r) { fill<<<148 * 8, 256>>>(db.Current(), n); cub::DeviceRadixSort::SortKeys(tmp, tb, db, (int)n); }
  float best = 1e9;
  for (int r = 0; r < 5; ++r) {
    fill<<<148 * 8, 256>>>(db.Current(), n);
    cudaEventRecord(e0);
    cub::DeviceRadixSort::SortKeys(tmp, tb, db, (int)n);
    cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms;
  }
  printf("{\"cub_sortkeys_u64_n\": %llu, \"ms\": %.3f, \"keys_per_s\": %.4g, \"err\": \"%s\"}\n",
         (unsigned long long)n, best, n / (best * 1e-3), cudaGetErrorString(cudaGetLastError()));
  return 0;
}
