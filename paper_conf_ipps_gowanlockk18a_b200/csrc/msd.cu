// msd.cu — MSD-first split (the hybrid radix sort idea of [5], PAPER.md
// P:70-72): a batch is partitioned into R key ranges ("buckets") by R - 1 sampled
// splitters while the next batch uploads; the segments of each bucket (one per batch, on every
// GPU) are then gathered to the GPU that owns the bucket -- peer loads over NVLink when the
// segment lies in another GPU's HBM -- and every bucket is LSD-sorted on its own and DMA'd to its
// place in B.  No merge follows: bucket r's keys all precede bucket r+1's.
//
//   K6a k_bucket_count    per 4096-key tile: bucket of each key (upper bound among the splitters,
//                         binary search in shared memory), tile histogram -> counts[tile][R]
//   K6b k_bucket_scan     per bucket: exclusive scan of its column over the tiles, batch total
//   K6c k_bucket_scatter  per tile: slot = batch base of the bucket + tile offset + shared-atomic
//                         rank (order inside a bucket is irrelevant: the bucket is sorted next and
//                         equal keys are bit-identical, reading A-4); the float64 -> key transform
//                         (A4) is applied on load, so buckets hold keys
//   K6d k_gather_segments one CTA per 8192-key piece of a segment list: dst[off + i] = src[i]
//
// HBM bytes per key: K6a 8, K6c 16, K6d 16 (+ the bucket sorts' LSD passes).  All integer.
#include <cuda_runtime.h>

#include <cstdint>

#include "internal.h"

namespace hsort {
namespace {

constexpr int kBkThreads = 256;
constexpr int kBkItems = 16;
constexpr int kBkTile = kBkThreads * kBkItems;  // 4096 keys per tile

__device__ __forceinline__ uint64_t key64(uint64_t u) {
  return u ^ ((uint64_t)((int64_t)u >> 63) | 0x8000000000000000ull);
}

// bucket of key k = number of splitters s < k: bucket r holds (s_{r-1}, s_r], so equal keys always
// share a bucket
__device__ __forceinline__ int bucket_of(const uint64_t* spl, int m, uint64_t k) {
  int lo = 0, hi = m;  // first splitter >= k
  while (lo < hi) {
    const int mid = (lo + hi) >> 1;
    if (spl[mid] < k) lo = mid + 1;
    else hi = mid;
  }
  return lo;
}

template <bool IN_F64>
__global__ void __launch_bounds__(kBkThreads) k_bucket_count(const uint64_t* __restrict__ in,
                                                             uint64_t n,
                                                             const uint64_t* __restrict__ spl,
                                                             int R, uint32_t* __restrict__ counts) {
  extern __shared__ __align__(16) unsigned char smem[];
  uint64_t* s_spl = (uint64_t*)smem;
  uint32_t* s_cnt = (uint32_t*)(s_spl + R);
  for (int i = threadIdx.x; i < R - 1; i += kBkThreads) s_spl[i] = spl[i];
  for (int i = threadIdx.x; i < R; i += kBkThreads) s_cnt[i] = 0;
  __syncthreads();
  const uint64_t base = (uint64_t)blockIdx.x * kBkTile;
#pragma unroll 4
  for (int q = 0; q < kBkItems; ++q) {
    const uint64_t i = base + (uint64_t)q * kBkThreads + threadIdx.x;
    if (i < n) {
      const uint64_t u = __ldcs(in + i);
      atomicAdd(&s_cnt[bucket_of(s_spl, R - 1, IN_F64 ? key64(u) : u)], 1u);
    }
  }
  __syncthreads();
  for (int r = threadIdx.x; r < R; r += kBkThreads) counts[(uint64_t)blockIdx.x * R + r] = s_cnt[r];
}

// one CTA per bucket r: counts[t][r] <- sum_{t' < t} counts[t'][r]; totals[r] = column sum
__global__ void __launch_bounds__(256) k_bucket_scan(uint32_t* __restrict__ counts, uint64_t tiles,
                                                     int R, uint32_t* __restrict__ totals) {
  __shared__ uint32_t s_w[8];
  const int r = blockIdx.x;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  uint32_t carry = 0;
  for (uint64_t t0 = 0; t0 < tiles; t0 += 256) {
    const uint64_t t = t0 + threadIdx.x;
    const uint32_t v = t < tiles ? counts[t * R + r] : 0u;
    uint32_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) s_w[w] = x;
    __syncthreads();
    uint32_t pre = 0, tot = 0;
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      pre += q < w ? s_w[q] : 0u;
      tot += s_w[q];
    }
    if (t < tiles) counts[t * R + r] = carry + pre + x - v;
    carry += tot;
    __syncthreads();
  }
  if (threadIdx.x == 0) totals[r] = carry;
}

template <bool IN_F64>
__global__ void __launch_bounds__(kBkThreads) k_bucket_scatter(
    const uint64_t* __restrict__ in, uint64_t n, const uint64_t* __restrict__ spl, int R,
    const uint32_t* __restrict__ counts, const uint32_t* __restrict__ totals,
    uint64_t* __restrict__ out) {
  extern __shared__ __align__(16) unsigned char smem[];
  uint64_t* s_spl = (uint64_t*)smem;
  uint32_t* s_cur = (uint32_t*)(s_spl + R);  // [R] next slot of each bucket in this tile
  __shared__ uint32_t s_w[kBkThreads / 32];
  for (int i = threadIdx.x; i < R - 1; i += kBkThreads) s_spl[i] = spl[i];
  // bucket bases inside the batch: exclusive scan of totals (chunks of 256 buckets)
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  uint32_t carry = 0;
  for (int r0 = 0; r0 < R; r0 += kBkThreads) {
    const int r = r0 + threadIdx.x;
    const uint32_t v = r < R ? totals[r] : 0u;
    uint32_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) s_w[w] = x;
    __syncthreads();
    uint32_t pre = 0, tot = 0;
#pragma unroll
    for (int q = 0; q < kBkThreads / 32; ++q) {
      pre += q < w ? s_w[q] : 0u;
      tot += s_w[q];
    }
    if (r < R) s_cur[r] = carry + pre + x - v + counts[(uint64_t)blockIdx.x * R + r];
    carry += tot;
    __syncthreads();
  }
  const uint64_t base = (uint64_t)blockIdx.x * kBkTile;
#pragma unroll 4
  for (int q = 0; q < kBkItems; ++q) {
    const uint64_t i = base + (uint64_t)q * kBkThreads + threadIdx.x;
    if (i < n) {
      const uint64_t u = __ldcs(in + i);
      const uint64_t k = IN_F64 ? key64(u) : u;
      const uint32_t slot = atomicAdd(&s_cur[bucket_of(s_spl, R - 1, k)], 1u);
      out[slot] = k;
    }
  }
}

constexpr uint64_t kSegPiece = 8192;

// segs[s] = {src, len, dst offset}; piece_start[s] = first piece of segment s (exclusive scan of
// ceil(len / kSegPiece)), pieces in total; every CTA copies one piece with 16-byte accesses when
// aligned.  src may point into a peer GPU's HBM (peer access enabled): the copy is the exchange.
__global__ void __launch_bounds__(256) k_gather_segments(const GatherSeg* __restrict__ segs,
                                                         const uint64_t* __restrict__ piece_start,
                                                         int nseg, uint64_t* __restrict__ dst) {
  const uint64_t piece = blockIdx.x;
  int lo = 0, hi = nseg - 1;  // last segment with piece_start <= piece
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (piece_start[mid] <= piece) lo = mid;
    else hi = mid - 1;
  }
  const GatherSeg sg = segs[lo];
  const uint64_t o = (piece - piece_start[lo]) * kSegPiece;
  if (o >= sg.len) return;
  const uint64_t len = sg.len - o < kSegPiece ? sg.len - o : kSegPiece;
  const uint64_t* s = sg.src + o;
  uint64_t* d = dst + sg.dst_off + o;
  if ((((uintptr_t)s | (uintptr_t)d) & 15) == 0) {
    const ulonglong2* s2 = (const ulonglong2*)s;
    ulonglong2* d2 = (ulonglong2*)d;
    for (uint64_t i = threadIdx.x; i < len / 2; i += blockDim.x) d2[i] = __ldcs(s2 + i);
    if (threadIdx.x == 0 && (len & 1)) d[len - 1] = s[len - 1];
  } else {
    for (uint64_t i = threadIdx.x; i < len; i += blockDim.x) d[i] = __ldcs(s + i);
  }
}

}  // namespace

uint64_t bucket_count_elems(uint64_t n, int R) {
  return ((n + kBkTile - 1) / kBkTile) * (uint64_t)R;
}

cudaError_t bucket_partition(const uint64_t* in, uint64_t n, bool in_f64, const uint64_t* d_spl,
                             int R, uint32_t* counts, uint32_t* totals, uint64_t* out,
                             cudaStream_t st) {
  if (R < 1 || R > kMaxBuckets) return cudaErrorInvalidValue;
  if (n == 0) return cudaMemsetAsync(totals, 0, R * sizeof(uint32_t), st);
  const uint64_t tiles = (n + kBkTile - 1) / kBkTile;
  const size_t smem = (size_t)R * 8 + (size_t)R * 4;
  if (in_f64) k_bucket_count<true><<<(unsigned)tiles, kBkThreads, smem, st>>>(in, n, d_spl, R, counts);
  else k_bucket_count<false><<<(unsigned)tiles, kBkThreads, smem, st>>>(in, n, d_spl, R, counts);
  cudaError_t e = launched();
  if (e != cudaSuccess) return e;
  k_bucket_scan<<<R, 256, 0, st>>>(counts, tiles, R, totals);
  if ((e = launched()) != cudaSuccess) return e;
  if (in_f64)
    k_bucket_scatter<true><<<(unsigned)tiles, kBkThreads, smem, st>>>(in, n, d_spl, R, counts, totals, out);
  else
    k_bucket_scatter<false><<<(unsigned)tiles, kBkThreads, smem, st>>>(in, n, d_spl, R, counts, totals, out);
  return launched();
}

uint64_t gather_pieces(uint64_t len) { return (len + kSegPiece - 1) / kSegPiece; }

cudaError_t gather_segments(const GatherSeg* d_segs, const uint64_t* d_piece_start, int nseg,
                            uint64_t pieces, uint64_t* dst, cudaStream_t st) {
  if (nseg == 0 || pieces == 0) return cudaSuccess;
  k_gather_segments<<<(unsigned)pieces, 256, 0, st>>>(d_segs, d_piece_start, nseg, dst);
  return launched();
}

}  // namespace hsort
