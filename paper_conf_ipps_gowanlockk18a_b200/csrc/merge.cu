// merge.cu — multiway merge of sorted batches on the GPU (§III-A), with
// merge-path partitioning (ref [18]) generalised to k runs.
//
// The paper merges on the CPU with GNU parallel multiway_merge.  On a B200 whose sorted runs are
// still resident in HBM the merge is an HBM-bound pass (16 B/key), so it runs here:
//
//   K4 k_corank     exact co-ranks (i_0..i_{k-1}) of each output-tile boundary o: the first o
//                   keys of the merge in which equal keys are taken in run order.  One warp per
//                   boundary, lanes own runs; bisection on the key value with per-run index
//                   windows, the value bracket tightened to keys still inside the windows.
//   K5 k_merge_tile each CTA owns one output tile [o_t, o_t+1): loads its k slices into shared
//                   memory, merges them by a pairwise merge-path tree in shared memory, and writes
//                   the tile with coalesced stores (inverse key transform fused).
#include <cuda_runtime.h>

#include <cstdint>

#include "internal.h"

namespace hsort {
namespace {

constexpr int kMaxC = kMaxMergeRuns / 32;

__device__ __forceinline__ uint64_t from_key(uint64_t k) {
  return k ^ ((uint64_t)((int64_t)(~k) >> 63) | 0x8000000000000000ull);
}

__device__ __forceinline__ uint64_t warp_sum(uint64_t v) {
#pragma unroll
  for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}
__device__ __forceinline__ uint64_t warp_min(uint64_t v) {
#pragma unroll
  for (int o = 16; o; o >>= 1) {
    uint64_t w = __shfl_xor_sync(0xffffffffu, v, o);
    v = w < v ? w : v;
  }
  return v;
}
__device__ __forceinline__ uint64_t warp_max(uint64_t v) {
#pragma unroll
  for (int o = 16; o; o >>= 1) {
    uint64_t w = __shfl_xor_sync(0xffffffffu, v, o);
    v = w > v ? w : v;
  }
  return v;
}

// number of elements <= v in a[lo, hi)  (returned as an absolute index)
__device__ __forceinline__ uint64_t upper_bound(const uint64_t* a, uint64_t lo, uint64_t hi,
                                                uint64_t v) {
  while (lo < hi) {
    uint64_t mid = lo + ((hi - lo) >> 1);
    if (a[mid] <= v) lo = mid + 1;
    else hi = mid;
  }
  return lo;
}

// K4.  ranks[b*k + j] = co-rank of run j at output position o_b = min(b*step, total).
template <int C>
__global__ void __launch_bounds__(128) k_corank(const uint64_t* __restrict__ keys,
                                                const uint64_t* __restrict__ off, int k,
                                                uint64_t total, uint64_t step, uint64_t b0,
                                                uint64_t nb, uint64_t* __restrict__ ranks) {
  const uint64_t b = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (b >= nb) return;
  const uint64_t o = (b0 + b) * step < total ? (b0 + b) * step : total;
  uint64_t base[C], lo[C], hi[C];
#pragma unroll
  for (int c = 0; c < C; ++c) {
    int j = c * 32 + lane;
    if (j < k) {
      base[c] = off[j] - off[0];
      lo[c] = 0;
      hi[c] = off[j + 1] - off[j];
    } else {
      base[c] = 0;
      lo[c] = hi[c] = 0;
    }
  }
  const uint64_t* K = keys + off[0];
  uint64_t* out = ranks + b * (uint64_t)k;
  if (o == total) {
#pragma unroll
    for (int c = 0; c < C; ++c)
      if (c * 32 + lane < k) out[c * 32 + lane] = hi[c];
    return;
  }
  // Find v = the key at merged position o: smallest v with count(<= v) > o.
  // Invariant: lo[c] = #(< L) in run, hi[c] = #(<= H) in run, count(<= H) > o, count(< L) <= o.
  uint64_t L = 0, H = ~0ull;
  while (true) {
    // tighten [L, H] to the keys still inside the windows
    uint64_t mn = ~0ull, mx = 0;
#pragma unroll
    for (int c = 0; c < C; ++c) {
      if (hi[c] > lo[c]) {
        uint64_t a = K[base[c] + lo[c]], z = K[base[c] + hi[c] - 1];
        mn = a < mn ? a : mn;
        mx = z > mx ? z : mx;
      }
    }
    mn = warp_min(mn);
    mx = warp_max(mx);
    if (mn > L) L = mn;
    if (mx < H) H = mx;
    if (L >= H) break;
    const uint64_t mid = L + ((H - L) >> 1);
    uint64_t ub[C];
    uint64_t s = 0;
#pragma unroll
    for (int c = 0; c < C; ++c) {
      ub[c] = upper_bound(K + base[c], lo[c], hi[c], mid);
      s += ub[c];
    }
    // elements <= mid overall = (elements < L, i.e. sum lo) + (in-window <= mid): the window
    // search counts from index 0 because lo/hi are absolute.
    s = warp_sum(s);
    if (s > o) {
      H = mid;
#pragma unroll
      for (int c = 0; c < C; ++c) hi[c] = ub[c];
    } else {
      L = mid + 1;
#pragma unroll
      for (int c = 0; c < C; ++c) lo[c] = ub[c];
    }
  }
  // v = L.  lo = #(< v), hi = #(<= v) restricted by the windows; recompute exactly to be safe.
  const uint64_t v = L;
  uint64_t lt = 0;
  uint64_t eq[C];
#pragma unroll
  for (int c = 0; c < C; ++c) {
    // lower bound and upper bound of v inside [lo, hi) (keys outside are < v or > v)
    uint64_t a = lo[c], z = hi[c];
    uint64_t l2 = a, h2 = z;
    while (l2 < h2) {  // first index with key >= v
      uint64_t mid = l2 + ((h2 - l2) >> 1);
      if (K[base[c] + mid] < v) l2 = mid + 1;
      else h2 = mid;
    }
    uint64_t u = upper_bound(K + base[c], l2, z, v);
    lo[c] = l2;
    eq[c] = u - l2;
    lt += l2;
  }
  lt = warp_sum(lt);
  // take the o - lt keys equal to v in run order (j = c*32 + lane)
  uint64_t rem = o - lt;
#pragma unroll
  for (int c = 0; c < C; ++c) {
    uint64_t e = eq[c];
    uint64_t x = e;  // inclusive scan over lanes
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      uint64_t y = __shfl_up_sync(0xffffffffu, x, d);
      if (lane >= d) x += y;
    }
    uint64_t excl = x - e;
    uint64_t tot = __shfl_sync(0xffffffffu, x, 31);
    uint64_t take = rem > excl ? (rem - excl < e ? rem - excl : e) : 0;
    if (c * 32 + lane < k) out[c * 32 + lane] = lo[c] + take;
    rem = rem > tot ? rem - tot : 0;
  }
}

// K5.  One CTA per output tile.  Dynamic smem: 2 x kMergeTile keys + bounds.
constexpr int kMergeThreads = 256;
constexpr int kMergeIPT = kMergeTile / kMergeThreads;

__global__ void __launch_bounds__(kMergeThreads) k_merge_tile(
    const uint64_t* __restrict__ keys, const uint64_t* __restrict__ off, int k, uint64_t total,
    const uint64_t* __restrict__ ranks, uint64_t rank_tile0, uint64_t tile_begin,
    uint64_t* __restrict__ out, uint64_t out_origin, int out_f64) {
  extern __shared__ __align__(16) unsigned char smem[];
  uint64_t* bufA = (uint64_t*)smem;
  uint64_t* bufB = bufA + kMergeTile;
  uint32_t* bnd = (uint32_t*)(bufB + kMergeTile);   // k+1 sequence boundaries
  uint32_t* bnd2 = bnd + (kMaxMergeRuns + 1);        // scratch for compaction
  uint64_t* s_src = (uint64_t*)(bnd2 + (kMaxMergeRuns + 1));  // absolute start of slice j
  __shared__ uint32_t s_carry;

  const uint64_t t = tile_begin + blockIdx.x;
  const uint64_t o0 = t * (uint64_t)kMergeTile;
  const uint64_t o1 = (o0 + kMergeTile < total) ? o0 + kMergeTile : total;
  const int L = (int)(o1 - o0);
  const uint64_t* r0 = ranks + (t - rank_tile0) * (uint64_t)k;
  const uint64_t* r1 = r0 + k;
  const int tid = threadIdx.x;

  // slice lengths -> exclusive prefix (sequential chunks of 256 runs)
  if (tid == 0) s_carry = 0;
  __syncthreads();
  for (int c0 = 0; c0 < k; c0 += kMergeThreads) {
    int j = c0 + tid;
    uint32_t len = 0;
    if (j < k) {
      len = (uint32_t)(r1[j] - r0[j]);
      s_src[j] = off[j] + r0[j];
    }
    // block inclusive scan of len
    uint32_t x = len;
    const int lane = tid & 31, w = tid >> 5;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      uint32_t y = __shfl_up_sync(0xffffffffu, x, d);
      if (lane >= d) x += y;
    }
    __shared__ uint32_t s_w[kMergeThreads / 32];
    if (lane == 31) s_w[w] = x;
    __syncthreads();
    uint32_t pre = 0, tot = 0;
    for (int q = 0; q < kMergeThreads / 32; ++q) {
      if (q < w) pre += s_w[q];
      tot += s_w[q];
    }
    if (j < k) bnd[j] = s_carry + pre + x - len;
    __syncthreads();
    if (tid == 0) s_carry += tot;
    __syncthreads();
  }
  if (tid == 0) bnd[k] = (uint32_t)L;
  __syncthreads();

  // gather slices into bufA (element p belongs to run j with bnd[j] <= p < bnd[j+1])
  for (int p = tid; p < L; p += kMergeThreads) {
    int a = 0, z = k;  // largest j with bnd[j] <= p
    while (z - a > 1) {
      int m = (a + z) >> 1;
      if (bnd[m] <= (uint32_t)p) a = m;
      else z = m;
    }
    // skip empty runs sharing the same boundary: a is the largest j with bnd[j] <= p, and since
    // p < bnd[k] = L, run a is non-empty at p
    bufA[p] = keys[s_src[a] + (p - bnd[a])];
  }
  __syncthreads();

  // pairwise merge-path tree in shared memory
  int nseq = k;
  uint64_t* srcb = bufA;
  uint64_t* dstb = bufB;
  while (nseq > 1) {
    const int npair = (nseq + 1) >> 1;
    const int p0 = tid * kMergeIPT;
    if (p0 < L) {
      int p = p0;
      int pend = p0 + kMergeIPT < L ? p0 + kMergeIPT : L;
      while (p < pend) {
        // pair m: largest m with bnd[2m] <= p
        int a = 0, z = npair;
        while (z - a > 1) {
          int m = (a + z) >> 1;
          if (bnd[2 * m] <= (uint32_t)p) a = m;
          else z = m;
        }
        const int m = a;
        const int s0 = bnd[2 * m];
        const int s1 = (2 * m + 1 <= nseq) ? bnd[2 * m + 1 < nseq ? 2 * m + 1 : nseq] : L;
        const int s2 = bnd[2 * m + 2 <= nseq ? 2 * m + 2 : nseq];
        const int lenA = s1 - s0, lenB = s2 - s1;
        const uint64_t* A = srcb + s0;
        const uint64_t* B = srcb + s1;
        const int d = p - s0;
        int lo = d > lenB ? d - lenB : 0, hi = d < lenA ? d : lenA;
        while (lo < hi) {
          int mid = (lo + hi) >> 1;
          if (A[mid] <= B[d - 1 - mid]) lo = mid + 1;
          else hi = mid;
        }
        int i = lo, jb = d - lo;
        const int stop = pend < s2 ? pend : s2;
        for (; p < stop; ++p) {
          uint64_t x;
          if (i < lenA && (jb >= lenB || A[i] <= B[jb])) x = A[i++];
          else x = B[jb++];
          dstb[p] = x;
        }
      }
    }
    __syncthreads();
    // new boundaries: bnd'[m] = bnd[2m], bnd'[npair] = L
    for (int m = tid; m <= npair; m += kMergeThreads) bnd2[m] = (m < npair) ? bnd[2 * m] : (uint32_t)L;
    __syncthreads();
    for (int m = tid; m <= npair; m += kMergeThreads) bnd[m] = bnd2[m];
    __syncthreads();
    nseq = npair;
    uint64_t* tsw = srcb;
    srcb = dstb;
    dstb = tsw;
  }

  uint64_t* o = out + (o0 - out_origin);
  if (out_f64) {
    for (int p = tid; p < L; p += kMergeThreads) o[p] = from_key(srcb[p]);
  } else {
    for (int p = tid; p < L; p += kMergeThreads) o[p] = srcb[p];
  }
}

// Splitter partition of one sorted run (multi-GPU exchange): out[i] = number of
// keys <= values[i].  One thread per value; values sorted or not.
__global__ void k_upper_bounds(const uint64_t* __restrict__ keys, uint64_t n,
                               const uint64_t* __restrict__ values, uint64_t m,
                               uint64_t* __restrict__ out) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < m) out[i] = upper_bound(keys, 0, n, values[i]);
}

constexpr size_t merge_smem_bytes() {
  return 2 * kMergeTile * sizeof(uint64_t) + 2 * (kMaxMergeRuns + 1) * sizeof(uint32_t) +
         kMaxMergeRuns * sizeof(uint64_t);
}

}  // namespace

cudaError_t merge_corank(const uint64_t* keys, const uint64_t* d_off, int k, uint64_t total,
                         uint64_t step, uint64_t bound_begin, uint64_t n_bounds, uint64_t* ranks,
                         cudaStream_t st) {
  if (k < 1 || k > kMaxMergeRuns) return cudaErrorInvalidValue;
  if (n_bounds == 0) return cudaSuccess;
  const unsigned grid = (unsigned)((n_bounds * 32 + 127) / 128);
  int C = (k + 31) / 32;
  if (C <= 1) k_corank<1><<<grid, 128, 0, st>>>(keys, d_off, k, total, step, bound_begin, n_bounds, ranks);
  else if (C <= 2) k_corank<2><<<grid, 128, 0, st>>>(keys, d_off, k, total, step, bound_begin, n_bounds, ranks);
  else if (C <= 4) k_corank<4><<<grid, 128, 0, st>>>(keys, d_off, k, total, step, bound_begin, n_bounds, ranks);
  else if (C <= 8) k_corank<8><<<grid, 128, 0, st>>>(keys, d_off, k, total, step, bound_begin, n_bounds, ranks);
  else k_corank<kMaxC><<<grid, 128, 0, st>>>(keys, d_off, k, total, step, bound_begin, n_bounds, ranks);
  return cudaGetLastError();
}

cudaError_t upper_bounds(const uint64_t* keys, uint64_t n, const uint64_t* values, uint64_t m,
                         uint64_t* out, cudaStream_t st) {
  if (m == 0) return cudaSuccess;
  k_upper_bounds<<<(unsigned)((m + 255) / 256), 256, 0, st>>>(keys, n, values, m, out);
  return cudaGetLastError();
}

cudaError_t merge_tiles(const uint64_t* keys, const uint64_t* d_off, int k, uint64_t total,
                        const uint64_t* ranks, uint64_t rank_tile0, uint64_t tile_begin,
                        uint64_t tile_count, uint64_t* out, uint64_t out_origin, bool out_f64,
                        cudaStream_t st) {
  if (tile_count == 0) return cudaSuccess;
  static bool attr_set[64] = {false};
  int dev = 0;
  cudaGetDevice(&dev);
  const size_t smem = merge_smem_bytes();
  if (dev >= 0 && dev < 64 && !attr_set[dev]) {
    cudaError_t e = cudaFuncSetAttribute(k_merge_tile, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)smem);
    if (e != cudaSuccess) return e;
    attr_set[dev] = true;
  }
  k_merge_tile<<<(unsigned)tile_count, kMergeThreads, smem, st>>>(keys, d_off, k, total, ranks,
                                                                  rank_tile0, tile_begin, out,
                                                                  out_origin, out_f64 ? 1 : 0);
  return cudaGetLastError();
}

}  // namespace hsort
