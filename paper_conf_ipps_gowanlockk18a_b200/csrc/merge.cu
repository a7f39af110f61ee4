// merge.cu — multiway merge of sorted batches on the GPU (§III-A), with
// merge-path partitioning (ref [18]) generalised to k runs.
//
// The paper merges on the CPU with GNU parallel multiway_merge.  On a B200 whose sorted runs are
// still resident in HBM the merge is an HBM-bound pass (16 B/key), so it runs here:
//
//   K4 k_corank     exact co-ranks (i_0..i_{k-1}) of each output-tile boundary o: the first o
//                   keys of the merge in which equal keys are taken in run order.  One warp per
//                   boundary (k <= 128: a G-lane segment, 32 / G boundaries per warp), lanes
//                   own runs; bisection on the key value with per-run index windows, the value
//                   bracket tightened to keys still inside the windows.
//   K5 k_merge_tile each CTA owns one output tile [o_t, o_t+1): loads its k slices into shared
//                   memory, merges them by a pairwise merge-path tree in shared memory, and writes
//                   the tile with coalesced stores (inverse key transform fused).
#include <cuda_runtime.h>

#include <cstdint>

#include "internal.h"

#ifndef HSORT_MERGE_GCACHE
#define HSORT_MERGE_GCACHE 1  // K5 gather: run source / end cached in registers
#endif
#ifndef HSORT_MERGE_ABS
#define HSORT_MERGE_ABS 1  // unrolled merge steps on absolute head indices
#endif
#ifndef HSORT_MERGE_CLAMP
// 0: a merge step may load the head one past an exhausted pair (pp(s2) <= BUF stays inside the
// dynamic shared allocation; the bounds test never takes it), saving the clamp per output
#define HSORT_MERGE_CLAMP 0  // (A/B: k = 12 11.38 -> 11.25 ms, k = 128 22.15 -> 21.7 ms)
#endif
namespace hsort {
namespace {

constexpr int kMaxC = kMaxMergeRuns / 32;

__device__ __forceinline__ uint64_t from_key(uint64_t k) {
  return k ^ ((uint64_t)((int64_t)(~k) >> 63) | 0x8000000000000000ull);
}

// reductions over one G-lane segment (sm = the segment's lanes)
template <int G>
__device__ __forceinline__ uint64_t seg_sum(unsigned sm, uint64_t v) {
#pragma unroll
  for (int o = G / 2; o; o >>= 1) v += __shfl_xor_sync(sm, v, o, G);
  return v;
}
template <int G>
__device__ __forceinline__ uint64_t seg_min(unsigned sm, uint64_t v) {
#pragma unroll
  for (int o = G / 2; o; o >>= 1) {
    const uint64_t w = __shfl_xor_sync(sm, v, o, G);
    v = w < v ? w : v;
  }
  return v;
}
template <int G>
__device__ __forceinline__ uint64_t seg_max(unsigned sm, uint64_t v) {
#pragma unroll
  for (int o = G / 2; o; o >>= 1) {
    const uint64_t w = __shfl_xor_sync(sm, v, o, G);
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
// first index i in [0, r] with a[i] >= v, given a[r] >= v (or r = end): gallop back from r
__device__ __forceinline__ uint64_t lower_bound_back(const uint64_t* a, uint64_t r, uint64_t v) {
  uint64_t hi = r, step = 1;
  while (hi > 0 && a[hi - 1] >= v) {  // a[hi - 1] >= v: the bound lies further back
    const uint64_t lo = hi > step ? hi - step : 0;
    if (a[lo] < v) {  // bound in (lo, hi - 1]
      uint64_t l = lo + 1, h = hi - 1;
      while (l < h) {
        const uint64_t m = l + ((h - l) >> 1);
        if (a[m] < v) l = m + 1;
        else h = m;
      }
      return l;
    }
    hi = lo;
    step <<= 1;
  }
  return hi;
}
// first index i in [r, len] with a[i] > v, given a[r - 1] <= v (or r = 0): gallop forward
__device__ __forceinline__ uint64_t upper_bound_fwd(const uint64_t* a, uint64_t r, uint64_t len,
                                                    uint64_t v) {
  uint64_t lo = r, step = 1;
  while (lo < len && a[lo] <= v) {
    const uint64_t hi = lo + step < len ? lo + step : len;
    if (hi == len || a[hi] > v) {  // bound in (lo, hi]
      uint64_t l = lo + 1, h = hi;
      while (l < h) {
        const uint64_t m = l + ((h - l) >> 1);
        if (a[m] <= v) l = m + 1;
        else h = m;
      }
      return l;
    }
    lo = hi;
    step <<= 1;
  }
  return lo;
}

// coarse != nullptr: row (c - coarse_b0) of `coarse` holds the co-ranks of output position
// min(c * coarse_step, total) (coarse_step a multiple of step); a fine boundary starts from the
// windows between its two coarse neighbours: with v_lo = the key at the lower coarse position and
// v_hi = the key just before the upper one, #(< v_lo) <= o_lo <= o < o_hi <= #(<= v_hi), so the
// bisection starts at [v_lo, v_hi] with lo/hi found by galloping from the coarse co-ranks.
template <int C, int G>
__global__ void __launch_bounds__(128) k_corank(const uint64_t* __restrict__ keys,
                                                const uint64_t* const* __restrict__ rp,
                                                const uint64_t* __restrict__ off, int k,
                                                uint64_t total, uint64_t step, uint64_t b0,
                                                uint64_t nb, uint64_t* __restrict__ ranks,
                                                const uint64_t* __restrict__ coarse,
                                                uint64_t coarse_step, uint64_t coarse_b0) {
  // G lanes per boundary, C runs per lane (run j = c G + lane); 32 / G boundaries share a warp on
  // their own lane segments, so more dependent-load chains are in flight per SM.  corank_launch
  // picks (C, G): k <= 16 -> (1, next power of two >= k); 16 < k <= 32 -> (2, 16);
  // 32 < k <= 64 -> (4, 16); 64 < k <= 128 -> (8, 16); k > 128 -> G = 32, C = 8 / 16 / 32
  // (k <= 256 / 512 / 1024).
  const int seg = (threadIdx.x & 31) / G;
  const int lane = threadIdx.x & (G - 1);
  const unsigned sm = G == 32 ? 0xffffffffu : ((1u << G) - 1u) << (seg * G);
  const uint64_t b =
      (((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5) * (uint64_t)(32 / G) + seg;
  if (b >= nb) return;
  const uint64_t o = (b0 + b) * step < total ? (b0 + b) * step : total;
  // run j = R[c] (j = c G + lane): back to back in `keys`, or anywhere (rp: a table of run
  // pointers, possibly into peer GPUs' HBM, read over NVLink)
  const uint64_t* R[C];
  uint64_t lo[C], hi[C];
#pragma unroll
  for (int c = 0; c < C; ++c) {
    int j = c * G + lane;
    if (j < k) {
      R[c] = rp ? rp[j] : keys + off[j];
      lo[c] = 0;
      hi[c] = off[j + 1] - off[j];
    } else {
      R[c] = keys;
      lo[c] = hi[c] = 0;
    }
  }
  uint64_t* out = ranks + b * (uint64_t)k;
  if (o == total) {
#pragma unroll
    for (int c = 0; c < C; ++c)
      if (c * G + lane < k) out[c * G + lane] = hi[c];
    return;
  }
  uint64_t L0 = 0, H0 = ~0ull;
  if (coarse) {
    const uint64_t ci = o / coarse_step;
    const uint64_t* r0 = coarse + (ci - coarse_b0) * (uint64_t)k;
    if (o == ci * coarse_step) {  // a coarse boundary itself
#pragma unroll
      for (int c = 0; c < C; ++c)
        if (c * G + lane < k) out[c * G + lane] = r0[c * G + lane];
      return;
    }
    const uint64_t* r1 = r0 + k;
    uint64_t rl[C], rh[C], mn = ~0ull, mx = 0;
#pragma unroll
    for (int c = 0; c < C; ++c) {
      const int j = c * G + lane;
      rl[c] = j < k ? r0[j] : 0;
      rh[c] = j < k ? r1[j] : 0;
      if (rl[c] < hi[c]) mn = R[c][rl[c]] < mn ? R[c][rl[c]] : mn;
      if (rh[c] > 0) mx = R[c][rh[c] - 1] > mx ? R[c][rh[c] - 1] : mx;
    }
    L0 = seg_min<G>(sm, mn);  // key at merged position o_lo
    H0 = seg_max<G>(sm, mx);  // key at merged position o_hi - 1
#pragma unroll
    for (int c = 0; c < C; ++c) {
      const uint64_t len = hi[c];
      lo[c] = lower_bound_back(R[c], rl[c], L0);
      hi[c] = upper_bound_fwd(R[c], rh[c], len, H0);
    }
  }
  // Find v = the key at merged position o: smallest v with count(<= v) > o.
  // Invariant: lo[c] = #(< L) in run, hi[c] = #(<= H) in run, count(<= H) > o, count(< L) <= o.
  // (An interpolated two-pivot variant was measured: 1.9x slower at k = 12 -- the float64 key
  // space is not uniform across binades, so the interpolation misses -- and removed.)
  uint64_t L = L0, H = H0;
  while (true) {
    // tighten [L, H] to the keys still inside the windows
    uint64_t mn = ~0ull, mx = 0;
#pragma unroll
    for (int c = 0; c < C; ++c) {
      if (hi[c] > lo[c]) {
        uint64_t a = R[c][lo[c]], z = R[c][hi[c] - 1];
        mn = a < mn ? a : mn;
        mx = z > mx ? z : mx;
      }
    }
    mn = seg_min<G>(sm, mn);
    mx = seg_max<G>(sm, mx);
    if (mn > L) L = mn;
    if (mx < H) H = mx;
    if (L >= H) break;
    const uint64_t mid = L + ((H - L) >> 1);
    uint64_t ub[C];
    uint64_t s = 0;
#pragma unroll
    for (int c = 0; c < C; ++c) {
      ub[c] = upper_bound(R[c], lo[c], hi[c], mid);
      s += ub[c];
    }
    // elements <= mid overall: the window searches count from index 0 (lo/hi are absolute)
    s = seg_sum<G>(sm, s);
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
      if (R[c][mid] < v) l2 = mid + 1;
      else h2 = mid;
    }
    uint64_t u = upper_bound(R[c], l2, z, v);
    lo[c] = l2;
    eq[c] = u - l2;
    lt += l2;
  }
  lt = seg_sum<G>(sm, lt);
  // take the o - lt keys equal to v in run order (j = c*32 + lane)
  uint64_t rem = o - lt;
#pragma unroll
  for (int c = 0; c < C; ++c) {
    uint64_t e = eq[c];
    uint64_t x = e;  // inclusive scan over lanes
#pragma unroll
    for (int d = 1; d < G; d <<= 1) {
      uint64_t y = __shfl_up_sync(sm, x, d, G);
      if (lane >= d) x += y;
    }
    uint64_t excl = x - e;
    uint64_t tot = __shfl_sync(sm, x, G - 1, G);
    uint64_t take = rem > excl ? (rem - excl < e ? rem - excl : e) : 0;
    if (c * G + lane < k) out[c * G + lane] = lo[c] + take;
    rem = rem > tot ? rem - tot : 0;
  }
}

// K5.  One CTA per output tile of kMergeTile keys, T threads x IPT = kMergeTile / T keys.
//   1. slice table: len_j = r1[j] - r0[j], bnd = exclusive prefix of len (tile-local starts);
//   2. gather: the k slices are copied into buf0 back to back.  Warp w loads elements
//      [32 IPT w, 32 IPT (w + 1)) lane-interleaved (coalesced within a slice); the run of an
//      element, max{j : bnd[j] <= p}, only grows along a lane's elements, so it is found once and
//      then advanced; all IPT loads are issued before any store (IPT HBM reads in flight);
//   3. ceil(log2 k) pairwise merge-path rounds between buf0 and buf1: in round r the sequences are
//      the groups of 2^r consecutive runs, so sequence m starts at bnd[min(m 2^r, k)] and no
//      boundary table is rewritten; the pair holding a thread's first output in round r is
//      j0 >> (r + 1), j0 the run holding it.  A thread owns outputs [IPT tid, IPT tid + IPT),
//      finds its split (A wins ties: stable, runs in order) by a merge-path search, and merges with
//      one shared-memory load per output;
//   4. the merged tile is stored with coalesced stores (inverse key transform fused).
// Shared-memory index of tile element p: one 8-byte pad after every IPT keys.  A thread's outputs
// start IPT keys after its neighbour's; without the pad (IPT = 8: 64 B stride) 16 lanes of a warp
// share one 8-byte bank pair on every merge-round load and store; with it the stride is IPT + 1
// keys (odd) and a half-warp hits 16 distinct bank pairs.
// Dynamic smem: 2 x (kMergeTile + kMergeTile / IPT) keys + k slice sources + (k + 1) bounds.
__device__ __forceinline__ uint64_t ld_stream_u64(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.global.cs.u64 %0, [%1];" : "=l"(v) : "l"(p));
  return v;
}

template <int T>
struct MergeCfg {
  static constexpr int IPT = kMergeTile / T;
  static_assert(T * IPT == kMergeTile, "merge tile");
  static constexpr int BUF = kMergeTile + kMergeTile / IPT;
  // p >= 0: unsigned division is one shift (a signed one costs three instructions)
  static __device__ __forceinline__ int pp(int p) { return p + (int)((unsigned)p / IPT); }
};

// largest j >= a with bnd[j] <= p (j < cnt), starting from a valid j = a: two linear steps (the
// usual distance when slices are longer than a thread's stride), then bisection of the rest
__device__ __forceinline__ int advance_run(const uint32_t* bnd, int a, int cnt, uint32_t p) {
#pragma unroll
  for (int s = 0; s < 2; ++s) {
    if (a + 1 >= cnt || bnd[a + 1] > p) return a;
    ++a;
  }
  int z = cnt;
  while (z - a > 1) {
    const int m = (a + z) >> 1;
    if (bnd[m] <= p) a = m;
    else z = m;
  }
  return a;
}

// KV (S§8(f) #3, the out-of-core key/value sort): every key carries a 64-bit value; values sit in
// their own shared buffers and move with their keys (the merge compares keys only, ties in run
// order, so the merge of stably sorted runs is the stable sort of the pairs).
template <int T, bool KV = false>
__global__ void __launch_bounds__(T) k_merge_tile(
    const uint64_t* __restrict__ keys, const uint64_t* const* __restrict__ rp,
    const uint64_t* __restrict__ off, int k, uint64_t total,
    const uint64_t* __restrict__ ranks, uint64_t rank_tile0, uint64_t tile_begin,
    uint64_t* __restrict__ out, uint64_t out_origin, int out_f64,
    const uint64_t* __restrict__ vkeys = nullptr, const uint64_t* const* __restrict__ vrp = nullptr,
    uint64_t* __restrict__ vout = nullptr) {
  using Cfg = MergeCfg<T>;
  constexpr int IPT = Cfg::IPT;
  extern __shared__ __align__(16) unsigned char smem[];
  uint64_t* buf0 = (uint64_t*)smem;
  uint64_t* buf1 = buf0 + Cfg::BUF;
  uint64_t* vbuf0 = buf1 + Cfg::BUF;                   // KV only
  uint64_t* vbuf1 = vbuf0 + Cfg::BUF;
  // [k] address of slice j's first key minus bnd[j] keys (slices may sit in peer GPUs' HBM)
  const uint64_t** s_src = (const uint64_t**)(buf1 + Cfg::BUF * (KV ? 3 : 1));
  const uint64_t** s_vsrc = s_src + k;                 // KV only: the values' slices
  uint32_t* bnd = (uint32_t*)(s_src + k * (KV ? 2 : 1));  // [k + 1] tile-local slice starts
  __shared__ uint32_t s_w[T / 32];

  const uint64_t t = tile_begin + blockIdx.x;
  const uint64_t o0 = t * (uint64_t)kMergeTile;
  const uint64_t o1 = (o0 + kMergeTile < total) ? o0 + kMergeTile : total;
  const int L = (int)(o1 - o0);
  const uint64_t* r0 = ranks + (t - rank_tile0) * (uint64_t)k;
  const uint64_t* r1 = r0 + k;
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;

  // 1. slice table (chunks of T runs, block scan); s_src[j] - bnd[j] is stored, so element p of
  //    slice j is s_src[j][p]
  uint32_t carry = 0;
  for (int c0 = 0; c0 < k; c0 += T) {
    const int j = c0 + tid;
    uint32_t len = 0;
    const uint64_t* srcj = nullptr;
    const uint64_t* vsrcj = nullptr;
    if (j < k) {
      const uint64_t a = r0[j];
      len = (uint32_t)(r1[j] - a);
      srcj = (rp ? rp[j] : keys + off[j]) + a;
      if (KV) vsrcj = (vrp ? vrp[j] : vkeys + off[j]) + a;
    }
    uint32_t x = len;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, x, d);
      if (lane >= d) x += y;
    }
    if (k <= 32) {  // one warp holds every run: no block scan
      if (j < k) {
        bnd[j] = x - len;
        s_src[j] = srcj - (x - len);
        if (KV) s_vsrc[j] = vsrcj - (x - len);
      }
      break;
    }
    if (lane == 31) s_w[w] = x;
    __syncthreads();
    uint32_t pre = 0, tot = 0;
#pragma unroll
    for (int q = 0; q < T / 32; ++q) {
      const uint32_t sq = s_w[q];
      pre += q < w ? sq : 0;
      tot += sq;
    }
    if (j < k) {
      const uint32_t bj = carry + pre + x - len;
      bnd[j] = bj;
      s_src[j] = srcj - bj;
      if (KV) s_vsrc[j] = vsrcj - bj;
    }
    carry += tot;
    __syncthreads();
  }
  if (tid == 0) bnd[k] = (uint32_t)L;
  __syncthreads();

  uint64_t* o = out + (o0 - out_origin);

  // 2. gather (k == 1: straight copy).  Warp w copies tile elements [w C, w C + C), C = 32 IPT,
  //    lane-interleaved (coalesced); a lane finds the run of its first element by bisection, then
  //    advances it (usually zero steps: slices are longer than 32 keys).
  constexpr int C = 32 * IPT;
  uint64_t v[IPT];
  uint64_t vv[KV ? IPT : 1];
  {
    const int e0 = w * C + lane;
    int a = (k > 1 && e0 < L) ? advance_run(bnd, 0, k, (uint32_t)e0) : 0;
#if HSORT_MERGE_GCACHE
    // the run's source and its end held in registers; they change only when e crosses a boundary
    const uint64_t* sp = s_src[a];
    const uint64_t* svp = KV ? s_vsrc[a] : nullptr;
    uint32_t nb = a + 1 < k ? bnd[a + 1] : 0xffffffffu;
#pragma unroll
    for (int q = 0; q < IPT; ++q) {
      const int e = e0 + 32 * q;
      if (e < L) {
        while ((uint32_t)e >= nb) {
          ++a;
          sp = s_src[a];
          if (KV) svp = s_vsrc[a];
          nb = a + 1 < k ? bnd[a + 1] : 0xffffffffu;
        }
        v[q] = ld_stream_u64(sp + e);
        if (KV) vv[q] = ld_stream_u64(svp + e);
      }
    }
#else
#pragma unroll
    for (int q = 0; q < IPT; ++q) {
      const int e = e0 + 32 * q;
      if (e < L) {
        while (a + 1 < k && bnd[a + 1] <= (uint32_t)e) ++a;
        v[q] = ld_stream_u64(s_src[a] + e);
        if (KV) vv[q] = ld_stream_u64(s_vsrc[a] + e);
      }
    }
#endif
  }
  uint64_t* vo = KV ? vout + (o0 - out_origin) : nullptr;
  if (k == 1) {
#pragma unroll
    for (int q = 0; q < IPT; ++q) {
      const int e = w * C + lane + 32 * q;
      if (e < L) {
        o[e] = out_f64 ? from_key(v[q]) : v[q];
        if (KV) vo[e] = vv[q];
      }
    }
    return;
  }
#pragma unroll
  for (int q = 0; q < IPT; ++q) {
    const int e = w * C + lane + 32 * q;
    if (e < L) {
      buf0[Cfg::pp(e)] = v[q];
      if (KV) vbuf0[Cfg::pp(e)] = vv[q];
    }
  }
  const int p0 = tid * IPT;
  const int pend = p0 + IPT < L ? p0 + IPT : L;
  const int j0 = p0 < L ? advance_run(bnd, 0, k, (uint32_t)p0) : 0;  // run holding output p0
  __syncthreads();

  // 3. pairwise merge-path rounds
  uint64_t* src = buf0;
  uint64_t* dst = buf1;
  uint64_t* vsrc = vbuf0;
  uint64_t* vdst = vbuf1;
  for (int sh = 0; (1 << sh) < k; ++sh) {
    int p = p0;
    int m = j0 >> (sh + 1);
    while (p < pend) {
      // pair m holds p: bnd[start(m)] <= p < bnd[start(m + 1)]; advance past pairs ending <= p
      const int q0 = (2 * m) << sh, q1 = (2 * m + 1) << sh, q2 = (2 * m + 2) << sh;
      const int s0 = bnd[q0 < k ? q0 : k];
      const int s1 = bnd[q1 < k ? q1 : k];
      const int s2 = bnd[q2 < k ? q2 : k];
      if (s2 <= p) {
        ++m;
        continue;
      }
      const int lenA = s1 - s0, lenB = s2 - s1;
      const int d = p - s0;
      int lo = d > lenB ? d - lenB : 0, hi = d < lenA ? d : lenA;
      while (lo < hi) {
        const int mid = (lo + hi) >> 1;
        if (src[Cfg::pp(s0 + mid)] <= src[Cfg::pp(s1 + d - 1 - mid)]) lo = mid + 1;
        else hi = mid;
      }
      int i = lo, jb = d - lo;
      const int stop = pend < s2 ? pend : s2;
      // heads (indices clamped into the pair; an exhausted side is never taken)
      uint64_t a = src[Cfg::pp(s0 + i < s2 - 1 ? s0 + i : s2 - 1)];
      uint64_t b = src[Cfg::pp(s1 + jb < s2 - 1 ? s1 + jb : s2 - 1)];
      if (stop - p == IPT) {
        // whole output range inside one pair (the common case): fully unrolled, output slots at
        // constant offsets from pp(p0) (p0 = IPT tid: no pad inside a thread's range)
        uint64_t* d = dst + Cfg::pp(p);
        uint64_t* dv = vdst + Cfg::pp(p);
#if HSORT_MERGE_ABS
        int ia = s0 + i, ib = s1 + jb;  // absolute heads; A = [s0, s1), B = [s1, s2)
#pragma unroll
        for (int q = 0; q < IPT; ++q) {
          const bool ta = ib >= s2 || (ia < s1 && a <= b);
          d[q] = ta ? a : b;
          if (KV) dv[q] = vsrc[Cfg::pp(ta ? ia : ib)];
          ia += ta;
          ib += !ta;
          const uint64_t y = src[Cfg::pp(ta ? ia : ib)];  // may be one past an exhausted pair
          a = ta ? y : a;
          b = ta ? b : y;
        }
#else
#pragma unroll
        for (int q = 0; q < IPT; ++q) {
          const bool ta = jb >= lenB || (i < lenA && a <= b);
          d[q] = ta ? a : b;
          if (KV) dv[q] = vsrc[Cfg::pp(ta ? s0 + i : s1 + jb)];
          i += ta;
          jb += !ta;
          int nx = ta ? s0 + i : s1 + jb;
#if HSORT_MERGE_CLAMP
          nx = nx < s2 - 1 ? nx : s2 - 1;
#endif
          const uint64_t y = src[Cfg::pp(nx)];
          a = ta ? y : a;
          b = ta ? b : y;
        }
#endif
        p = stop;
      }
      for (; p < stop; ++p) {
        const bool ta = jb >= lenB || (i < lenA && a <= b);
        const uint64_t x = ta ? a : b;
        dst[Cfg::pp(p)] = x;
        if (KV) vdst[Cfg::pp(p)] = vsrc[Cfg::pp(ta ? s0 + i : s1 + jb)];
        i += ta;
        jb += !ta;
        int nx = ta ? s0 + i : s1 + jb;
#if HSORT_MERGE_CLAMP
        nx = nx < s2 - 1 ? nx : s2 - 1;
#endif
        const uint64_t y = src[Cfg::pp(nx)];
        a = ta ? y : a;
        b = ta ? b : y;
      }
      ++m;
    }
    __syncthreads();
    uint64_t* tsw = src;
    src = dst;
    dst = tsw;
    tsw = vsrc;
    vsrc = vdst;
    vdst = tsw;
  }

  // 4. coalesced store of the tile (src holds the merged, transformed keys)
  if (out_f64) {
#pragma unroll
    for (int q = 0; q < IPT; ++q) {
      const int p = q * T + tid;
      if (p < L) __stcs(o + p, from_key(src[Cfg::pp(p)]));
    }
  } else {
#pragma unroll
    for (int q = 0; q < IPT; ++q) {
      const int p = q * T + tid;
      if (p < L) __stcs(o + p, src[Cfg::pp(p)]);
    }
  }
  if (KV) {
#pragma unroll
    for (int q = 0; q < IPT; ++q) {
      const int p = q * T + tid;
      if (p < L) __stcs(vo + p, vsrc[Cfg::pp(p)]);
    }
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

#ifndef HSORT_MERGE_THREADS
#define HSORT_MERGE_THREADS 256  // 256 x 16 keys: 12.9 ms vs 14.8 ms (512 x 8) per 2^30 keys, k = 12
#endif
constexpr int kMergeThreads = HSORT_MERGE_THREADS;

size_t merge_smem_bytes(int k, bool kv = false) {
  return (kv ? 4 : 2) * MergeCfg<kMergeThreads>::BUF * sizeof(uint64_t) +
         (size_t)k * sizeof(void*) * (kv ? 2 : 1) +
         ((size_t)k + 1) * sizeof(uint32_t);
}

}  // namespace

#ifndef HSORT_CORANK_SEG
#define HSORT_CORANK_SEG 1  // k <= 16: 32 / G co-rank searches per warp (K4)
#endif
constexpr bool kCorankSeg = HSORT_CORANK_SEG != 0;
#ifndef HSORT_CORANK_SEG2
#define HSORT_CORANK_SEG2 1  // 16 < k <= 32: two 16-lane segments per warp, 2 runs per lane
#endif
constexpr bool kCorankSeg2 = HSORT_CORANK_SEG2 != 0;
#ifndef HSORT_CORANK_ILP
#define HSORT_CORANK_ILP 1  // 32 < k <= 128: 16-lane segments, k / 16 runs per lane (2 runs per
                            // lane at k <= 16 was measured 18-30% slower)
#endif
constexpr bool kCorankIlp = HSORT_CORANK_ILP != 0;

namespace {
cudaError_t corank_launch(const uint64_t* keys, const uint64_t* const* rp, const uint64_t* d_off,
                          int k, uint64_t total, uint64_t step, uint64_t bound_begin,
                          uint64_t n_bounds, uint64_t* ranks, const uint64_t* coarse,
                          uint64_t cstep, uint64_t cb0, cudaStream_t st) {
  const int C = (k + 31) / 32;
#define HS_CORANK_G(CC, GG)                                                                        \
  k_corank<CC, GG><<<(unsigned)((n_bounds * GG + 127) / 128), 128, 0, st>>>(                      \
      keys, rp, d_off, k, total, step, bound_begin, n_bounds, ranks, coarse, cstep, cb0)
#define HS_CORANK(CC) HS_CORANK_G(CC, 32)
  if (kCorankIlp && k > 32 && k <= 64) HS_CORANK_G(4, 16);
  else if (kCorankIlp && k > 64 && k <= 128) HS_CORANK_G(8, 16);
  else if (kCorankSeg && k <= 2) HS_CORANK_G(1, 2);
  else if (kCorankSeg && k <= 4) HS_CORANK_G(1, 4);
  else if (kCorankSeg && k <= 8) HS_CORANK_G(1, 8);
  else if (kCorankSeg && k <= 16) HS_CORANK_G(1, 16);
  else if (kCorankSeg2 && k <= 32) HS_CORANK_G(2, 16);
  else if (C <= 1) HS_CORANK(1);
  else if (C <= 2) HS_CORANK(2);
  else if (C <= 4) HS_CORANK(4);
  else if (C <= 8) HS_CORANK(8);
  else if (C <= 16) HS_CORANK(16);
  else HS_CORANK(kMaxC);
#undef HS_CORANK
#undef HS_CORANK_G
  return launched();
}
}  // namespace

// K4 in two levels: co-ranks every kCoarse fine steps first (full-range search), then every
// fine boundary from the windows between its coarse neighbours (K4).
#ifndef HSORT_CORANK_COARSE
#define HSORT_CORANK_COARSE 16  // A/B at 2^30 keys: 8 / 16 / 32 / 64 -> 2.55 / 2.39 / 2.30 / 2.34 ms (k = 12)
#endif
constexpr uint64_t kCoarse = HSORT_CORANK_COARSE;
#ifndef HSORT_CORANK_LEVELS
#define HSORT_CORANK_LEVELS 0  // co-rank levels (2: one coarse level); 0: 3 from k = 32 runs, else 2
                               // (A/B at 2^30 keys, profiles/r03bi: 3 levels cost 0.1-0.16 ms more
                               // at k <= 12, save 0.1 / 0.8 ms at k = 32 / 128)
#endif
static int corank_levels(int k) { return HSORT_CORANK_LEVELS ? HSORT_CORANK_LEVELS : (k >= 32 ? 3 : 2); }

namespace {
// coarse rows c0 .. c0 + nc - 1 bracketing every requested bound (0 rows: single level)
void coarse_rows(uint64_t total, uint64_t step, uint64_t bound_begin, uint64_t n_bounds, int k,
                 uint64_t* c0, uint64_t* nc) {
  *c0 = *nc = 0;
  if (n_bounds < 4 * kCoarse || k == 1) return;
  const uint64_t cstep = step * kCoarse;
  const uint64_t o_first = bound_begin * step < total ? bound_begin * step : total;
  const uint64_t o_last0 = (bound_begin + n_bounds - 1) * step;
  const uint64_t o_last = o_last0 < total ? o_last0 : total;
  *c0 = o_first / cstep;
  *nc = (o_last + cstep - 1) / cstep - *c0 + 1;
}
}  // namespace

// levels: 2 = a coarse level (full-range search) + the requested bounds; more: the coarse level
// is itself computed from a coarser one, recursively (each level kCoarse times sparser)
static uint64_t corank_scratch_rec(int k, uint64_t total, uint64_t step, uint64_t bound_begin,
                                   uint64_t n_bounds, int levels) {
  uint64_t c0, nc;
  coarse_rows(total, step, bound_begin, n_bounds, k, &c0, &nc);
  if (nc == 0 || levels < 2) return 0;
  return nc * (uint64_t)k + corank_scratch_rec(k, total, step * kCoarse, c0, nc, levels - 1);
}
uint64_t merge_corank_scratch_elems(int k, uint64_t total, uint64_t step, uint64_t bound_begin,
                                    uint64_t n_bounds) {
  return corank_scratch_rec(k, total, step, bound_begin, n_bounds, corank_levels(k));
}

cudaError_t merge_corank_rec(const uint64_t* keys, const uint64_t* const* rp, const uint64_t* d_off,
                             int k, uint64_t total, uint64_t step, uint64_t bound_begin,
                             uint64_t n_bounds, uint64_t* ranks, uint64_t* scratch,
                             uint64_t scratch_elems, int levels, cudaStream_t st);
cudaError_t merge_corank(const uint64_t* keys, const uint64_t* const* rp, const uint64_t* d_off,
                         int k, uint64_t total, uint64_t step, uint64_t bound_begin,
                         uint64_t n_bounds, uint64_t* ranks, uint64_t* scratch,
                         uint64_t scratch_elems, cudaStream_t st) {
  return merge_corank_rec(keys, rp, d_off, k, total, step, bound_begin, n_bounds, ranks, scratch,
                          scratch_elems, corank_levels(k), st);
}

cudaError_t merge_corank_rec(const uint64_t* keys, const uint64_t* const* rp, const uint64_t* d_off,
                             int k, uint64_t total, uint64_t step, uint64_t bound_begin,
                             uint64_t n_bounds, uint64_t* ranks, uint64_t* scratch,
                             uint64_t scratch_elems, int levels, cudaStream_t st) {
  if (k < 1 || k > kMaxMergeRuns) return cudaErrorInvalidValue;
  if (n_bounds == 0) return cudaSuccess;
  uint64_t c0, nc;
  coarse_rows(total, step, bound_begin, n_bounds, k, &c0, &nc);
  if (levels < 2 || nc == 0 || !scratch || scratch_elems < nc * (uint64_t)k)  // single level
    return corank_launch(keys, rp, d_off, k, total, step, bound_begin, n_bounds, ranks, nullptr, 1,
                         0, st);
  const uint64_t cstep = step * kCoarse;
  cudaError_t e = merge_corank_rec(keys, rp, d_off, k, total, cstep, c0, nc, scratch,
                                   scratch + nc * (uint64_t)k, scratch_elems - nc * (uint64_t)k,
                                   levels - 1, st);
  if (e != cudaSuccess) return e;
  return corank_launch(keys, rp, d_off, k, total, step, bound_begin, n_bounds, ranks, scratch,
                       cstep, c0, st);
}

cudaError_t upper_bounds(const uint64_t* keys, uint64_t n, const uint64_t* values, uint64_t m,
                         uint64_t* out, cudaStream_t st) {
  if (m == 0) return cudaSuccess;
  k_upper_bounds<<<(unsigned)((m + 255) / 256), 256, 0, st>>>(keys, n, values, m, out);
  return launched();
}

cudaError_t merge_tiles(const uint64_t* keys, const uint64_t* const* rp, const uint64_t* d_off,
                        int k, uint64_t total,
                        const uint64_t* ranks, uint64_t rank_tile0, uint64_t tile_begin,
                        uint64_t tile_count, uint64_t* out, uint64_t out_origin, bool out_f64,
                        cudaStream_t st, const uint64_t* vkeys, const uint64_t* const* vrp,
                        uint64_t* vout) {
  if (tile_count == 0) return cudaSuccess;
  static bool attr_set[64] = {false};
  static bool attr_kv[64] = {false};
  int dev = 0;
  cudaGetDevice(&dev);
  const bool kv = vout != nullptr;
  const size_t smem = merge_smem_bytes(k, kv);
  if (dev >= 0 && dev < 64 && !(kv ? attr_kv : attr_set)[dev]) {
    cudaError_t e = kv ? cudaFuncSetAttribute(k_merge_tile<kMergeThreads, true>,
                                              cudaFuncAttributeMaxDynamicSharedMemorySize,
                                              (int)merge_smem_bytes(kMaxMergeRuns, true))
                       : cudaFuncSetAttribute(k_merge_tile<kMergeThreads>,
                                              cudaFuncAttributeMaxDynamicSharedMemorySize,
                                              (int)merge_smem_bytes(kMaxMergeRuns));
    if (e != cudaSuccess) return e;
    (kv ? attr_kv : attr_set)[dev] = true;
  }
  if (kv)
    k_merge_tile<kMergeThreads, true><<<(unsigned)tile_count, kMergeThreads, smem, st>>>(
        keys, rp, d_off, k, total, ranks, rank_tile0, tile_begin, out, out_origin, out_f64 ? 1 : 0,
        vkeys, vrp, vout);
  else
    k_merge_tile<kMergeThreads><<<(unsigned)tile_count, kMergeThreads, smem, st>>>(
        keys, rp, d_off, k, total, ranks, rank_tile0, tile_begin, out, out_origin, out_f64 ? 1 : 0);
  return launched();
}

}  // namespace hsort
