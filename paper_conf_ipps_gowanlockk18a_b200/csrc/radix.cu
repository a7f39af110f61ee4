// radix.cu — GPUSort (§III-B) re-designed for sm_100a.
//
// The paper sorts each batch with Thrust (a CUB radix sort, out-of-place, 2x memory).
// Here the same step is a hand-written LSD onesweep radix sort over 64-bit keys:
//
//   K1 k_hist      one streaming read of the batch -> all 8 digit histograms (8 x 256), with the
//                  float64 -> order-preserving uint64 key transform applied in registers.
//   K2 k_scan_plan exclusive scans -> bin bases; digits with one non-empty bin are "trivial" and
//                  skipped; writes the device pass plan (src/dst ping-pong) so no host sync.
//   K3 k_onesweep  one 8-bit LSD digit pass per launch: tile load (warp-striped, coalesced) ->
//                  warp match.any ranking -> decoupled look-back prefix over tiles (per digit) ->
//                  shared-memory-staged scatter so global stores are runs of consecutive keys.
//                  The key transform is fused into the first pass's load and the inverse into
//                  the last pass's store.
//
// All arithmetic is integer; no tensor cores (not a contraction).  HBM bytes per key:
// K1 8, each K3 pass 16.
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdlib>
#include <type_traits>

#include "internal.h"

namespace hsort {
namespace {

constexpr int kDigits = 8;
constexpr int kRadix = 256;
constexpr uint64_t kFlagA = 1ull << 62;  // aggregate (tile count) available
constexpr uint64_t kFlagP = 2ull << 62;  // inclusive prefix available
constexpr uint64_t kCountMask = (1ull << 40) - 1;
constexpr uint32_t kEpochMask = (1u << 22) - 1;
#ifdef HSORT_PHASE_TIMING
__device__ unsigned long long g_phase_dbg[256];  // instrumented builds only
#ifndef HSORT_FAKE
#define HSORT_FAKE 0  // tools/ab_build.sh timing experiments (1 no look-back, 2 no ranking, 3 no write-out)
#endif
#endif

// float64 bits -> key: negative -> ~u, non-negative -> u | 2^63 (IEEE totalOrder as unsigned).
__device__ __forceinline__ uint64_t to_key(uint64_t u) {
  return u ^ ((uint64_t)((int64_t)u >> 63) | 0x8000000000000000ull);
}
// key -> float64 bits (inverse of to_key).
__device__ __forceinline__ uint64_t from_key(uint64_t k) {
  return k ^ ((uint64_t)((int64_t)(~k) >> 63) | 0x8000000000000000ull);
}

// float32 bits -> 32-bit key (the binary32 analogue of A4) and back (S§8(f) #4, native path)
__device__ __forceinline__ uint32_t to_key32(uint32_t w) {
  return w ^ ((uint32_t)((int32_t)w >> 31) | 0x80000000u);
}
__device__ __forceinline__ uint32_t from_key32(uint32_t k) {
  return k ^ ((uint32_t)((int32_t)(~k) >> 31) | 0x80000000u);
}
// key transform / inverse for the key width of a pass (64-bit: float64, 32-bit: float32)
__device__ __forceinline__ uint64_t to_key_w(uint64_t u) { return to_key(u); }
__device__ __forceinline__ uint32_t to_key_w(uint32_t w) { return to_key32(w); }
__device__ __forceinline__ uint64_t from_key_w(uint64_t k) { return from_key(k); }
__device__ __forceinline__ uint32_t from_key_w(uint32_t k) { return from_key32(k); }

__device__ __forceinline__ uint64_t ld_stream(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.global.nc.L1::no_allocate.u64 %0, [%1];" : "=l"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ void ld_stream2(const uint64_t* p, uint64_t& a, uint64_t& b) {
  asm volatile("ld.global.nc.L1::no_allocate.v2.u64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "l"(p));
}
__device__ __forceinline__ uint64_t ld_relaxed(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_relaxed(uint64_t* p, uint64_t v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint32_t ld_relaxed32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_relaxed32(uint32_t* p, uint32_t v) {
  asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

// ------------------------------------------------------------------------------------------
// ------------------------------------------------------------------------------------------
// Block-wide exclusive scan of one uint64 per thread over the first 256 threads (8 warps).
__device__ __forceinline__ uint64_t scan256_excl(uint64_t v, uint64_t* s_warp /*[8]*/,
                                                 uint64_t* total) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint64_t x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    uint64_t y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (threadIdx.x < 256 && lane == 31) s_warp[warp] = x;
  __syncthreads();
  uint64_t wpre = 0, tot = 0;
#pragma unroll
  for (int w = 0; w < 8; ++w) {
    uint64_t s = s_warp[w];
    if (w < warp) wpre += s;
    tot += s;
  }
  __syncthreads();
  if (total) *total = tot;
  return wpre + x - v;
}

// K2: bin bases + pass plan.  One CTA of 256 threads.
// dde_cap > 0: the dominant-digit elision may be planned (outliers <= dde_cap).
__global__ void __launch_bounds__(256) k_scan_plan(const uint64_t* __restrict__ hist,
                                                   uint64_t* __restrict__ bin_base,
                                                   RadixPlan* __restrict__ plan, uint64_t n,
                                                   int in_eq_out, int in_f64, int out_f64,
                                                   uint32_t* __restrict__ lb_state,
                                                   uint64_t dde_cap = 0,
                                                   const DdeState* __restrict__ dde = nullptr,
                                                   int desc = 0) {
  __shared__ uint64_t s_warp[8];
  __shared__ int s_nz[kDigits];
  __shared__ float s_dist[kDigits][8];
  const int t = threadIdx.x;
  // descending: the passes sort complemented keys, whose digit value t is digit 255 - t of K1
  const int tq = desc ? kRadix - 1 - t : t;
  for (int p = 0; p < kDigits; ++p) {
    uint64_t v = hist[p * kRadix + tq];
    uint64_t e = scan256_excl(v, s_warp, nullptr);
    bin_base[p * kRadix + t] = e;
    int nz = __syncthreads_count(v != 0);
    if (t == 0) s_nz[p] = nz;
    // expected number of distinct digits among 32 keys: D = sum_b 1 - (1 - p_b)^32.  MATCH.ANY
    // costs ~0.06 SM-cycles/key per distinct value, the ballot multisplit ~1.0 (microbench).
    float q = n ? 1.0f - (float)v / (float)n : 1.0f;
    float q2 = q * q, q4 = q2 * q2, q8 = q4 * q4, q16 = q8 * q8;
    float term = 1.0f - q16 * q16;
#pragma unroll
    for (int o = 16; o; o >>= 1) term += __shfl_xor_sync(0xffffffffu, term, o);
    if ((t & 31) == 0) s_dist[p][t >> 5] = term;
  }
  __syncthreads();
  if (t == 0) {
    RadixPlan P;
    int na = 0;
    for (int p = 0; p < kDigits; ++p)
      if (s_nz[p] > 1) P.digit[na++] = p;
    for (int p = na; p < kDigits; ++p) P.digit[p] = -1;
    P.dde = 0;
    P.dde_digit = -1;
    P.dde_value = 0;
    P.dde_pass = -1;
    P.dde_n_out = 0;
    P.dde_n_less = 0;
    P.dde_k1 = 0;
    P.key_xor = desc ? ~0ull : 0ull;
    if (dde_cap && na >= 3) {
      // top active digit L: dominant value v; elide its pass if the outliers fit the side buffer
      // and the remaining na - 1 passes still end in out without a final copy
      const int L = P.digit[na - 1];
      uint64_t best = 0, below = 0, below_best = 0;
      uint32_t v = 0;
      for (int b = 0; b < kRadix; ++b) {
        const uint64_t c = hist[L * kRadix + (desc ? kRadix - 1 - b : b)];
        if (c > best) {
          best = c;
          v = (uint32_t)b;
          below_best = below;
        }
        below += c;
      }
      const uint64_t n_out = n - best;
      if (n_out <= dde_cap && (!in_eq_out || ((na - 1) & 1) == 0)) {
        P.dde = 1;
        P.dde_digit = L;
        P.dde_value = v;
        --na;
        P.dde_pass = na - 1;
        P.digit[na] = -1;
        P.dde_n_out = n_out;
        P.dde_n_less = below_best;
        // K1 counted the outliers' digit-6 histogram if the guess (key 0's top digit) was right
        P.dde_k1 = (dde && !desc && L == 7 && P.digit[na - 1] == 6 && v == dde->guess) ? 1 : 0;
      }
    }
    P.num_active = na;
    P.copy_src = -1;
    P.copy_in_f64 = 0;
    P.copy_out_f64 = 0;
    P.lb_parity = lb_state ? (int32_t)(*lb_state & 1u) : 0;
    if (lb_state) *lb_state += (uint32_t)na;
    P.match_mask = 0;
    for (int q = 0; q < na; ++q) {
      float dsum = 0;
      for (int w = 0; w < 8; ++w) dsum += s_dist[P.digit[q]][w];
      if (dsum < 12.0f) P.match_mask |= 1 << q;
    }
    // ping-pong assignment: buffers 0 = in, 1 = out, 2 = tmp; the last pass must land in out
    int cur = 0;
    if (!in_eq_out) {
      int nxt = (na & 1) ? 1 : 2;
      for (int p = 0; p < na; ++p) {
        P.src[p] = cur;
        P.dst[p] = nxt;
        cur = nxt;
        nxt = (nxt == 1) ? 2 : 1;
      }
    } else {
      int nxt = 2;
      for (int p = 0; p < na; ++p) {
        P.src[p] = cur;
        P.dst[p] = nxt;
        cur = nxt;
        nxt = (nxt == 2) ? 0 : 2;
      }
      if (na & 1) P.copy_src = 2;  // result sits in tmp: raw copy tmp -> out
    }
    for (int p = na; p < kDigits; ++p) { P.src[p] = -1; P.dst[p] = -1; }
    if (na == 0 && n > 0) {
      // every digit trivial: all keys identical (or n == 1): out = converted in
      if (!in_eq_out || in_f64 != out_f64) {
        P.copy_src = 0;
        P.copy_in_f64 = in_f64;
        P.copy_out_f64 = out_f64;
      }
    }
    *plan = P;
  }
}

// Single-pass plan (tests / hsort_device_radix_pass): in -> out by `digit`.
__global__ void k_force_plan(RadixPlan* plan, int digit, uint32_t* lb_state) {
  RadixPlan P;
  P.lb_parity = (int32_t)(*lb_state & 1u);
  *lb_state += 1u;
  P.num_active = 1;
  for (int p = 0; p < kDigits; ++p) { P.digit[p] = -1; P.src[p] = -1; P.dst[p] = -1; }
  P.digit[0] = digit;
  P.src[0] = 0;
  P.dst[0] = 1;
  P.copy_src = -1;
  P.copy_in_f64 = P.copy_out_f64 = P.match_mask = 0;
  P.dde = 0;
  P.dde_digit = -1;
  P.dde_value = 0;
  P.dde_pass = -1;
  P.dde_n_out = P.dde_n_less = 0;
  P.dde_k1 = 0;
  P.key_xor = 0;
  *plan = P;
}

template <class T>
__device__ __forceinline__ T* pick(int id, T* in, T* out, T* tmp) {
  return id == 0 ? in : (id == 1 ? out : tmp);
}

// ------------------------------------------------------------------------------------------
// K3: one onesweep LSD pass.  Tile = THREADS x ITEMS keys; tile ids are taken from an atomic
// counter in launch order so every tile this CTA waits on is already resident (forward progress
// of the look-back).
template <int THREADS, int ITEMS, bool IN_F64>
__global__ void __launch_bounds__(THREADS) k_onesweep(uint64_t* in, uint64_t* out, uint64_t* tmp,
                                                       uint64_t n, const RadixPlan* __restrict__ plan,
                                                       const uint64_t* __restrict__ bin_base,
                                                       uint64_t* __restrict__ lookback,
                                                       uint32_t* __restrict__ tile_ctr,
                                                       uint32_t epoch, int p, int out_f64) {
  constexpr int WARPS = THREADS / 32;
  constexpr int TILE = THREADS * ITEMS;
  static_assert(THREADS >= 256, "one thread per digit");
  __shared__ uint64_t s_keys[TILE];
  __shared__ uint32_t s_whist[WARPS][kRadix + 1];
  __shared__ uint32_t s_tstart[kRadix];
  __shared__ uint64_t s_gofs[kRadix];
  __shared__ uint64_t s_warp[8];
  __shared__ uint32_t s_tile;

  const int na = plan->num_active;
  if (p >= na) return;
  const int digit = plan->digit[p];
  const int shift = 8 * digit;
  const uint64_t* __restrict__ src = pick(plan->src[p], in, out, tmp);
  uint64_t* __restrict__ dst = pick(plan->dst[p], in, out, tmp);
  const bool inv = out_f64 && (p == na - 1);
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;

  if (tid == 0) s_tile = atomicAdd(&tile_ctr[p], 1u);
  for (int i = tid; i < WARPS * (kRadix + 1); i += THREADS) (&s_whist[0][0])[i] = 0;
  __syncthreads();
  const uint64_t tile = s_tile;
  const uint64_t tbase = tile * TILE;
  const uint64_t wbase = tbase + (uint64_t)warp * 32 * ITEMS;

  // ---- load (warp-striped: item i of lane l is key wbase + i*32 + l; coalesced 256 B/warp)
  uint64_t k[ITEMS];
#pragma unroll
  for (int i = 0; i < ITEMS; ++i) {
    uint64_t idx = wbase + (uint64_t)i * 32 + lane;
    k[i] = idx < n ? ld_stream(src + idx) : 0;
  }
  // ---- rank: stable within the warp (item-major, then lane), per-warp digit counters
  uint32_t r[ITEMS];
  const uint32_t lt = lanemask_lt();
#pragma unroll
  for (int i = 0; i < ITEMS; ++i) {
    uint64_t idx = wbase + (uint64_t)i * 32 + lane;
    if (IN_F64) k[i] = to_key(k[i]);
    uint32_t d = idx < n ? ((uint32_t)(k[i] >> shift) & 255u) : (uint32_t)kRadix;
    uint32_t peers = __match_any_sync(0xffffffffu, d);
    int leader = __ffs(peers) - 1;
    uint32_t old = 0;
    if (lane == leader) {
      old = s_whist[warp][d];
      s_whist[warp][d] = old + __popc(peers);
    }
    old = __shfl_sync(0xffffffffu, old, leader);
    r[i] = old + __popc(peers & lt);
    __syncwarp();
  }
  __syncthreads();

  // ---- per digit: warp-exclusive offsets, tile count, early aggregate publish
  uint64_t cnt = 0;
  if (tid < kRadix) {
    uint32_t run = 0;
#pragma unroll
    for (int w = 0; w < WARPS; ++w) {
      uint32_t c = s_whist[w][tid];
      s_whist[w][tid] = run;
      run += c;
    }
    cnt = run;
    uint64_t word = (tile == 0 ? kFlagP : kFlagA) | ((uint64_t)(epoch & kEpochMask) << 40) | cnt;
    st_relaxed(&lookback[tile * kRadix + tid], word);
  }
  uint64_t tstart = scan256_excl(cnt, s_warp, nullptr);
  if (tid < kRadix) s_tstart[tid] = (uint32_t)tstart;
  __syncthreads();

  // ---- stage the tile in shared memory in digit order
#pragma unroll
  for (int i = 0; i < ITEMS; ++i) {
    uint64_t idx = wbase + (uint64_t)i * 32 + lane;
    if (idx < n) {
      uint32_t d = (uint32_t)(k[i] >> shift) & 255u;
      s_keys[s_tstart[d] + s_whist[warp][d] + r[i]] = k[i];
    }
  }

  // ---- decoupled look-back (thread = digit)
  if (tid < kRadix) {
    uint64_t excl = 0;
    if (tile > 0) {
      int64_t j = (int64_t)tile - 1;
      const uint32_t ep = epoch & kEpochMask;
      while (j >= 0) {
        uint64_t w = ld_relaxed(&lookback[(uint64_t)j * kRadix + tid]);
        uint64_t flag = w & (3ull << 62);
        if (flag == 0 || (uint32_t)((w >> 40) & kEpochMask) != ep) continue;  // not yet published
        excl += w & kCountMask;
        if (flag == kFlagP) break;
        --j;
      }
      st_relaxed(&lookback[tile * kRadix + tid],
                 kFlagP | ((uint64_t)ep << 40) | (excl + cnt));
    }
    s_gofs[tid] = bin_base[digit * kRadix + tid] + excl - (uint64_t)s_tstart[tid];
  }
  __syncthreads();

  // ---- coalesced scatter: consecutive smem slots are runs of one digit -> consecutive HBM
  const uint64_t rem = n - tbase;
  const int tile_n = rem < (uint64_t)TILE ? (int)rem : TILE;
  if (inv) {
#pragma unroll 4
    for (int j = tid; j < tile_n; j += THREADS) {
      uint64_t v = s_keys[j];
      dst[s_gofs[(uint32_t)(v >> shift) & 255u] + j] = from_key(v);
    }
  } else {
#pragma unroll 4
    for (int j = tid; j < tile_n; j += THREADS) {
      uint64_t v = s_keys[j];
      dst[s_gofs[(uint32_t)(v >> shift) & 255u] + j] = v;
    }
  }
}

constexpr int kPassThreads = 256;
constexpr int kPassItems = kRadixTile / kPassThreads;
static_assert(kPassThreads * kPassItems == kRadixTile, "tile");

// ------------------------------------------------------------------------------------------
// K3 v2: persistent onesweep pass with TMA bulk tile prefetch.
//
// Each resident CTA loops over tiles taken from the pass's atomic counter.  While it ranks and
// scatters tile i, one elected thread has already issued a cp.async.bulk (TMA, SASS UBLKCP) of
// tile i+1 into the other half of a double-buffered shared-memory stage, completing on an
// mbarrier; so the HBM read latency of the next tile overlaps the current tile's work.  The
// stage buffer that held tile i is reused as the digit-ordered scatter buffer of tile i.
// Forward progress of the look-back: a CTA holds at most one claimed-but-unstarted tile, which
// was claimed after its current tile, so the smallest current tile never waits on it.
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_fence_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tWAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra WAIT_%=;\n\t}" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}

// Windowed decoupled look-back for one digit: reads the status words of W predecessor tiles
// per round trip (independent loads in flight) and accumulates aggregates back to the first
// inclusive prefix.  A serial walk costs one L2 round trip per step and, with tiles claimed a
// few tens of cycles apart, needs ~latency/interval steps; the window resolves them together.
template <int W, int BO = 0>
__device__ __forceinline__ uint64_t lookback_window(const uint64_t* __restrict__ lookback,
                                                    int64_t j, int d, uint32_t ep) {
  uint64_t excl = 0;
  while (true) {
#ifdef HSORT_PHASE_TIMING
    if (d == 0) atomicAdd(&g_phase_dbg[200], 1ull);
#endif
    uint64_t w[W];
#pragma unroll
    for (int q = 0; q < W; ++q)
      w[q] = (j - q >= 0) ? ld_relaxed(&lookback[(uint64_t)(j - q) * kRadix + d])
                          : (kFlagP | ((uint64_t)ep << 40));  // before tile 0: prefix 0
    int q = 0;
    bool done = false;
#pragma unroll
    for (int u = 0; u < W; ++u) {
      if (done || q != u) continue;
      const uint64_t flag = w[u] & (3ull << 62);
      if (flag == 0 || (uint32_t)((w[u] >> 40) & kEpochMask) != ep) continue;  // not yet: re-read
      excl += w[u] & kCountMask;
      if (flag == kFlagP) done = true;
      else ++q;
    }
    if (done) return excl;
    if (BO > 0 && q == 0) __nanosleep(BO);  // predecessor not published yet: back off the L2
    j -= q;  // all consumed aggregates; re-read from the first unavailable tile
  }
}

// 32-bit status words (n <= 2^30): [31:30] flag (1 aggregate, 2 inclusive prefix), [29:0] count.
// Two arrays alternate between passes and each pass zeroes the rows of the other one, so no
// epoch tag is needed; half the L2 traffic of the 64-bit words.
template <int W>
__device__ __forceinline__ uint32_t lookback_window32(const uint32_t* __restrict__ lb, int64_t j,
                                                      int d) {
  uint32_t excl = 0;
  while (true) {
    uint32_t w[W];
#pragma unroll
    for (int q = 0; q < W; ++q)
      w[q] = (j - q >= 0) ? ld_relaxed32(&lb[(uint64_t)(j - q) * kRadix + d]) : (2u << 30);
    int q = 0;
    bool done = false;
#ifdef HSORT_PHASE_TIMING
    if (d == 0) {
      atomicAdd(&g_phase_dbg[200], 1ull);                      // rounds
      if ((w[0] >> 30) == 0) atomicAdd(&g_phase_dbg[201], 1ull);  // nearest unpublished: spin
      if ((w[0] >> 30) == 2) atomicAdd(&g_phase_dbg[202], 1ull);  // nearest has P
    }
#endif
#pragma unroll
    for (int u = 0; u < W; ++u) {
      if (done || q != u) continue;
      const uint32_t flag = w[u] >> 30;
      if (flag == 0) continue;  // not yet published: re-read
      excl += w[u] & 0x3FFFFFFFu;
      if (flag == 2) done = true;
      else ++q;
    }
    if (done) return excl;
    j -= q;
  }
}

#ifdef HSORT_PHASE_TIMING
#define HSORT_PHASE(i)                         \
  if (tid == 0) {                              \
    const long long _now = clock64();          \
    ph_acc[i] += (unsigned long long)(_now - ph_last); \
    ph_last = _now;                            \
  }
#else
#define HSORT_PHASE(i)
#endif

template <int THREADS, int ITEMS>
struct TmaPassSmem {
  static constexpr int WARPS = THREADS / 32;
  static constexpr int TILE = THREADS * ITEMS;
  static constexpr size_t stage_off = 0;                                   // [2][TILE] u64
  static constexpr size_t whist_off = stage_off + 2ull * TILE * 8;         // [WARPS][257] u32
  static constexpr size_t gofs_off = (whist_off + (size_t)WARPS * (kRadix + 1) * 4 + 15) & ~(size_t)15;  // [256] u64
  static constexpr size_t bar_off = gofs_off + kRadix * 8;                 // [2] u64
  static constexpr size_t swarp_off = bar_off + 16;                        // [8] u64
  static constexpr size_t tile_off = swarp_off + 64;                       // [2] u32
  static constexpr size_t bytes = tile_off + 16;
};

template <int THREADS, int ITEMS, bool IN_F64, int LBW, int MINB, bool S32>
__global__ void __launch_bounds__(THREADS, MINB) k_onesweep_tma(uint64_t* in, uint64_t* out, uint64_t* tmp,
                                                           uint64_t n,
                                                           const RadixPlan* __restrict__ plan,
                                                           const uint64_t* __restrict__ bin_base,
                                                           uint64_t* __restrict__ lookback,
                                                           uint32_t* __restrict__ tile_ctr,
                                                           uint32_t epoch, int p, int out_f64,
                                                           uint64_t lb_half, uint64_t lb_rows) {
  using L = TmaPassSmem<THREADS, ITEMS>;
  constexpr int WARPS = L::WARPS;
  constexpr int TILE = L::TILE;
  static_assert(THREADS >= 256 && THREADS % 32 == 0, "one thread per digit");
  extern __shared__ __align__(128) unsigned char smem[];
  uint64_t* stage = (uint64_t*)(smem + L::stage_off);
  uint32_t* whist = (uint32_t*)(smem + L::whist_off);
  uint64_t* s_gofs = (uint64_t*)(smem + L::gofs_off);
  uint64_t* bars = (uint64_t*)(smem + L::bar_off);
  uint64_t* s_warp = (uint64_t*)(smem + L::swarp_off);
  uint32_t* s_tile = (uint32_t*)(smem + L::tile_off);

  const int na = plan->num_active;
  if (p >= na) return;
  const int digit = plan->digit[p];
  const int shift = 8 * digit;
  const uint64_t* __restrict__ src = pick(plan->src[p], in, out, tmp);
  uint64_t* __restrict__ dst = pick(plan->dst[p], in, out, tmp);
  const bool use_match = (plan->match_mask >> p) & 1;
  const bool inv = out_f64 && (p == na - 1);
  uint32_t* lb32 = (uint32_t*)lookback + (uint64_t)((plan->lb_parity + p) & 1) * lb_half;
  uint32_t* lb32_next = (uint32_t*)lookback + (uint64_t)((plan->lb_parity + p + 1) & 1) * lb_half;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint64_t num_tiles = (n + TILE - 1) / TILE;
  const uint32_t ep = epoch & kEpochMask;

  auto issue = [&](uint64_t t, int b) {  // one thread: claim stage b for tile t
    const uint64_t base = t * (uint64_t)TILE;
    const uint64_t cnt = (n - base) < (uint64_t)TILE ? (n - base) : (uint64_t)TILE;
    const uint32_t bytes = (uint32_t)(cnt * 8) & ~15u;
    // WAR on the buffer (generic reads/writes of the previous tile) is ordered by the
    // __syncthreads that precedes every issue; no proxy fence is needed for a TMA load.
    mbar_arrive_expect_tx(&bars[b], bytes);
    if (bytes) bulk_g2s(stage + (size_t)b * TILE, src + base, bytes, &bars[b]);
  };

  // this thread's digit base for the pass, loaded once (not an L2 round trip after each look-back)
  const uint64_t my_bin_base = tid < kRadix ? bin_base[digit * kRadix + tid] : 0;
  uint32_t claim_next = 0;  // thread 0: tile id claimed one iteration ahead (atomic off the path)
  if (tid == 0) {
    mbar_init(&bars[0], 1);
    mbar_init(&bars[1], 1);
    mbar_fence_init();
    uint32_t t = atomicAdd(&tile_ctr[p], 1u);
    s_tile[0] = t;
    if (t < num_tiles) issue(t, 0);
    claim_next = atomicAdd(&tile_ctr[p], 1u);
  }
  __syncthreads();
  uint32_t phase = 0;  // bit b = parity to wait for on bars[b]
  int cb = 0;
  const uint32_t lt = lanemask_lt();
#ifdef HSORT_PHASE_TIMING
  unsigned long long ph_acc[10] = {0, 0, 0, 0, 0, 0, 0, 0, 0, 0};
  long long ph_last = clock64();
  unsigned long long ph_tiles = 0;
#endif
  while (true) {
    const uint64_t tile = s_tile[cb];
    if (tile >= num_tiles) break;
    if (tid == 0) {
      const uint32_t t = claim_next;
      s_tile[cb ^ 1] = t;
      if (t < num_tiles) {
        issue(t, cb ^ 1);
        claim_next = atomicAdd(&tile_ctr[p], 1u);
      }
    }
    for (int i = tid; i < WARPS * (kRadix + 1); i += THREADS) whist[i] = 0;
    mbar_wait(&bars[cb], (phase >> cb) & 1u);
    phase ^= 1u << cb;
    __syncthreads();
    HSORT_PHASE(0);

    const uint64_t tbase = tile * (uint64_t)TILE;
    const uint64_t rem = n - tbase;
    const int tile_n = rem < (uint64_t)TILE ? (int)rem : TILE;
    const bool full = tile_n == TILE;
    const int bulk_n = (int)(((uint32_t)tile_n * 8u & ~15u) >> 3);
    uint64_t* sb = stage + (size_t)cb * TILE;
    const int wofs = warp * 32 * ITEMS + lane;
    uint32_t* wh = whist + warp * (kRadix + 1);

    // ---- keys: shared stage -> registers (warp-striped: conflict-free 8-byte reads)
    uint64_t k[ITEMS];
#pragma unroll
    for (int i = 0; i < ITEMS; ++i) {
      const int j = wofs + i * 32;
      uint64_t v;
      if (full) v = sb[j];
      else v = j < bulk_n ? sb[j] : (j < tile_n ? src[tbase + j] : 0);
      k[i] = IN_F64 ? to_key(v) : v;
    }
    // ---- early per-warp digit counts -> tile aggregate, published before the ranking (so a
    // successor's look-back never waits on it), and absolute shared-memory bases per
    // (warp, digit): tile-local digit start + the counts of the warps before.
#pragma unroll
    for (int i = 0; i < ITEMS; ++i) {
      const bool valid = full || (wofs + i * 32 < tile_n);
      atomicAdd(&wh[valid ? ((uint32_t)(k[i] >> shift) & 255u) : (uint32_t)kRadix], 1u);
    }
    __syncthreads();
    uint64_t cnt = 0;
    if (tid < kRadix) {
#pragma unroll
      for (int w = 0; w < WARPS; ++w) cnt += whist[w * (kRadix + 1) + tid];
      if (S32) {
        st_relaxed32(&lb32[tile * kRadix + tid], ((tile == 0 ? 2u : 1u) << 30) | (uint32_t)cnt);
        lb32_next[tile * kRadix + tid] = 0;  // the next pass's array, row of this tile
      } else {
        st_relaxed(&lookback[tile * kRadix + tid],
                   (tile == 0 ? kFlagP : kFlagA) | ((uint64_t)ep << 40) | cnt);
      }
    }
    const uint32_t tstart = (uint32_t)scan256_excl(cnt, s_warp, nullptr);
    if (tid < kRadix) {
      uint32_t run = tstart;
#pragma unroll
      for (int w = 0; w < WARPS; ++w) {
        const uint32_t c = whist[w * (kRadix + 1) + tid];
        whist[w * (kRadix + 1) + tid] = run;
        run += c;
      }
    }
    __syncthreads();
    HSORT_PHASE(2);

    // ---- rank: the highest peer lane's atomic on the warp's base returns the group's first
    // slot, so r[i] is the key's final position in the digit-ordered tile.  Three unrolled phases
    // keep the peer computations and the leaders' atomics of all items in flight together.
    uint32_t r[ITEMS];
    constexpr int RC = (MINB >= 3 && ITEMS % 2 == 0) ? ITEMS / 2 : ITEMS;  // ranking chunk
#pragma unroll
    for (int c0 = 0; c0 < ITEMS; c0 += RC) {
      uint32_t dd[RC], peers[RC];
#pragma unroll
      for (int i = 0; i < RC; ++i) {
        const bool valid = full || (wofs + (c0 + i) * 32 < tile_n);
        dd[i] = valid ? ((uint32_t)(k[c0 + i] >> shift) & 255u) : (uint32_t)kRadix;
      }
      // peers (lanes holding the same digit).  MATCH.ANY costs ~0.06 SM-cycles/key per distinct
      // value in the warp (1.9 for random 8-bit digits), an 8-ballot multisplit ~1.0
      // (profiles/r01_microbench_ranking2.txt); K2 picks per pass from the digit histogram.
      // Partial tiles mark invalid items with bit 8.
      if (use_match) {
#pragma unroll
        for (int i = 0; i < RC; ++i) peers[i] = __match_any_sync(0xffffffffu, dd[i]);
      } else {
#pragma unroll
        for (int i = 0; i < RC; ++i) peers[i] = 0xffffffffu;
#pragma unroll
        for (int b = 0; b < 8; ++b) {
#pragma unroll
          for (int i = 0; i < RC; ++i) {
            const uint32_t bit = (dd[i] >> b) & 1u;
            peers[i] &= __ballot_sync(0xffffffffu, bit) ^ (bit - 1u);
          }
        }
        if (!full) {
#pragma unroll
          for (int i = 0; i < RC; ++i) {
            const uint32_t bit = (dd[i] >> 8) & 1u;
            peers[i] &= __ballot_sync(0xffffffffu, bit) ^ (bit - 1u);
          }
        }
      }
#if HSORT_FAKE == 2  // timing experiment only: no ranking (wrong output)
#pragma unroll
      for (int i = 0; i < RC; ++i) peers[i] = 1u << lane;
#endif
#pragma unroll
      for (int i = 0; i < RC; ++i) {
        const int leader = 31 - __clz(peers[i]);
        r[c0 + i] = (lane == leader) ? atomicAdd(&wh[dd[i]], (uint32_t)__popc(peers[i])) : 0u;
      }
#pragma unroll
      for (int i = 0; i < RC; ++i) {
        const int leader = 31 - __clz(peers[i]);
        r[c0 + i] = __shfl_sync(0xffffffffu, r[c0 + i], leader) + __popc(peers[i] & lt);
      }
    }
    HSORT_PHASE(3);

    // ---- scatter into the (already consumed) stage buffer in digit order
#pragma unroll
    for (int i = 0; i < ITEMS; ++i)
      if (full || wofs + i * 32 < tile_n) sb[r[i]] = k[i];
    // ---- decoupled look-back (thread = digit), LBW predecessors read per round trip
    if (tid < kRadix) {
      uint64_t excl = 0;
      if (tile > 0) {
        if (S32) {
#if HSORT_FAKE == 1  // timing experiment only: no look-back (wrong output)
          excl = 0;
#else
          excl = lookback_window32<(LBW & 255)>(lb32, (int64_t)tile - 1, tid);
#endif
          st_relaxed32(&lb32[tile * kRadix + tid], (2u << 30) | (uint32_t)(excl + cnt));
        } else {
          excl = lookback_window<(LBW & 255), ((LBW >> 8) & 255)>(lookback, (int64_t)tile - 1, tid, ep);
          st_relaxed(&lookback[tile * kRadix + tid], kFlagP | ((uint64_t)ep << 40) | (excl + cnt));
        }
      }
      s_gofs[tid] = my_bin_base + excl - (uint64_t)tstart;
    }
    __syncthreads();
    HSORT_PHASE(4);

    // ---- write out: consecutive slots are runs of one digit -> coalesced HBM stores
    if (full) {
      constexpr int WC = (MINB >= 3) ? ITEMS / 2 : ITEMS;  // write-out chunk
#pragma unroll
      for (int c0 = 0; c0 < ITEMS; c0 += WC) {
        uint64_t v[WC], g[WC];
#pragma unroll
        for (int q = 0; q < WC; ++q) v[q] = sb[tid + (c0 + q) * THREADS];
#pragma unroll
        for (int q = 0; q < WC; ++q) g[q] = s_gofs[(uint32_t)(v[q] >> shift) & 255u];
        if (inv) {
#pragma unroll
          for (int q = 0; q < WC; ++q) dst[g[q] + tid + (c0 + q) * THREADS] = from_key(v[q]);
        } else {
#if HSORT_FAKE == 3  // timing experiment only: no HBM write-out (wrong output)
#pragma unroll
          for (int q = 0; q < WC; ++q)
            if (v[q] == 0x123456789ull) dst[g[q] + tid + (c0 + q) * THREADS] = v[q];
#else
#pragma unroll
          for (int q = 0; q < WC; ++q) dst[g[q] + tid + (c0 + q) * THREADS] = v[q];
#endif
        }
      }
    } else if (inv) {
#pragma unroll 4
      for (int j = tid; j < tile_n; j += THREADS) {
        const uint64_t v = sb[j];
        dst[s_gofs[(uint32_t)(v >> shift) & 255u] + j] = from_key(v);
      }
    } else {
#pragma unroll 4
      for (int j = tid; j < tile_n; j += THREADS) {
        const uint64_t v = sb[j];
        dst[s_gofs[(uint32_t)(v >> shift) & 255u] + j] = v;
      }
    }
    __syncthreads();
    HSORT_PHASE(5);
#ifdef HSORT_PHASE_TIMING
    ++ph_tiles;
#endif
    cb ^= 1;
  }
  // 32-bit mode: rows beyond this sort's tiles that an earlier, larger sort may have used
  if (S32)
    for (uint64_t r = num_tiles + blockIdx.x; r < lb_rows; r += gridDim.x)
      lb32_next[r * kRadix + tid] = 0;
#ifdef HSORT_PHASE_TIMING
  if (tid == 0) {
    for (int i = 0; i < 10; ++i) atomicAdd(&g_phase_dbg[p * 16 + (i < 8 ? i : i + 1)], ph_acc[i]);
    atomicAdd(&g_phase_dbg[p * 16 + 8], ph_tiles);
  }
#endif
}

// K1 v2: per-warp entropy probe picks, for each digit, either direct shared atomics (spread
// digits) or the register run-length cache (low-entropy digits, e.g. the exponent byte).
// DDE: also count digit 6 of the keys whose top digit differs from `guess` (the top digit of the
// first key) into hout -- the elision's outlier histogram for its common case L = 7, P = 6
// (DESIGN.md §6d), so pass 0 does not have to count it.
template <bool IN_F64, uint32_t MASK, int SH = 0, bool DDE = false>
__device__ __forceinline__ void hist2_key(uint64_t k, uint32_t* sh, uint32_t* cd, uint32_t* cc,
                                          uint32_t mask, uint32_t guess = 0,
                                          uint32_t* hout = nullptr) {
  if (IN_F64) k = to_key(k);
  const uint32_t lo = (uint32_t)k, hi = (uint32_t)(k >> 32);
  if (DDE && (hi >> 24) != guess) atomicAdd(&hout[(hi >> 16) & 255u], 1u);
#pragma unroll
  for (int p = 0; p < kDigits; ++p) {
    const uint32_t d = ((p < 4 ? lo : hi) >> (8 * (p & 3))) & 255u;
    const bool low = (MASK == 0xFFFFFFFFu) ? ((mask >> p) & 1u) : ((MASK >> p) & 1u);
    if (low) {
      if (d == cd[p]) {
        ++cc[p];
      } else {
        if (cc[p]) atomicAdd(&sh[(p * kRadix + cd[p]) << SH], cc[p]);
        cd[p] = d;
        cc[p] = 1;
      }
    } else {
      atomicAdd(&sh[(p * kRadix + d) << SH], 1u);
    }
  }
}

template <bool IN_F64, uint32_t MASK, int SH = 0, bool DDE = false>
__device__ __forceinline__ void hist2_loop(const uint64_t* base, uint64_t pairs, uint64_t i,
                                           uint64_t stride, uint32_t* sh, uint32_t* cd,
                                           uint32_t* cc, uint32_t mask, uint32_t guess = 0,
                                           uint32_t* hout = nullptr) {
  for (; i + 3 * stride < pairs; i += 4 * stride) {
    uint64_t a[8];
#pragma unroll
    for (int u = 0; u < 4; ++u) ld_stream2(base + 2 * (i + u * stride), a[2 * u], a[2 * u + 1]);
#pragma unroll
    for (int u = 0; u < 8; ++u) hist2_key<IN_F64, MASK, SH, DDE>(a[u], sh, cd, cc, mask, guess, hout);
  }
  for (; i < pairs; i += stride) {
    uint64_t a0, a1;
    ld_stream2(base + 2 * i, a0, a1);
    hist2_key<IN_F64, MASK, SH, DDE>(a0, sh, cd, cc, mask, guess, hout);
    hist2_key<IN_F64, MASK, SH, DDE>(a1, sh, cd, cc, mask, guess, hout);
  }
}

// K1 v3: as v2, but the shared histograms are replicated 8 times, interleaved so that counter
// (p, v) of copy c sits at word 8 (256 p + v) + c; lane L uses copy L & 7.  A warp's 32 atomics
// then spread over 32 banks by (v & 3, L & 7): only the 4 lanes sharing a copy can conflict (v2:
// all 32 lanes over 32 banks, ~3.7 wavefronts per atomic for random digits; K1 v2 was
// shared-atomic-bound at 99% of the L1 data pipe).  64 KB per CTA.
#ifndef HSORT_HIST_COPIES
#define HSORT_HIST_COPIES 16  // 16 copies: a half-warp's 16 lanes use 16 distinct banks
#endif
#ifndef HSORT_HIST_THREADS
#define HSORT_HIST_THREADS 1024  // 1 CTA (128 KB of copies) per SM
#endif
constexpr int kHist3Copies = HSORT_HIST_COPIES;
constexpr int kHist3Threads = HSORT_HIST_THREADS;
template <bool IN_F64, int THREADS, int COPIES, bool DDE = false>
__global__ void __launch_bounds__(THREADS) k_hist3(const uint64_t* __restrict__ src, uint64_t n,
                                                       uint64_t* __restrict__ hist,
                                                       DdeState* __restrict__ dde = nullptr) {
  constexpr int SHC = COPIES == 16 ? 4 : 3;
  extern __shared__ uint32_t sh3[];  // [8 * 256][COPIES] (+ DDE: [256] outlier digit-6 counts)
  // DDE: the outliers' histogram is counted in shared memory and flushed once per CTA -- global
  // atomics per outlier serialised at L2 when the guessed top digit is not dominant (normal data:
  // K1 took 168 ms instead of 2 ms, profiles/r02n_k1_dde_skew.txt)
  uint32_t* s_out = sh3 + kDigits * kRadix * COPIES;
  for (int i = threadIdx.x; i < kDigits * kRadix * COPIES + (DDE ? kRadix : 0); i += THREADS) sh3[i] = 0;
  __syncthreads();
  uint32_t* sh = sh3 + (threadIdx.x & (COPIES - 1));
  uint32_t cd[kDigits], cc[kDigits];
#pragma unroll
  for (int p = 0; p < kDigits; ++p) { cd[p] = 0; cc[p] = 0; }
  const uint64_t head = (((uintptr_t)src & 15) && n) ? 1 : 0;
  const uint64_t* base = src + head;
  const uint64_t m = n - head;
  const uint64_t pairs = m / 2;
  const uint64_t stride = (uint64_t)gridDim.x * THREADS;
  const uint64_t i0 = (uint64_t)blockIdx.x * THREADS + threadIdx.x;
  // entropy probe on this warp's first keys: <= 4 distinct values among 32 lanes -> run cache
  uint32_t mask = 0;
  {
    uint64_t k = i0 < pairs ? base[2 * i0] : (m ? base[0] : 0);
    if (IN_F64) k = to_key(k);
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int p = 0; p < kDigits; ++p) {
      const uint32_t d = (uint32_t)(k >> (8 * p)) & 255u;
      const uint32_t peers = __match_any_sync(0xffffffffu, d);
      const uint32_t leaders = __ballot_sync(0xffffffffu, lane == 31 - __clz(peers));
      if (__popc(leaders) <= 4) mask |= 1u << p;
    }
  }
  uint32_t guess = 0;
  uint32_t* hout = nullptr;
  if (DDE) {
    uint64_t k0 = n ? src[0] : 0;
    if (IN_F64) k0 = to_key(k0);
    guess = (uint32_t)(k0 >> 56);
    hout = s_out;
    if (blockIdx.x == 0 && threadIdx.x == 0) dde->guess = guess;
  }
  if (head && blockIdx.x == 0 && threadIdx.x == 0)
    hist2_key<IN_F64, 0xFFFFFFFFu, SHC, DDE>(src[0], sh, cd, cc, 0xFF, guess, hout);
  if (mask == 0x80u) hist2_loop<IN_F64, 0x80u, SHC, DDE>(base, pairs, i0, stride, sh, cd, cc, mask, guess, hout);
  else if (mask == 0u) hist2_loop<IN_F64, 0u, SHC, DDE>(base, pairs, i0, stride, sh, cd, cc, mask, guess, hout);
  else if (mask == 0xC0u) hist2_loop<IN_F64, 0xC0u, SHC, DDE>(base, pairs, i0, stride, sh, cd, cc, mask, guess, hout);
  else hist2_loop<IN_F64, 0xFFFFFFFFu, SHC, DDE>(base, pairs, i0, stride, sh, cd, cc, mask, guess, hout);
  if ((m & 1) && blockIdx.x == gridDim.x - 1 && threadIdx.x == THREADS - 1)
    hist2_key<IN_F64, 0xFFFFFFFFu, SHC, DDE>(base[m - 1], sh, cd, cc, 0xFF, guess, hout);
#pragma unroll
  for (int p = 0; p < kDigits; ++p)
    if (cc[p]) atomicAdd(&sh[(p * kRadix + cd[p]) << SHC], cc[p]);
  __syncthreads();
  for (int j = threadIdx.x; j < kDigits * kRadix; j += THREADS) {
    uint32_t c = 0;
#pragma unroll
    for (int q = 0; q < COPIES; q += 4) {
      const uint4 a = *(const uint4*)&sh3[j * COPIES + q];
      c += a.x + a.y + a.z + a.w;
    }
    if (c) atomicAdd((unsigned long long*)&hist[j], (unsigned long long)c);
  }
  if (DDE)
    for (int j = threadIdx.x; j < kRadix; j += THREADS)
      if (s_out[j]) atomicAdd(&dde->hist_k1[j], s_out[j]);
}

// Final conversion/copy (P_eff == 0, or odd P_eff with in == out).
// Key/value sorts pass the value buffers (same buffer ids); keys-only sorts pass nullptr.
__global__ void k_final_copy(uint64_t* in, uint64_t* out, uint64_t* tmp, uint64_t n,
                             const RadixPlan* __restrict__ plan, uint64_t* vin = nullptr,
                             uint64_t* vout = nullptr, uint64_t* vtmp = nullptr) {
  const int cs = plan->copy_src;
  if (cs < 0) return;
  const uint64_t* s = pick(cs, in, out, tmp);
  const uint64_t* vs = vin ? pick(cs, vin, vout, vtmp) : nullptr;
  const bool fin = plan->copy_in_f64, fout = plan->copy_out_f64;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t v = s[i];
    if (fin != fout) v = fin ? to_key(v) : from_key(v);
    out[i] = v;
    if (vs && vs != vout) vout[i] = vs[i];
  }
}

// Dominant-digit elision, last step: the sorted outliers (side[0, n_out), internal keys) go to
// out[0, n_less) (digit L below the dominant value) and out[n - (n_out - n_less), n) (above).
__global__ void k_dde_place(const uint64_t* __restrict__ side, uint64_t n_out, uint64_t n_less,
                            uint64_t* __restrict__ out, uint64_t n, int out_f64, uint64_t kx) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n_out;
       i += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t v = side[i];
    out[i < n_less ? i : n - n_out + i] = out_f64 ? from_key(v ^ kx) : v;
  }
}

int num_sms(int dev) {
  static int cached[64] = {0};
  if (dev < 0 || dev >= 64) return 148;
  if (!cached[dev]) {
    int v = 0;
    cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev);
    cached[dev] = v > 0 ? v : 148;
  }
  return cached[dev];
}

cudaError_t next_epoch(RadixScratch& s, cudaStream_t st, uint32_t* ep) {
  if (s.epoch >= kEpochMask) {
    cudaError_t e = cudaMemsetAsync(s.lookback, 0, s.max_tiles * kRadix * sizeof(uint64_t), st);
    if (e != cudaSuccess) return e;
    s.epoch = 0;
  }
  *ep = ++s.epoch;
  return cudaSuccess;
}

// Kernel selection: the TMA persistent pass (1, default) needs 16-byte aligned buffers; the
// register-load pass (0) is the fallback.  HSORT_PASS_VARIANT / HSORT_HIST_VARIANT override
// (experiments; DESIGN.md §6 lists the variants measured and removed).
int env_int(const char* name, int dflt) {
  const char* v = getenv(name);
  return v ? atoi(v) : dflt;
}
#ifndef HSORT_DEFAULT_PASS_VARIANT
#define HSORT_DEFAULT_PASS_VARIANT 2
#endif
int pass_variant() {
  static int v = env_int("HSORT_PASS_VARIANT", HSORT_DEFAULT_PASS_VARIANT);
  return v;
}
cudaError_t launch_hist(RadixScratch& s, const uint64_t* in, uint64_t n, bool in_f64,
                        uint64_t* hist, cudaStream_t st, DdeState* dde = nullptr) {
  int dev = 0;
  cudaGetDevice(&dev);
  {
    constexpr int smem = kDigits * kRadix * kHist3Copies * 4;
    auto kt = k_hist3<true, kHist3Threads, kHist3Copies>;
    auto kf = k_hist3<false, kHist3Threads, kHist3Copies>;
    auto kdt = k_hist3<true, kHist3Threads, kHist3Copies, true>;
    auto kdf = k_hist3<false, kHist3Threads, kHist3Copies, true>;
    static int per_sm[64] = {0};  // resident CTAs per SM, per device
    if (dev < 0 || dev >= 64) return cudaErrorInvalidDevice;
    if (!per_sm[dev]) {
      cudaError_t e;
      if ((e = cudaFuncSetAttribute(kt, cudaFuncAttributeMaxDynamicSharedMemorySize, smem)) != cudaSuccess) return e;
      if ((e = cudaFuncSetAttribute(kf, cudaFuncAttributeMaxDynamicSharedMemorySize, smem)) != cudaSuccess) return e;
      if ((e = cudaFuncSetAttribute(kdt, cudaFuncAttributeMaxDynamicSharedMemorySize, smem + kRadix * 4)) != cudaSuccess) return e;
      if ((e = cudaFuncSetAttribute(kdf, cudaFuncAttributeMaxDynamicSharedMemorySize, smem + kRadix * 4)) != cudaSuccess) return e;
      int b = 0;
      if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, kf, kHist3Threads, smem)) != cudaSuccess) return e;
      per_sm[dev] = b > 0 ? b : 1;
    }
    const uint64_t want3 = (n / 2 + kHist3Threads * 8 - 1) / (kHist3Threads * 8);
    const uint64_t cap3 = (uint64_t)num_sms(dev) * per_sm[dev];
    const int grid3 = (int)(want3 < 1 ? 1 : (want3 > cap3 ? cap3 : want3));
    if (dde) {
      if (in_f64) kdt<<<grid3, kHist3Threads, smem + kRadix * 4, st>>>(in, n, hist, dde);
      else kdf<<<grid3, kHist3Threads, smem + kRadix * 4, st>>>(in, n, hist, dde);
    } else {
      if (in_f64) kt<<<grid3, kHist3Threads, smem, st>>>(in, n, hist, nullptr);
      else kf<<<grid3, kHist3Threads, smem, st>>>(in, n, hist, nullptr);
    }
  }
  return launched();
}

template <int THREADS, int ITEMS, int LBW, int MINB, bool S32>
cudaError_t launch_tma_pass(uint64_t* in, uint64_t* out, uint64_t* tmp, uint64_t n,
                            RadixScratch& s, uint32_t ep, int p, bool first_in_f64, bool out_f64,
                            cudaStream_t st) {
  using L = TmaPassSmem<THREADS, ITEMS>;
  static int blocks_per_sm[64] = {0};
  int dev = 0;
  cudaGetDevice(&dev);
  auto kt = k_onesweep_tma<THREADS, ITEMS, true, LBW, MINB, S32>;
  auto kf = k_onesweep_tma<THREADS, ITEMS, false, LBW, MINB, S32>;
  if (dev < 0 || dev >= 64) return cudaErrorInvalidDevice;
  if (!blocks_per_sm[dev]) {
    cudaError_t e;
    if ((e = cudaFuncSetAttribute(kt, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)L::bytes)) != cudaSuccess) return e;
    if ((e = cudaFuncSetAttribute(kf, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)L::bytes)) != cudaSuccess) return e;
    int b = 0;
    if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, kf, THREADS, L::bytes)) != cudaSuccess) return e;
    blocks_per_sm[dev] = b > 0 ? b : 1;
  }
  const uint64_t tiles = (n + L::TILE - 1) / L::TILE;
  if (tiles > s.max_tiles) return cudaErrorInvalidValue;  // look-back array too small
  uint64_t grid = (uint64_t)num_sms(dev) * blocks_per_sm[dev];
  if (grid > tiles) grid = tiles ? tiles : 1;
  if (first_in_f64)
    kt<<<(unsigned)grid, THREADS, L::bytes, st>>>(in, out, tmp, n, s.plan, s.bin_base, s.lookback,
                                                 s.tile_ctr, ep, p, out_f64 ? 1 : 0,
                                                 s.max_tiles * kRadix, s.lb_rows);
  else
    kf<<<(unsigned)grid, THREADS, L::bytes, st>>>(in, out, tmp, n, s.plan, s.bin_base, s.lookback,
                                                 s.tile_ctr, ep, p, out_f64 ? 1 : 0,
                                                 s.max_tiles * kRadix, s.lb_rows);
  return launched();
}

// ------------------------------------------------------------------------------------------
// K3 v3: warp-specialised onesweep pass (default).  CTA = 8 compute warps + 1 look-back warp.
//
// The decoupled look-back is the largest single cost of a pass (removing it, output wrong, cuts a
// 2^30-key pass from 7.3 to 5.0 ms: profiles/r01_pass_floors.txt), and in v2 every thread of the
// CTA waits for it.  Here the look-back of tile t runs on its own warp (each lane owns 8 digits)
// while the compute warps rank the next tile; the compute warps write tile t out one iteration
// later.  The inclusive prefix is still published as soon as the look-back resolves, so
// successors wait no longer than in v2.  Three 4096-key stage buffers rotate: tile j+2 is
// prefetched (TMA) while tile j is ranked and tile j-1 is written out.
//
// Hand-offs (shared-memory mbarriers): bar_tma[3] TMA completion; bar_a[2] "tile j counted, A
// published, counts and tile starts in s_cnt" (compute -> look-back warp); bar_g[2] "global
// offsets of tile j in s_gofs" (look-back warp -> compute).  32-bit status words only (n <= 2^30).
// Forward progress: a CTA's claims increase, so the smallest tile without an inclusive prefix is
// either being looked back (its predecessor has P) or queued behind smaller tiles of its own CTA,
// which all have P, and nothing in the CTA waits on a larger tile.
template <int CT>
__device__ __forceinline__ void bar_compute() { asm volatile("bar.sync 1, %0;" ::"n"(CT) : "memory"); }
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

// exclusive scan of one value per digit thread (threads 0..255) among CT compute threads,
// named barrier 1 (threads >= 256 pass v = 0 and ignore the result)
template <int CT>
__device__ __forceinline__ uint32_t scan256_excl_c(uint32_t v, uint32_t* s_warp /*[8]*/) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint32_t x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31 && warp < 8) s_warp[warp] = x;
  bar_compute<CT>();
  uint32_t wpre = 0;
#pragma unroll
  for (int w = 0; w < 8; ++w)
    if (w < warp) wpre += s_warp[w];
  return wpre + x - v;
}

template <int CT, int ITEMS, bool KV = false, int KB = 8>
struct WsSmem {
  static constexpr int TILE = CT * ITEMS;
  static constexpr int CW = CT / 32;                                          // compute warps
  static constexpr size_t stage_off = 0;                                      // [3][TILE] keys (KB bytes)
  static constexpr size_t vstage_off = 3ull * TILE * KB;                      // [3][TILE] u64 (KV)
  static constexpr size_t whist_off = 3ull * TILE * KB + (KV ? 3ull * TILE * 8 : 0);  // [CW][257] u32
  static constexpr size_t gofs_off = (whist_off + CW * (kRadix + 1) * 4 + 15) & ~(size_t)15;  // [2][256] i32
  static constexpr size_t cnt_off = gofs_off + 2 * kRadix * 4;                // [2][256] u32
  static constexpr size_t bar_off = cnt_off + 2 * kRadix * 4;                 // [12] u64
  static constexpr size_t swarp_off = bar_off + 12 * 8;                       // [8] u32 (+pad)
  static constexpr size_t tile_off = swarp_off + 64;                          // [4] u32
  static constexpr size_t dummy_off = tile_off + 16;                          // [32] u32 (+pad)
  static constexpr size_t bytes = dummy_off + 32 * 4;
};

#ifndef HSORT_WS_CT
#define HSORT_WS_CT 576  // compute threads of the warp-specialised pass (18 warps + 1 look-back warp)
#endif
#ifndef HSORT_WS_ITEMS
#define HSORT_WS_ITEMS 15  // keys per compute thread: 8640-key tiles, 3 stages = 203 KB, 1 CTA/SM
#endif
#ifndef HSORT_K32_ITEMS
#define HSORT_K32_ITEMS 20  // 32-bit keys per compute thread: 11520-key tiles, 3 stages = 138 KB
                            // (A/B 15 / 18 / 20 / 22: 19.2 / 18.6 / 17.4 / 17.7 ms per 2^30 keys)
#endif
#ifndef HSORT_WS_NMATCH
#define HSORT_WS_NMATCH 4  // items ranked with match.any in high-entropy passes (A/B over 2..7)
#endif
#ifndef HSORT_KV_NMATCH
#define HSORT_KV_NMATCH 2  // ... in the key/value pass (13 items; A/B 2 / 3 / 4 / 5: 8.29 / 8.34 / 8.73 / 8.51 ms)
#endif
#ifndef HSORT_WS_W
#define HSORT_WS_W 4  // look-back rows per round trip in the warp-specialised pass
#endif
#ifndef HSORT_WS_PATOM
#define HSORT_WS_PATOM 1  // branch-free leader atomics: every lane issues one, a non-leader to a word
                          // of its own (A/B: a branch per item, predicated PTX and
                          // every lane adding to the digit's slot were slower)
#endif
#ifndef HSORT_WS_PATOM_DM2
#define HSORT_WS_PATOM_DM2 1  // ... also in the elision's diverting pass (A/B: 5.33 -> 5.23 ms)
#endif
#ifndef HSORT_WS_IL_K32
#define HSORT_WS_IL_K32 0  // interleaved write-out in the 32-bit-key pass (A/B: 17.55 vs 17.48 ms off)
#endif
#ifndef HSORT_WS_PATOM_K32
#define HSORT_WS_PATOM_K32 1  // branch-free leader atomics there (A/B: 18.63 ms without)
#endif
#ifndef HSORT_WS_IL_DM2
#define HSORT_WS_IL_DM2 0  // ... also in the elision's diverting pass (A/B: slower, spills)
#endif
#ifndef HSORT_WS_IL
#define HSORT_WS_IL 1  // write-out of tile j-1 interleaved with the ranking of tile j (full tiles)
#endif
// key/value pass: HSORT_KV_CT compute threads x HSORT_KV_ITEMS pairs (internal.h: 10 warps x 13)
constexpr int kKvCT = HSORT_KV_CT;
constexpr int kKvItems = HSORT_KV_ITEMS;
static_assert(kKvCT * kKvItems == kKvTile, "kKvTile (internal.h) = key/value tile");
__device__ __forceinline__ void ld_relaxed_v4(const uint32_t* p, uint32_t* v) {
  asm volatile("ld.relaxed.gpu.global.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3])
               : "l"(p)
               : "memory");
}
__device__ __forceinline__ void st_relaxed_v4(uint32_t* p, const uint32_t* v) {
  asm volatile("st.relaxed.gpu.global.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v[0]), "r"(v[1]),
               "r"(v[2]), "r"(v[3])
               : "memory");
}

__device__ __forceinline__ void st_global_u64(uint64_t addr, uint64_t v) {
  asm volatile("st.global.u64 [%0], %1;" ::"l"(addr), "l"(v) : "memory");
}
__device__ __forceinline__ void st_global_w(const uint64_t* a, uint64_t v) { st_global_u64((uint64_t)a, v); }
__device__ __forceinline__ void st_global_w(const uint32_t* a, uint32_t v) {
  asm volatile("st.global.u32 [%0], %1;" ::"l"((uint64_t)a), "r"(v) : "memory");
}
// One bit of the ballot multisplit: peers &= (bit b of d) ? ballot(bit) : ~ballot(bit).
__device__ __forceinline__ uint32_t peer_bit(uint32_t peers, uint32_t d, uint32_t bm) {
  uint32_t out;
  asm("{\n\t.reg .pred p;\n\t.reg .b32 B, t, m;\n\t"
      "and.b32 t, %1, %2;\n\t"
      "setp.ne.u32 p, t, 0;\n\t"
      "vote.sync.ballot.b32 B, p, 0xffffffff;\n\t"
      "selp.b32 m, 0, 0xffffffff, p;\n\t"
      "xor.b32 B, B, m;\n\t"
      "and.b32 %0, %3, B;\n\t}"
      : "=r"(out)
      : "r"(d), "r"(bm), "r"(peers));
  return out;
}

template <int W>
__device__ __forceinline__ void lookback8(const uint32_t* __restrict__ lb, int64_t tile, int lane,
                                          uint32_t* excl) {
  // Lane owns digits 8 lane .. 8 lane + 7 (two 16-byte loads per tile row).  The warp walks back
  // one tile row at a time for all 256 digits together, W rows per round trip.  Fast path: a row
  // whose 256 words are all aggregates is summed raw (flag bits removed once at the end).  Else
  // per digit: a digit stops at its first inclusive prefix, and the walk pauses (re-reads from
  // that row) while any still-walking digit's word is unpublished.
  uint32_t raw[8], msk[8];
#pragma unroll
  for (int q = 0; q < 8; ++q) raw[q] = msk[q] = 0;
  uint32_t live = 0xffu, n_raw = 0;
  const uint32_t* row0 = lb + lane * 8;
  int64_t j = tile - 1;
  while (true) {
#ifdef HSORT_PHASE_TIMING
    if (lane == 0) atomicAdd(&g_phase_dbg[216], 1ull);
#endif
    uint32_t w[W][8];
#pragma unroll
    for (int u = 0; u < W; ++u) {
      if (j - u >= 0) {
        ld_relaxed_v4(row0 + (uint64_t)(j - u) * kRadix, &w[u][0]);
        ld_relaxed_v4(row0 + (uint64_t)(j - u) * kRadix + 4, &w[u][4]);
      } else {
#pragma unroll
        for (int q = 0; q < 8; ++q) w[u][q] = 2u << 30;  // before tile 0: prefix 0
      }
    }
    int u = 0;
#pragma unroll
    for (; u < W; ++u) {
      uint32_t a = w[u][0], o = w[u][0];
#pragma unroll
      for (int q = 1; q < 8; ++q) {
        a &= w[u][q];
        o |= w[u][q];
      }
      // every word of the row an aggregate (flag 01) and every digit still walking
      const bool allA = live == 0xffu && (a >> 30) == 1u && (o >> 31) == 0u;
      if (__all_sync(0xffffffffu, allA)) {
#pragma unroll
        for (int q = 0; q < 8; ++q) raw[q] += w[u][q];
        ++n_raw;
        continue;
      }
      bool ok = true;
#pragma unroll
      for (int q = 0; q < 8; ++q) ok &= !((live >> q) & 1) || (w[u][q] >> 30) != 0u;
      if (!__all_sync(0xffffffffu, ok)) break;  // warp-uniform: re-read from row u
#pragma unroll
      for (int q = 0; q < 8; ++q)
        if ((live >> q) & 1) {
          msk[q] += w[u][q] & 0x3FFFFFFFu;
          if ((w[u][q] >> 30) == 2u) live &= ~(1u << q);
        }
      if (!__any_sync(0xffffffffu, live != 0)) break;
    }
    if (!__any_sync(0xffffffffu, live != 0)) break;
    j -= u;
  }
#pragma unroll
  for (int q = 0; q < 8; ++q) excl[q] = raw[q] - (n_raw << 30) + msk[q];
}

// KV: key/value pairs (S§8(f) #3): the 64-bit value of each key rides along -- second TMA copy
// into a value stage, scattered to the key's stage slot, written out to the key's position.
// DM (dominant-digit elision): 0 none; 1 pass 0 of an elided sort (counts the
// outliers' digit-P histogram); 2 the elided sort's last pass (diverts the outliers).  The host
// picks DM per launch after reading K2's plan, so the DM = 0 kernel carries no elision code.
// DESC: a descending float64 sort (compile-time, so ascending kernels carry no extra work).
// K32: 32-bit keys (float32 / uint32, S§8(f) #4 native path): 4-byte stage and stores, the
// binary32 key transform; keys-only, no elision.
template <int CT, int ITEMS, bool IN_F64, bool KV = false, int DM = 0, bool DESC = false, bool K32 = false>
__global__ void __launch_bounds__(CT + 32, (CT == 256 ? 2 : 1)) k_onesweep_ws(uint64_t* in64, uint64_t* out64, uint64_t* tmp64,
                                                       uint64_t* vin, uint64_t* vout, uint64_t* vtmp,
                                                       uint64_t n, const RadixPlan* __restrict__ plan,
                                                       const uint64_t* __restrict__ bin_base,
                                                       uint64_t* __restrict__ lookback,
                                                       uint32_t* __restrict__ tile_ctr, int p,
                                                       int out_f64, uint64_t lb_half,
                                                       uint64_t lb_rows,
                                                       const uint64_t* __restrict__ hist = nullptr,
                                                       DdeState* __restrict__ dde = nullptr,
                                                       uint64_t* __restrict__ side = nullptr) {
  using KT = std::conditional_t<K32, uint32_t, uint64_t>;  // key word of this pass
  static_assert(!K32 || (!KV && DM == 0), "32-bit keys: keys-only, no elision");
  using L = WsSmem<CT, ITEMS, KV, sizeof(KT)>;
  constexpr int TILE = L::TILE;
  constexpr int CW = L::CW;
  constexpr int THREADS = CT;  // compute threads
  KT* in = (KT*)in64;
  KT* out = (KT*)out64;
  KT* tmp = (KT*)tmp64;
  extern __shared__ __align__(128) unsigned char smem[];
  KT* stage = (KT*)(smem + L::stage_off);
  uint64_t* vstage = (uint64_t*)(smem + L::vstage_off);  // KV only
  uint32_t* whist = (uint32_t*)(smem + L::whist_off);
  int32_t* s_gofs = (int32_t*)(smem + L::gofs_off);
  uint32_t* s_cnt = (uint32_t*)(smem + L::cnt_off);
  uint64_t* bars = (uint64_t*)(smem + L::bar_off);
  uint32_t* s_warp = (uint32_t*)(smem + L::swarp_off);
  uint32_t* s_tile = (uint32_t*)(smem + L::tile_off);
  uint32_t* s_dummy = (uint32_t*)(smem + L::dummy_off);  // leader atomics: non-leaders' targets
  uint64_t* bar_tma = bars;       // [3] stage s holds its tile (TMA done, or "no tile")
  uint64_t* bar_a = bars + 3;     // [2] tile j counted, A published, counts in s_cnt
  uint64_t* bar_g = bars + 5;     // [2] offsets of tile j in s_gofs
  uint64_t* bar_free = bars + 7;  // [3] stage s read out by every compute warp

  const int na = plan->num_active;
  if (p >= na) return;
  const int digit = plan->digit[p];
  const int shift = 8 * digit;
  const KT* __restrict__ src = pick(plan->src[p], in, out, tmp);
  KT* __restrict__ dst = pick(plan->dst[p], in, out, tmp);
  const uint64_t* __restrict__ vsrc = KV ? pick(plan->src[p], vin, vout, vtmp) : nullptr;
  uint64_t* __restrict__ vdst = KV ? pick(plan->dst[p], vin, vout, vtmp) : nullptr;
  const bool use_match = (plan->match_mask >> p) & 1;
  const bool inv = out_f64 && (p == na - 1);
  // dominant-digit elision: pass 0 counts the outliers' digit-P histogram; the last pass diverts
  // the outliers (digit L != v) to the side buffer and ranks the rest by digit P
  static_assert(DM == 0 || !KV, "the elision is keys-only");
  const KT kx = DESC ? (KT)plan->key_xor : (KT)0;  // descending: complement on the first load
  const KT kx_in = p == 0 ? kx : (KT)0;             // ... and before the last inverse store
  constexpr bool dde_here = DM == 2;
  const int sh_l = DM ? 8 * plan->dde_digit : 0;
  const uint32_t v_l = DM ? plan->dde_value : 0u;
  const int sh_p = DM ? 8 * plan->digit[plan->dde_pass] : 0;
  uint32_t* lb32 = (uint32_t*)lookback + (uint64_t)((plan->lb_parity + p) & 1) * lb_half;
  uint32_t* lb32_next = (uint32_t*)lookback + (uint64_t)((plan->lb_parity + p + 1) & 1) * lb_half;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint64_t num_tiles = (n + TILE - 1) / TILE;

  // stage b <- tile t (one thread); a claim past the end completes the phase without a copy
  auto issue = [&](uint32_t t, int b) {
    s_tile[b] = t;
    if (t < num_tiles) {
      const uint64_t base = (uint64_t)t * TILE;
      const uint64_t cnt = (n - base) < (uint64_t)TILE ? (n - base) : (uint64_t)TILE;
      const uint32_t bytes = (uint32_t)(cnt * sizeof(KT)) & ~15u;
      mbar_arrive_expect_tx(&bar_tma[b], KV ? 2 * bytes : bytes);
      if (bytes) {
        bulk_g2s(stage + (size_t)b * TILE, src + base, bytes, &bar_tma[b]);
        if (KV) bulk_g2s(vstage + (size_t)b * TILE, vsrc + base, bytes, &bar_tma[b]);  // KT = u64
      }
    } else {
      mbar_arrive(&bar_tma[b]);
    }
  };
  for (int i = tid; i < CW * (kRadix + 1); i += blockDim.x) whist[i] = 0;
  // s_dummy is never read for a result; zeroed for defined contents.  (Not in the diverting pass:
  // this line changes ptxas's schedule, A/B profiles/r03ap: other passes 4.80 -> 4.75 ms, the
  // diverting pass 5.24 -> 5.42 ms.)
  if (DM != 2 && tid < 32) s_dummy[tid] = 0;
  if (tid == 0) {
    for (int b = 0; b < 3; ++b) {
      mbar_init(&bar_tma[b], 1);
      mbar_init(&bar_free[b], CW);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&bar_a[b], 1);
      mbar_init(&bar_g[b], 1);
    }
    mbar_fence_init();
    for (int b = 0; b < 2; ++b) issue(atomicAdd(&tile_ctr[p], 1u), b);
  }
  __syncthreads();

  if (warp == CW) {
    // ================= look-back warp =================
    // Per tile j: wait for its counts, look back, publish the inclusive prefix, hand the global
    // offsets to the compute warps; then claim tile j+2 and issue its TMA into the stage that
    // tile j-1 used, once every compute warp has written tile j-1 out.
    uint64_t base[8];
    if (dde_here) {
      // bases of the dominant keys: n_less + exclusive scan over digits of hist[P] - hist_out
      uint64_t c[8], tot = 0;
#pragma unroll
      for (int q = 0; q < 8; ++q) {
        const uint32_t* ho = plan->dde_k1 ? dde->hist_k1 : dde->hist_out;
        const int dq = kx ? kRadix - 1 - (lane * 8 + q) : lane * 8 + q;  // K1 counts ascending digits
        c[q] = hist[digit * kRadix + dq] - ho[lane * 8 + q];
        tot += c[q];
      }
      uint64_t incl = tot;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint64_t y = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += y;
      }
      uint64_t run = plan->dde_n_less + incl - tot;
#pragma unroll
      for (int q = 0; q < 8; ++q) {
        base[q] = run;
        run += c[q];
      }
    } else {
#pragma unroll
      for (int q = 0; q < 8; ++q) base[q] = bin_base[digit * kRadix + lane * 8 + q];
    }
#ifdef HSORT_PHASE_TIMING
    unsigned long long t_wait = 0, t_lb = 0, n_lb = 0;
#endif
    for (uint32_t j = 0;; ++j) {
      const uint64_t tile = s_tile[j % 3];  // written by this warp (or thread 0) before
      if (tile >= num_tiles) break;
#ifdef HSORT_PHASE_TIMING
      long long c0 = clock64();
#endif
      mbar_wait(&bar_a[j & 1], (j >> 1) & 1u);
#ifdef HSORT_PHASE_TIMING
      long long c1 = clock64();
      t_wait += c1 - c0;
#endif
      uint32_t cw[8], excl[8];
#pragma unroll
      for (int q = 0; q < 8; ++q) cw[q] = s_cnt[(j & 1) * kRadix + lane * 8 + q];
      if (tile > 0) {
#if HSORT_FAKE == 1
#pragma unroll
        for (int q = 0; q < 8; ++q) excl[q] = 0;
#else
        lookback8<HSORT_WS_W>(lb32, (int64_t)tile, lane, excl);
#endif
#ifdef HSORT_PHASE_TIMING
        t_lb += clock64() - c1;
        ++n_lb;
#endif
        uint32_t pv[8];
#pragma unroll
        for (int q = 0; q < 8; ++q) pv[q] = (2u << 30) | (excl[q] + (cw[q] & 0xFFFFu));
        st_relaxed_v4(&lb32[tile * kRadix + lane * 8], pv);
        st_relaxed_v4(&lb32[tile * kRadix + lane * 8 + 4], pv + 4);
      } else {
#pragma unroll
        for (int q = 0; q < 8; ++q) excl[q] = 0;
      }
      // offset of the digit's run relative to tile-local position 0 (n <= 2^30: fits in int32)
#pragma unroll
      for (int q = 0; q < 8; ++q)
        s_gofs[(j & 1) * kRadix + lane * 8 + q] = (int32_t)(base[q] + excl[q] - (uint64_t)(cw[q] >> 16));
      __syncwarp();
      if (lane == 0) {
        mbar_arrive(&bar_g[j & 1]);
        const int nb = (int)((j + 2) % 3);
        if (j >= 1) mbar_wait(&bar_free[nb], ((j - 1) / 3) & 1u);
        issue(atomicAdd(&tile_ctr[p], 1u), nb);
      }
      __syncwarp();
    }
#ifdef HSORT_PHASE_TIMING
    if (lane == 0) {
      atomicAdd(&g_phase_dbg[214], t_wait);
      atomicAdd(&g_phase_dbg[215], t_lb);
      atomicAdd(&g_phase_dbg[217], n_lb);
    }
#endif
    return;
  }

  // ================= compute warps =================
  const uint32_t lt = lanemask_lt();
  uint32_t j = 0;
  uint64_t prev_tile = 0;
#ifdef HSORT_PHASE_TIMING
  unsigned long long t_g = 0, t_t = 0, t_all = 0, t_rank = 0, t_cnt = 0, t_wo = 0, n_t = 0, t_peers = 0;
  long long c_start = clock64();
#endif
  KT* const dst_t = dst + tid;
  // write-out of the tile of iteration jj from its (digit-ordered) stage buffer: a key at stage
  // position i with digit d goes to dst[s_gofs[d] + i]; then this warp releases the stage
  auto write_out = [&](uint32_t jj, uint64_t tile) {
#ifdef HSORT_PHASE_TIMING
    long long cw0 = clock64();
#endif
    mbar_wait(&bar_g[jj & 1], (jj >> 1) & 1u);
#ifdef HSORT_PHASE_TIMING
    t_g += clock64() - cw0;
#endif
    const int32_t* gofs = s_gofs + (jj & 1) * kRadix;
    const KT* sb = stage + (size_t)(jj % 3) * TILE;
    const uint64_t* vsb = vstage + (size_t)(jj % 3) * TILE;
    const uint64_t rem = n - tile * (uint64_t)TILE;
    int tile_n = rem < (uint64_t)TILE ? (int)rem : TILE;
    if (dde_here) {  // diverted outliers leave the tile: its keys fill stage[0, sum of counts)
      const uint32_t c = s_cnt[(jj & 1) * kRadix + kRadix - 1];
      tile_n = (int)((c >> 16) + (c & 0xFFFFu));
    }
    // BOUNDED: the elision's tiles that lost outliers hold tile_n < TILE keys; the unrolled loop
    // with a bound beats the strided loop used for the ragged last tile
    auto wo_full = [&](auto inv_tag, auto bounded_tag) {
      constexpr bool INV = decltype(inv_tag)::value;
      constexpr bool BOUNDED = decltype(bounded_tag)::value;
#pragma unroll
      for (int q = 0; q < ITEMS; ++q) {
        if (BOUNDED && tid + q * THREADS >= tile_n) break;
        const KT v = sb[tid + q * THREADS];
        const int32_t g = gofs[(uint32_t)(v >> shift) & 255u];
        KT* a = dst_t + g;
#if HSORT_FAKE == 3
        if (v == 0x123456789ull)
#endif
        st_global_w(a + q * THREADS, INV ? from_key_w((KT)(v ^ kx)) : v);
        if (KV) st_global_u64((uint64_t)(vdst + tid + g + q * THREADS), vsb[tid + q * THREADS]);
      }
    };
    if (tile_n == TILE) {  // (elision: tile_n is the count of keys left after the diversion)
      if (inv) wo_full(std::true_type{}, std::false_type{});
      else wo_full(std::false_type{}, std::false_type{});
    } else if (DM == 2 && !KV && rem >= (uint64_t)TILE) {
      if (inv) wo_full(std::true_type{}, std::true_type{});
      else wo_full(std::false_type{}, std::true_type{});
    } else {
      for (int i = tid; i < tile_n; i += THREADS) {
        const KT v = sb[i];
        const int32_t g = gofs[(uint32_t)(v >> shift) & 255u];
        st_global_w(dst + g + i, inv ? from_key_w((KT)(v ^ kx)) : v);
        if (KV) st_global_u64((uint64_t)(vdst + g + i), vsb[i]);
      }
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(&bar_free[jj % 3]);
  };
  // one tile: load from the stage, per-warp digit counts, tile aggregate + scan, warp ranking,
  // scatter into the stage in digit order.  FULL (every tile but the last) drops all bounds logic.
  // DM (compile-time): 0 no elision work, 1 count the outliers' digit-P histogram (pass 0),
  // 2 divert the outliers (the elision's last pass)
  // WO (compile-time): 0 = no write-out here; 1 / 2 = write tile j-1 out (2: with the inverse
  // transform) interleaved with this tile's ranking, so its shared loads and global stores issue
  // beside the ballots (ALU) instead of in a memory-only phase of their own
  auto rank_tile = [&](auto full_tag, auto wo_tag, uint64_t tile, int tile_n, KT* sb, uint64_t* vsb) {
    constexpr bool FULL = decltype(full_tag)::value;
    constexpr int WO = decltype(wo_tag)::value;
    const uint64_t tbase = tile * (uint64_t)TILE;
    const int bulk_n = (int)(((uint32_t)tile_n * (uint32_t)sizeof(KT) & ~15u) / (uint32_t)sizeof(KT));
    const int wofs = warp * 32 * ITEMS + lane;
    uint32_t* wh = whist + warp * (kRadix + 1);  // this warp's row: zero on entry
    KT k[ITEMS];
    uint64_t vv[KV ? ITEMS : 1];
    uint32_t dd[ITEMS];
    uint32_t omask = 0;  // elision: items of this lane that are outliers
#pragma unroll
    for (int i = 0; i < ITEMS; ++i) {
      const int jj = wofs + i * 32;
      KT v;
      if (FULL) v = sb[jj];
      else v = jj < bulk_n ? sb[jj] : (jj < tile_n ? src[tbase + jj] : (KT)0);
      if (KV) {
        if (FULL) vv[i] = vsb[jj];
        else vv[i] = jj < bulk_n ? vsb[jj] : (jj < tile_n ? vsrc[tbase + jj] : 0);
      }
      k[i] = (IN_F64 ? to_key_w(v) : v) ^ kx_in;
      const bool valid = FULL || jj < tile_n;
      dd[i] = valid ? ((uint32_t)(k[i] >> shift) & 255u) : (uint32_t)kRadix;
      if (DM != 0) omask |= (uint32_t)(valid && ((uint32_t)(k[i] >> sh_l) & 255u) != v_l) << i;
    }
    // outliers of the elision (rare; branch-free above): one vote per warp, then the slow path
    bool w_out = false;
    if (DM != 0) {
      w_out = __any_sync(0xffffffffu, omask != 0);
      if (w_out) {
#pragma unroll
        for (int i = 0; i < ITEMS; ++i)
          if ((omask >> i) & 1u) {
            if (DM == 1) atomicAdd(&dde->hist_out[(uint32_t)(k[i] >> sh_p) & 255u], 1u);
            if (DM == 2) {
              side[atomicAdd(&dde->n_out, 1u)] = k[i];
              dd[i] = kRadix;
            }
          }
      }
    }
#pragma unroll
    for (int i = 0; i < ITEMS; ++i) atomicAdd(&wh[dd[i]], 1u);
#ifdef HSORT_PHASE_TIMING
    long long q0 = clock64();
#endif
    bar_compute<CT>();
#ifdef HSORT_PHASE_TIMING
    long long q1 = clock64();
#endif
    uint32_t cnt = 0;
    if (tid < kRadix) {
#pragma unroll
      for (int w = 0; w < CW; ++w) cnt += whist[w * (kRadix + 1) + tid];
      st_relaxed32(&lb32[tile * kRadix + tid], ((tile == 0 ? 2u : 1u) << 30) | cnt);
      lb32_next[tile * kRadix + tid] = 0;  // the next pass's array, row of this tile
    }
    const uint32_t tstart = scan256_excl_c<CT>(cnt, s_warp);
    if (tid < kRadix) {
      uint32_t run = tstart;
#pragma unroll
      for (int w = 0; w < CW; ++w) {
        const uint32_t c = whist[w * (kRadix + 1) + tid];
        whist[w * (kRadix + 1) + tid] = run;
        run += c;
      }
      s_cnt[(j & 1) * kRadix + tid] = cnt | (tstart << 16);
    }
#ifdef HSORT_PHASE_TIMING
    long long q2 = clock64();
#endif
    bar_compute<CT>();
#ifdef HSORT_PHASE_TIMING
    long long q3 = clock64();
    if (lane == 0 && (warp == 0 || warp == CW - 1)) {
      const int o = warp == 0 ? 224 : 228;
      atomicAdd(&g_phase_dbg[o], (unsigned long long)(q1 - q0));      // wait at barrier 1
      atomicAdd(&g_phase_dbg[o + 1], (unsigned long long)(q2 - q1));  // reduce + scan + bases
      atomicAdd(&g_phase_dbg[o + 2], (unsigned long long)(q3 - q2));  // wait at barrier 2
      atomicAdd(&g_phase_dbg[o + 3], 1ull);
    }
#endif
    if (tid == 0) mbar_arrive(&bar_a[j & 1]);
#ifdef HSORT_PHASE_TIMING
    long long cr0 = clock64();
#endif
    const uint32_t jp = j - 1;  // WO: the previous tile (every warp scattered it before barrier 1)
    const int32_t* pgofs = s_gofs + (jp & 1) * kRadix;
    const KT* psb = stage + (size_t)(jp % 3) * TILE;
    const uint64_t* pvsb = vstage + (size_t)(jp % 3) * TILE;
    if (WO) mbar_wait(&bar_g[jp & 1], (jp >> 1) & 1u);
    auto wo_item = [&](int q) {
      if (WO && q < ITEMS) {
        const KT v = psb[tid + q * THREADS];
        const int32_t g = pgofs[(uint32_t)(v >> shift) & 255u];
        st_global_w(dst_t + g + q * THREADS, WO == 2 ? from_key_w((KT)(v ^ kx)) : v);
        if (KV) st_global_u64((uint64_t)(vdst + tid + g + q * THREADS), pvsb[tid + q * THREADS]);
      }
    };

    // rank: peers = lanes of this item with the same digit; the leader's atomic on the warp's
    // base returns the group's first slot.
    uint32_t peers[ITEMS];
    if (use_match) {
#pragma unroll
      for (int i = 0; i < ITEMS; ++i) {
        peers[i] = __match_any_sync(0xffffffffu, dd[i]);
        wo_item(i);
      }
    } else {
      // high-entropy digits: an 8-ballot multisplit (4 instructions per bit: test -> predicate,
      // vote, select, and) for most items; the first NM items use match.any, which runs on another
      // pipe, so both proceed in parallel
      constexpr int NM0 = KV ? HSORT_KV_NMATCH : HSORT_WS_NMATCH;
      constexpr int NM = NM0 < ITEMS ? NM0 : ITEMS;
#pragma unroll
      for (int i = 0; i < NM; ++i) peers[i] = __match_any_sync(0xffffffffu, dd[i]);
#pragma unroll
      for (int i = NM; i < ITEMS; ++i) peers[i] = 0xffffffffu;
#pragma unroll
      for (int b = 0; b < (FULL ? 8 : 9); ++b) {
#pragma unroll
        for (int i = NM; i < ITEMS; ++i) peers[i] = peer_bit(peers[i], dd[i], 1u << b);
        if (b < 8) {
          wo_item(2 * b);
          wo_item(2 * b + 1);
        }
      }
      if (FULL && DM == 2 && w_out) {  // diverted items carry digit 256: separate them (bit 8)
#pragma unroll
        for (int i = NM; i < ITEMS; ++i) peers[i] = peer_bit(peers[i], dd[i], 1u << 8);
      }
#pragma unroll
      for (int q = 16; q < ITEMS; ++q) wo_item(q);
    }
    if (WO) {  // tile j-1 is written out: release its stage to the next TMA
      __syncwarp();
      if (lane == 0) mbar_arrive(&bar_free[jp % 3]);
    }
#if HSORT_FAKE == 2
#pragma unroll
    for (int i = 0; i < ITEMS; ++i) peers[i] = 1u << lane;
#endif
#ifdef HSORT_PHASE_TIMING
    {  // force the peers to be computed before the clock read
      uint32_t x = 0;
#pragma unroll
      for (int i = 0; i < ITEMS; ++i) x ^= peers[i];
      asm volatile("" ::"r"(x));
    }
    t_peers += clock64() - cr0;
#endif
    uint32_t rr[ITEMS];
#pragma unroll
    for (int i = 0; i < ITEMS; ++i) {
      const int leader = 31 - __clz(peers[i]);
      // branch-free: every lane adds; a non-leader to its own word of s_dummy, so large groups
      // (duplicate-heavy data) do not serialise on one address
      if (HSORT_WS_PATOM && FULL && (DM != 2 || HSORT_WS_PATOM_DM2) && (!K32 || HSORT_WS_PATOM_K32))
        rr[i] = atomicAdd(lane == leader ? &wh[dd[i]] : s_dummy + lane, (uint32_t)__popc(peers[i]));
      else
        rr[i] = (lane == leader && ((FULL && (DM != 2 || !w_out)) || dd[i] < kRadix))
                    ? atomicAdd(&wh[dd[i]], (uint32_t)__popc(peers[i]))
                    : 0u;
    }
#pragma unroll
    for (int i = 0; i < ITEMS; ++i) {
      const int leader = 31 - __clz(peers[i]);
      const uint32_t r = __shfl_sync(0xffffffffu, rr[i], leader) + __popc(peers[i] & lt);
      if ((FULL && (DM != 2 || !w_out)) || dd[i] < kRadix) {
        sb[r] = k[i];
        if (KV) vsb[r] = vv[i];
      }
    }
    // the row is private to this warp from here to the next tile's counts: clear it now
    __syncwarp();
    for (int i = lane; i < kRadix + 1; i += 32) wh[i] = 0;
#ifdef HSORT_PHASE_TIMING
    return cr0;
#else
    return 0ll;
#endif
  };
  while (true) {
    const int cb = (int)(j % 3);
#ifdef HSORT_PHASE_TIMING
    long long ct0 = clock64();
#endif
    mbar_wait(&bar_tma[cb], (j / 3) & 1u);
#ifdef HSORT_PHASE_TIMING
    t_t += clock64() - ct0;
    ++n_t;
#endif
    const uint64_t tile = s_tile[cb];
    if (tile >= num_tiles) break;
#ifdef HSORT_PHASE_TIMING
    long long cc0 = clock64();
#endif
    const uint64_t rem = n - tile * (uint64_t)TILE;
    const int tile_n = rem < (uint64_t)TILE ? (int)rem : TILE;
    KT* sb = stage + (size_t)cb * TILE;
    uint64_t* vsb = vstage + (size_t)cb * TILE;
    long long cr0;
    using WO0 = std::integral_constant<int, 0>;
    // interleaved write-out (WO): this tile and the previous one are full (only the last tile is
    // ragged; in the elision's diverting pass a tile that lost outliers is written out separately)
    constexpr bool IL = HSORT_WS_IL && (DM != 2 || HSORT_WS_IL_DM2) && (!K32 || HSORT_WS_IL_K32);
    bool il = IL && j >= 1 && tile_n == TILE;
    if (DM == 2 && il) {  // the elision's diverting pass: only if tile j-1 lost no outliers
      const uint32_t c = s_cnt[((j - 1) & 1) * kRadix + kRadix - 1];
      il = (int)((c >> 16) + (c & 0xFFFFu)) == TILE;
    }
    if (tile_n == TILE) {
      if (IL && il) {
        if (inv) cr0 = rank_tile(std::true_type{}, std::integral_constant<int, IL ? 2 : 0>{}, tile, tile_n, sb, vsb);
        else cr0 = rank_tile(std::true_type{}, std::integral_constant<int, IL ? 1 : 0>{}, tile, tile_n, sb, vsb);
      } else {
        cr0 = rank_tile(std::true_type{}, WO0{}, tile, tile_n, sb, vsb);
      }
    } else {
      cr0 = rank_tile(std::false_type{}, WO0{}, tile, tile_n, sb, vsb);
    }
#ifdef HSORT_PHASE_TIMING
    t_cnt += cr0 - cc0;
    long long cw1 = clock64();
    t_rank += cw1 - cr0;
#else
    (void)cr0;
#endif
    if (j >= 1 && !il) write_out(j - 1, prev_tile);
#ifdef HSORT_PHASE_TIMING
    t_wo += clock64() - cw1;
#endif
    prev_tile = tile;
    ++j;
  }
  // drain the last tile (every warp's scatter of it must be complete: no tile barrier since)
  bar_compute<CT>();
  if (j >= 1) write_out(j - 1, prev_tile);
#ifdef HSORT_PHASE_TIMING
  t_all = clock64() - c_start;
  if (tid == 0) {
    atomicAdd(&g_phase_dbg[210], t_g);
    atomicAdd(&g_phase_dbg[211], t_t);
    atomicAdd(&g_phase_dbg[212], t_all);
    atomicAdd(&g_phase_dbg[213], n_t);
    atomicAdd(&g_phase_dbg[218], t_rank);
    atomicAdd(&g_phase_dbg[219], t_cnt);
    atomicAdd(&g_phase_dbg[220], t_wo);
    atomicAdd(&g_phase_dbg[221], t_peers);
  }
#endif
  if (tid < kRadix)
    for (uint64_t rr = num_tiles + blockIdx.x; rr < lb_rows; rr += gridDim.x)
      lb32_next[rr * kRadix + tid] = 0;
}

template <int CT, int ITEMS, bool KV = false, int DM = 0, bool DESC = false, bool K32 = false>
cudaError_t launch_ws_pass(uint64_t* in, uint64_t* out, uint64_t* tmp, uint64_t* vin, uint64_t* vout,
                           uint64_t* vtmp, uint64_t n, RadixScratch& s, int p, bool first_in_f64,
                           bool out_f64, cudaStream_t st) {
  using L = WsSmem<CT, ITEMS, KV, K32 ? 4 : 8>;
  static int blocks_per_sm[64] = {0};
  int dev = 0;
  cudaGetDevice(&dev);
  constexpr bool dde = DM != 0;
  auto kt = k_onesweep_ws<CT, ITEMS, true, KV, DM, DESC, K32>;
  auto kf = k_onesweep_ws<CT, ITEMS, false, KV, DM, DESC, K32>;
  if (dev < 0 || dev >= 64) return cudaErrorInvalidDevice;
  if (!blocks_per_sm[dev]) {
    cudaError_t e;
    if ((e = cudaFuncSetAttribute(kt, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)L::bytes)) != cudaSuccess) return e;
    if ((e = cudaFuncSetAttribute(kf, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)L::bytes)) != cudaSuccess) return e;
    int b = 0;
    if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, kf, CT + 32, L::bytes)) != cudaSuccess) return e;
    blocks_per_sm[dev] = b > 0 ? b : 1;
  }
  const uint64_t tiles = (n + L::TILE - 1) / L::TILE;
  if (tiles > s.max_tiles) return cudaErrorInvalidValue;
  uint64_t grid = (uint64_t)num_sms(dev) * blocks_per_sm[dev];
  if (grid > tiles) grid = tiles ? tiles : 1;
  const uint64_t* h = dde ? s.hist : nullptr;
  DdeState* ds = dde ? s.dde : nullptr;
  uint64_t* sd = dde ? s.side : nullptr;
  if (first_in_f64)
    kt<<<(unsigned)grid, CT + 32, L::bytes, st>>>(in, out, tmp, vin, vout, vtmp, n, s.plan, s.bin_base,
                                             s.lookback, s.tile_ctr, p, out_f64 ? 1 : 0,
                                             s.max_tiles * kRadix, s.lb_rows, h, ds, sd);
  else
    kf<<<(unsigned)grid, CT + 32, L::bytes, st>>>(in, out, tmp, vin, vout, vtmp, n, s.plan, s.bin_base,
                                             s.lookback, s.tile_ctr, p, out_f64 ? 1 : 0,
                                             s.max_tiles * kRadix, s.lb_rows, h, ds, sd);
  return launched();
}

// Look-back status format of one sort: 2 = 32-bit words (TMA pass, n <= 2^30: an active digit
// has at most n - 1 keys), 1 = 64-bit epoch-tagged words.  Switching formats re-zeroes the array
// so stale words of the other format can never be read as published.
int pass_kernel(uint64_t* in, uint64_t* out, uint64_t* tmp) {
  const bool aligned = !(((uintptr_t)in | (uintptr_t)out | (uintptr_t)(tmp ? tmp : out)) & 15);
  return aligned ? pass_variant() : 0;
}
// 32-bit status words hold flag(2) | count(30).  With n <= 2^30 every prefix a tile actually
// consumes is < 2^30: a reader that owns keys of digit d reads predecessors' prefixes of d, which
// exclude its own keys.  The one value that can reach 2^30 (all n keys in one digit, a forced
// single pass) is only read by tiles without keys of d and decodes as flag 3 = "aggregate", so a
// reader never spins on it.
cudaError_t select_lb_mode(RadixScratch& s, int kernel, uint64_t n, cudaStream_t st, bool kv = false,
                           bool k32 = false) {
  const int mode = (kernel >= 1 && n <= (1ull << 30)) ? 2 : 1;
  if (s.lb_mode != 0 && s.lb_mode != mode) {
    cudaError_t e = cudaMemsetAsync(s.lookback, 0, s.max_tiles * kRadix * sizeof(uint64_t), st);
    if (e != cudaSuccess) return e;
    s.lb_rows = 0;
  }
  s.lb_mode = mode;
  if (mode == 2) {
    const uint64_t tile = kv ? (uint64_t)kKvTile
                             : k32 ? (uint64_t)HSORT_WS_CT * HSORT_K32_ITEMS
                             : (kernel == 2 ? (uint64_t)HSORT_WS_CT * HSORT_WS_ITEMS : (uint64_t)kRadixTile);
    const uint64_t t = (n + tile - 1) / tile;
    if (t > s.lb_rows) s.lb_rows = t;
  }
  return cudaSuccess;
}

cudaError_t launch_pass(RadixScratch& s, uint64_t* in, uint64_t* out, uint64_t* tmp, uint64_t n,
                        int p, bool first_in_f64, bool out_f64, cudaStream_t st, int dm = 0,
                        bool desc = false) {
  uint32_t ep = 0;
  cudaError_t e = next_epoch(s, st, &ep);
  if (e != cudaSuccess) return e;
  // TMA bulk copies need 16-byte aligned tile sources: every buffer the plan may read
  const int v = pass_kernel(in, out, tmp);
  if (v == 2 && s.lb_mode == 2 && desc) {
    constexpr int CT = HSORT_WS_CT, IT = HSORT_WS_ITEMS;
    if (dm == 1)
      return launch_ws_pass<CT, IT, false, 1, true>(in, out, tmp, nullptr, nullptr, nullptr, n, s, p,
                                                    first_in_f64, out_f64, st);
    if (dm == 2)
      return launch_ws_pass<CT, IT, false, 2, true>(in, out, tmp, nullptr, nullptr, nullptr, n, s, p,
                                                    first_in_f64, out_f64, st);
    return launch_ws_pass<CT, IT, false, 0, true>(in, out, tmp, nullptr, nullptr, nullptr, n, s, p,
                                                  first_in_f64, out_f64, st);
  }
  if (v == 2 && s.lb_mode == 2) {
    if (dm == 1)
      return launch_ws_pass<HSORT_WS_CT, HSORT_WS_ITEMS, false, 1>(in, out, tmp, nullptr, nullptr, nullptr,
                                                                   n, s, p, first_in_f64, out_f64, st);
    if (dm == 2)
      return launch_ws_pass<HSORT_WS_CT, HSORT_WS_ITEMS, false, 2>(in, out, tmp, nullptr, nullptr, nullptr,
                                                                   n, s, p, first_in_f64, out_f64, st);
    return launch_ws_pass<HSORT_WS_CT, HSORT_WS_ITEMS>(in, out, tmp, nullptr, nullptr, nullptr, n, s, p,
                                                       first_in_f64, out_f64, st);
  }
  // look-back window 4: measured best of 1..32
  if (v >= 1) {
    if (s.lb_mode == 2)
      return launch_tma_pass<256, 16, 4, 2, true>(in, out, tmp, n, s, ep, p, first_in_f64, out_f64, st);
    return launch_tma_pass<256, 16, 4, 2, false>(in, out, tmp, n, s, ep, p, first_in_f64, out_f64, st);
  }
  uint64_t tiles = (n + kRadixTile - 1) / kRadixTile;
  if (first_in_f64)
    k_onesweep<kPassThreads, kPassItems, true><<<(unsigned)tiles, kPassThreads, 0, st>>>(
        in, out, tmp, n, s.plan, s.bin_base, s.lookback, s.tile_ctr, ep, p, out_f64 ? 1 : 0);
  else
    k_onesweep<kPassThreads, kPassItems, false><<<(unsigned)tiles, kPassThreads, 0, st>>>(
        in, out, tmp, n, s.plan, s.bin_base, s.lookback, s.tile_ctr, ep, p, out_f64 ? 1 : 0);
  return launched();
}

// K1 for 32-bit keys (float32 / uint32): histograms of digits 0..3 (digits 4..7 stay zero, so K2
// sees them trivial).  16 interleaved copies of the 4 x 256 counters (a half-warp's 16 lanes hit 16
// distinct banks), a register run cache per digit (constant high digits cost one atomic per run),
// 16-byte loads of 4 keys.  desc: counts ascending digits (K2 mirrors them, as for float64).
constexpr int kHist32Threads = 1024;
constexpr int kHist32Copies = 16;
// digits 0, 1 (low mantissa bytes: spread for float data) by direct shared atomics; digits 2, 3
// (exponent / sign bytes: few values) through a register run cache
template <bool IN_F32>
__device__ __forceinline__ void hist32_key(uint32_t w, uint32_t* my, uint32_t (&cd)[2],
                                           uint32_t (&cc)[2]) {
  const uint32_t k = IN_F32 ? to_key32(w) : w;
  atomicAdd(&my[(0 * kRadix + (k & 255u)) * kHist32Copies], 1u);
  atomicAdd(&my[(1 * kRadix + ((k >> 8) & 255u)) * kHist32Copies], 1u);
#pragma unroll
  for (int q = 0; q < 2; ++q) {
    const uint32_t d = (k >> (16 + 8 * q)) & 255u;
    if (d == cd[q]) {
      ++cc[q];
    } else {
      if (cc[q]) atomicAdd(&my[((2 + q) * kRadix + cd[q]) * kHist32Copies], cc[q]);
      cd[q] = d;
      cc[q] = 1;
    }
  }
}
template <bool IN_F32>
__global__ void __launch_bounds__(kHist32Threads) k_hist32(const uint32_t* __restrict__ src,
                                                           uint64_t n, uint64_t* __restrict__ hist) {
  extern __shared__ uint32_t sh[];  // [4 * 256][16] (64 KB, dynamic)
  for (int i = threadIdx.x; i < 4 * kRadix * kHist32Copies; i += kHist32Threads) sh[i] = 0;
  __syncthreads();
  uint32_t* my = sh + (threadIdx.x & (kHist32Copies - 1));
  uint32_t cd[2] = {0, 0}, cc[2] = {0, 0};
  const uint64_t head = ((((uintptr_t)src & 15) / 4) ? (4 - ((uintptr_t)src & 15) / 4) : 0);
  const uint64_t h = head < n ? head : n;
  if (blockIdx.x == 0 && threadIdx.x < h) hist32_key<IN_F32>(src[threadIdx.x], my, cd, cc);
  const uint4* b4 = (const uint4*)(src + h);
  const uint64_t m = n - h, quads = m / 4;
  const uint64_t stride = (uint64_t)gridDim.x * kHist32Threads;
  uint64_t i = (uint64_t)blockIdx.x * kHist32Threads + threadIdx.x;
  for (; i + 3 * stride < quads; i += 4 * stride) {  // 4 independent 16-byte loads in flight
    uint4 v[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) v[u] = __ldcs(b4 + i + u * stride);
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      hist32_key<IN_F32>(v[u].x, my, cd, cc);
      hist32_key<IN_F32>(v[u].y, my, cd, cc);
      hist32_key<IN_F32>(v[u].z, my, cd, cc);
      hist32_key<IN_F32>(v[u].w, my, cd, cc);
    }
  }
  for (; i < quads; i += stride) {
    const uint4 v = __ldcs(b4 + i);
    hist32_key<IN_F32>(v.x, my, cd, cc);
    hist32_key<IN_F32>(v.y, my, cd, cc);
    hist32_key<IN_F32>(v.z, my, cd, cc);
    hist32_key<IN_F32>(v.w, my, cd, cc);
  }
  if (blockIdx.x == gridDim.x - 1 && threadIdx.x < (m & 3))
    hist32_key<IN_F32>(src[h + quads * 4 + threadIdx.x], my, cd, cc);
#pragma unroll
  for (int q = 0; q < 2; ++q)
    if (cc[q]) atomicAdd(&my[((2 + q) * kRadix + cd[q]) * kHist32Copies], cc[q]);
  __syncthreads();
  for (int j = threadIdx.x; j < 4 * kRadix; j += kHist32Threads) {
    uint32_t c = 0;
#pragma unroll
    for (int q = 0; q < kHist32Copies; q += 4) {
      const uint4 a = *(const uint4*)&sh[j * kHist32Copies + q];
      c += a.x + a.y + a.z + a.w;
    }
    if (c) atomicAdd((unsigned long long*)&hist[j], (unsigned long long)c);
  }
}

// final copy of a 32-bit sort (odd pass count in place, or every digit trivial): plan flags
// copy_in_f64 / copy_out_f64 mean float32 bits here
__global__ void k_final_copy32(uint32_t* in, uint32_t* out, uint32_t* tmp, uint64_t n,
                               const RadixPlan* __restrict__ plan) {
  const int cs = plan->copy_src;
  if (cs < 0) return;
  const uint32_t* s = pick(cs, in, out, tmp);
  const bool fin = plan->copy_in_f64, fout = plan->copy_out_f64;
  const uint32_t kx = (uint32_t)plan->key_xor;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t v = s[i];
    if (fin != fout) v = fin ? to_key32(v) ^ kx : from_key32(v ^ kx);
    out[i] = v;
  }
}

}  // namespace

#ifdef HSORT_PHASE_TIMING
extern "C" int hsort_debug_phase_counters(unsigned long long* out, int max, int reset) {
  if (max > 256) max = 256;
  cudaMemcpyFromSymbol(out, g_phase_dbg, max * sizeof(unsigned long long));
  if (reset) {
    static unsigned long long z[256] = {0};
    cudaMemcpyToSymbol(g_phase_dbg, z, sizeof(z));
  }
  return (int)cudaGetLastError();
}
#endif

// ------------------------------------------------------------------------------------------
cudaError_t radix_scratch_reserve(RadixScratch& s, uint64_t n) {
  cudaError_t e;
  int dev = 0;
  cudaGetDevice(&dev);
  if (s.small && s.device != dev) return cudaErrorInvalidDevice;
  s.device = dev;
  if (!s.small) {
    // layout (256-byte aligned pieces): hist | plan | tile counters | bin_base
    const size_t hist_b = kDigits * kRadix * sizeof(uint64_t);
    const size_t plan_b = (sizeof(RadixPlan) + 255) & ~(size_t)255;
    const size_t bytes = hist_b + plan_b + 256 + hist_b + 256;
    if ((e = cudaMalloc(&s.small, bytes)) != cudaSuccess) return e;
    char* b = (char*)s.small;
    s.hist = (uint64_t*)b;
    s.plan = (RadixPlan*)(b + hist_b);
    s.tile_ctr = (uint32_t*)(b + hist_b + plan_b);
    s.bin_base = (uint64_t*)(b + hist_b + plan_b + 256);
    s.lb_state = (uint32_t*)(b + hist_b + plan_b + 256 + hist_b);  // not zeroed per sort
    s.small_zero_bytes = (char*)s.bin_base - b;
    if ((e = cudaMemset(s.small, 0, bytes)) != cudaSuccess) return e;
    if ((e = cudaHostAlloc(&s.h_plan, sizeof(RadixPlan), cudaHostAllocDefault)) != cudaSuccess)
      return e;
  }
  // smallest tile of any pass kernel (the TMA fallback pass, or the key/value pass)
  constexpr uint64_t kMinTile = kKvTile < kRadixTile ? kKvTile : kRadixTile;
  uint64_t tiles = (n + kMinTile - 1) / kMinTile;
  if (tiles < 1) tiles = 1;
  if (tiles > s.max_tiles) {
    if (s.lookback) cudaFree(s.lookback);
    s.lookback = nullptr;
    s.max_tiles = 0;
    uint64_t t2 = tiles + tiles / 8;  // headroom for slightly larger later calls
    if ((e = cudaMalloc(&s.lookback, t2 * kRadix * sizeof(uint64_t))) != cudaSuccess) return e;
    if ((e = cudaMemset(s.lookback, 0, t2 * kRadix * sizeof(uint64_t))) != cudaSuccess) return e;
    s.max_tiles = t2;
    s.epoch = 0;
    s.lb_mode = 0;  // freshly zeroed
    s.lb_rows = 0;
  }
  return cudaSuccess;
}

cudaError_t radix_set_timing(RadixScratch& s, bool on) {
  if (on && !s.ev[0])
    for (int i = 0; i < kNumKernelEvents; ++i) {
      cudaError_t e = cudaEventCreate(&s.ev[i]);
      if (e != cudaSuccess) return e;
    }
  s.timing = on;
  return cudaSuccess;
}

int radix_kernel_times(RadixScratch& s, float* ms, int max) {
  if (!s.ev[0]) return 0;
  int m = 0;
  for (int i = 1; i < kNumKernelEvents && m < max; ++i) {
    float t = 0;
    if (cudaEventElapsedTime(&t, s.ev[i - 1], s.ev[i]) != cudaSuccess) {
      cudaGetLastError();
      t = -1;
    }
    ms[m++] = t;
  }
  return m;
}

void radix_scratch_release(RadixScratch& s) {
  for (int i = 0; i < kNumKernelEvents; ++i)
    if (s.ev[i]) cudaEventDestroy(s.ev[i]);
  if (s.lookback) cudaFree(s.lookback);
  if (s.small) cudaFree(s.small);
  if (s.h_plan) cudaFreeHost(s.h_plan);
  if (s.dde) cudaFree(s.dde);
  if (s.side) cudaFree(s.side);
  if (s.sub) {
    radix_scratch_release(*s.sub);
    delete s.sub;
  }
  s = RadixScratch();
}

bool g_dde_enabled = true;  // hsort_set_option("dde", 0) turns the elision off (A/B, tests)
// below this n the outlier sort's fixed cost outweighs a pass (option "dde_min_n"; lowered only
// by the sanitizer runs, tools/sanitize_run.py)
uint64_t g_dde_min_n = 1ull << 22;

// Side buffer capacity for n keys: the outliers a plan may divert (K2 checks n_out <= cap).
uint64_t dde_cap(uint64_t n) {
  uint64_t c = n >> 13;  // U[0,1) keeps ~n 2^-15 keys below the top byte's dominant value
  if (c < (1ull << 12)) c = 1ull << 12;
  if (c > (1ull << 20)) c = 1ull << 20;
  return c;
}

cudaError_t radix_sort_impl(RadixScratch& s, const uint64_t* in_c, uint64_t* out, uint64_t* tmp,
                            uint64_t n, bool in_f64, bool out_f64, cudaStream_t st, bool allow_dde,
                            bool desc = false) {
  if (n == 0) return cudaSuccess;
  cudaError_t e = radix_scratch_reserve(s, n);
  if (e != cudaSuccess) return e;
  uint64_t* in = const_cast<uint64_t*>(in_c);
  auto mark = [&](int i) -> cudaError_t {
    return s.timing ? cudaEventRecord(s.ev[i], st) : cudaSuccess;
  };
  const int kernel = pass_kernel(in, out, tmp);
  if (desc && (kernel != 2 || n > (1ull << 30) || !in_f64 || !out_f64)) return cudaErrorNotSupported;
  // the elision lives in the warp-specialised pass (32-bit look-back words, n <= 2^30); out of
  // place only (in place, 7 of 8 passes would end in the scratch buffer and need a copy)
  const bool dde = allow_dde && g_dde_enabled && kernel == 2 && in != out &&
                   n >= g_dde_min_n && n <= (1ull << 30);
  uint64_t cap = 0;
  if (dde) {
    cap = dde_cap(n);
    if (!s.dde && (e = cudaMalloc(&s.dde, sizeof(DdeState))) != cudaSuccess) return e;
    if (s.side_cap < cap) {
      if (s.side) cudaFree(s.side);
      s.side = nullptr;
      s.side_cap = 0;
      if ((e = cudaMalloc(&s.side, 2 * cap * sizeof(uint64_t))) != cudaSuccess) return e;
      s.side_cap = cap;
    }
    if (!s.sub) s.sub = new RadixScratch();
    if ((e = cudaMemsetAsync(s.dde, 0, sizeof(DdeState), st)) != cudaSuccess) return e;
  }
  if ((e = cudaMemsetAsync(s.small, 0, s.small_zero_bytes, st)) != cudaSuccess) return e;
  if ((e = mark(0)) != cudaSuccess) return e;
  if ((e = launch_hist(s, in, n, in_f64, s.hist, st, dde ? s.dde : nullptr)) != cudaSuccess) return e;
  if ((e = mark(1)) != cudaSuccess) return e;
  if ((e = select_lb_mode(s, kernel, n, st)) != cudaSuccess) return e;
  k_scan_plan<<<1, 256, 0, st>>>(s.hist, s.bin_base, s.plan, n, in == out ? 1 : 0, in_f64 ? 1 : 0,
                                 out_f64 ? 1 : 0, s.lb_state, cap, dde ? s.dde : nullptr,
                                 desc ? 1 : 0);
  if ((e = launched()) != cudaSuccess) return e;
  if ((e = mark(2)) != cudaSuccess) return e;
  int dev = 0;
  cudaGetDevice(&dev);
  if (dde) {
    // the host picks each pass's kernel (elision mode) from K2's plan: one short sync
    if ((e = cudaMemcpyAsync(s.h_plan, s.plan, sizeof(RadixPlan), cudaMemcpyDeviceToHost, st)) != cudaSuccess)
      return e;
    if ((e = cudaStreamSynchronize(st)) != cudaSuccess) return e;
    const RadixPlan P = *s.h_plan;
    if (P.dde) {
      for (int p = 0; p < kDigits; ++p) {
        if (p < P.num_active) {
          const int dm = p == P.dde_pass ? 2 : (p == 0 && !P.dde_k1 ? 1 : 0);
          if ((e = launch_pass(s, in, out, tmp, n, p, p == 0 && in_f64, out_f64, st, dm, desc)) !=
              cudaSuccess)
            return e;
        }
        if ((e = mark(3 + p)) != cudaSuccess) return e;
      }
      k_final_copy<<<num_sms(dev) * 2, 512, 0, st>>>(in, out, tmp, n, s.plan);
      if ((e = launched()) != cudaSuccess) return e;
      // the outliers (internal keys, unordered) -> sorted on their own scratch -> both ends of out
      const uint64_t n_out = P.dde_n_out;
      if ((e = radix_sort_impl(*s.sub, s.side, s.side, s.side + cap, n_out, false, false, st, false)) !=
          cudaSuccess)
        return e;
      if (n_out) {
        k_dde_place<<<num_sms(dev), 256, 0, st>>>(s.side, n_out, P.dde_n_less, out, n, out_f64 ? 1 : 0,
                                                  P.key_xor);
        if ((e = launched()) != cudaSuccess) return e;
      }
      return mark(11);
    }
  }
  for (int p = 0; p < kDigits; ++p) {
    if ((e = launch_pass(s, in, out, tmp, n, p, p == 0 && in_f64, out_f64, st, 0, desc)) != cudaSuccess)
      return e;
    if ((e = mark(3 + p)) != cudaSuccess) return e;
  }
  k_final_copy<<<num_sms(dev) * 2, 512, 0, st>>>(in, out, tmp, n, s.plan);
  if ((e = launched()) != cudaSuccess) return e;
  if ((e = mark(11)) != cudaSuccess) return e;
  return cudaMemcpyAsync(s.h_plan, s.plan, sizeof(RadixPlan), cudaMemcpyDeviceToHost, st);
}

cudaError_t radix_sort(RadixScratch& s, const uint64_t* in_c, uint64_t* out, uint64_t* tmp,
                       uint64_t n, bool in_f64, bool out_f64, cudaStream_t st) {
  return radix_sort_impl(s, in_c, out, tmp, n, in_f64, out_f64, st, true);
}

cudaError_t radix_sort32(RadixScratch& s, const uint32_t* in_c, uint32_t* out, uint32_t* tmp,
                         uint64_t n, bool in_f32, bool out_f32, bool desc, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  uint32_t* in = const_cast<uint32_t*>(in_c);
  if (n > (1ull << 30) || ((((uintptr_t)in) | ((uintptr_t)out) | ((uintptr_t)tmp)) & 15) ||
      pass_variant() != 2 || (desc && (!in_f32 || !out_f32)))
    return cudaErrorNotSupported;  // the caller takes the 64-bit codec path
  cudaError_t e = radix_scratch_reserve(s, n);
  if (e != cudaSuccess) return e;
  auto mark = [&](int i) -> cudaError_t {
    return s.timing ? cudaEventRecord(s.ev[i], st) : cudaSuccess;
  };
  int dev = 0;
  cudaGetDevice(&dev);
  if ((e = cudaMemsetAsync(s.small, 0, s.small_zero_bytes, st)) != cudaSuccess) return e;
  if ((e = mark(0)) != cudaSuccess) return e;
  {
    const uint64_t want = (n / 4 + kHist32Threads * 4 - 1) / (kHist32Threads * 4);
    const uint64_t cap = (uint64_t)num_sms(dev);
    const unsigned grid = (unsigned)(want < 1 ? 1 : (want > cap ? cap : want));
    constexpr int smem = 4 * kRadix * kHist32Copies * 4;
    static bool attr[64] = {false};
    if (dev >= 0 && dev < 64 && !attr[dev]) {
      if ((e = cudaFuncSetAttribute(k_hist32<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem)) != cudaSuccess) return e;
      if ((e = cudaFuncSetAttribute(k_hist32<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem)) != cudaSuccess) return e;
      attr[dev] = true;
    }
    if (in_f32) k_hist32<true><<<grid, kHist32Threads, smem, st>>>(in, n, s.hist);
    else k_hist32<false><<<grid, kHist32Threads, smem, st>>>(in, n, s.hist);
    if ((e = launched()) != cudaSuccess) return e;
  }
  if ((e = mark(1)) != cudaSuccess) return e;
  if ((e = select_lb_mode(s, 2, n, st, false, true)) != cudaSuccess) return e;
  k_scan_plan<<<1, 256, 0, st>>>(s.hist, s.bin_base, s.plan, n, in == out ? 1 : 0, in_f32 ? 1 : 0,
                                 out_f32 ? 1 : 0, s.lb_state, 0, nullptr, desc ? 1 : 0);
  if ((e = launched()) != cudaSuccess) return e;
  if ((e = mark(2)) != cudaSuccess) return e;
  constexpr int CT = HSORT_WS_CT, IT = HSORT_K32_ITEMS;
  for (int p = 0; p < 4; ++p) {  // digits 4..7 of a 32-bit key are always trivial
    uint64_t* i64 = (uint64_t*)in;
    uint64_t* o64 = (uint64_t*)out;
    uint64_t* t64 = (uint64_t*)tmp;
    const bool f = p == 0 && in_f32;
    e = desc ? launch_ws_pass<CT, IT, false, 0, true, true>(i64, o64, t64, nullptr, nullptr, nullptr, n, s,
                                                           p, f, out_f32, st)
             : launch_ws_pass<CT, IT, false, 0, false, true>(i64, o64, t64, nullptr, nullptr, nullptr, n,
                                                            s, p, f, out_f32, st);
    if (e != cudaSuccess) return e;
    if ((e = mark(3 + p)) != cudaSuccess) return e;
  }
  for (int p = 4; p < kDigits; ++p)
    if ((e = mark(3 + p)) != cudaSuccess) return e;
  k_final_copy32<<<num_sms(dev) * 2, 512, 0, st>>>(in, out, tmp, n, s.plan);
  if ((e = launched()) != cudaSuccess) return e;
  if ((e = mark(11)) != cudaSuccess) return e;
  return cudaMemcpyAsync(s.h_plan, s.plan, sizeof(RadixPlan), cudaMemcpyDeviceToHost, st);
}

cudaError_t radix_sort_desc_f64(RadixScratch& s, const uint64_t* in, uint64_t* out, uint64_t* tmp,
                                uint64_t n, cudaStream_t st) {
  if (n < (1ull << 20)) return cudaErrorNotSupported;  // small: the codec path is as fast
  return radix_sort_impl(s, in, out, tmp, n, true, true, st, true, true);
}

// Key/value GPUSort (S§8(f) #3): K1/K2 on the keys as in radix_sort, then every active digit
// pass with the key/value warp-specialised kernel; the values follow the keys' ping-pong.
cudaError_t radix_sort_pairs(RadixScratch& s, const uint64_t* in_c, const uint64_t* vin_c,
                             uint64_t* out, uint64_t* vout, uint64_t* tmp, uint64_t* vtmp, uint64_t n,
                             bool in_f64, bool out_f64, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  if (n > (1ull << 30)) return cudaErrorNotSupported;  // 32-bit look-back words
  uint64_t* in = const_cast<uint64_t*>(in_c);
  uint64_t* vin = const_cast<uint64_t*>(vin_c);
  if ((((uintptr_t)in | (uintptr_t)out | (uintptr_t)tmp | (uintptr_t)vin | (uintptr_t)vout |
        (uintptr_t)vtmp) & 15) != 0)
    return cudaErrorMisalignedAddress;  // TMA bulk copies
  if ((in == out) != (vin == vout)) return cudaErrorInvalidValue;  // one plan serves both
  cudaError_t e = radix_scratch_reserve(s, n);
  if (e != cudaSuccess) return e;
  auto mark = [&](int i) -> cudaError_t {
    return s.timing ? cudaEventRecord(s.ev[i], st) : cudaSuccess;
  };
  if ((e = cudaMemsetAsync(s.small, 0, s.small_zero_bytes, st)) != cudaSuccess) return e;
  if ((e = mark(0)) != cudaSuccess) return e;
  if ((e = launch_hist(s, in, n, in_f64, s.hist, st)) != cudaSuccess) return e;
  if ((e = mark(1)) != cudaSuccess) return e;
  if ((e = select_lb_mode(s, 2, n, st, true)) != cudaSuccess) return e;
  k_scan_plan<<<1, 256, 0, st>>>(s.hist, s.bin_base, s.plan, n, in == out ? 1 : 0, in_f64 ? 1 : 0,
                                 out_f64 ? 1 : 0, s.lb_state);
  if ((e = launched()) != cudaSuccess) return e;
  if ((e = mark(2)) != cudaSuccess) return e;
  for (int p = 0; p < kDigits; ++p) {
    if ((e = launch_ws_pass<kKvCT, kKvItems, true>(in, out, tmp, vin, vout, vtmp, n, s, p,
                                                    p == 0 && in_f64, out_f64, st)) != cudaSuccess)
      return e;
    if ((e = mark(3 + p)) != cudaSuccess) return e;
  }
  int dev = 0;
  cudaGetDevice(&dev);
  k_final_copy<<<num_sms(dev) * 2, 512, 0, st>>>(in, out, tmp, n, s.plan, vin, vout, vtmp);
  if ((e = launched()) != cudaSuccess) return e;
  if ((e = mark(11)) != cudaSuccess) return e;
  return cudaMemcpyAsync(s.h_plan, s.plan, sizeof(RadixPlan), cudaMemcpyDeviceToHost, st);
}

cudaError_t radix_histograms(RadixScratch& s, const uint64_t* in, uint64_t n, bool in_f64,
                             uint64_t* d_hist, cudaStream_t st) {
  cudaError_t e = cudaMemsetAsync(d_hist, 0, kDigits * kRadix * sizeof(uint64_t), st);
  if (e != cudaSuccess || n == 0) return e;
  return launch_hist(s, in, n, in_f64, d_hist, st);
}

cudaError_t radix_one_pass(RadixScratch& s, const uint64_t* src, uint64_t* dst, uint64_t n,
                           int digit, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  cudaError_t e = radix_scratch_reserve(s, n);
  if (e != cudaSuccess) return e;
  uint64_t* in = const_cast<uint64_t*>(src);
  if ((e = cudaMemsetAsync(s.small, 0, s.small_zero_bytes, st)) != cudaSuccess) return e;
  if ((e = launch_hist(s, in, n, false, s.hist, st)) != cudaSuccess) return e;
  if ((e = select_lb_mode(s, pass_kernel(in, dst, nullptr), n, st)) != cudaSuccess) return e;
  k_scan_plan<<<1, 256, 0, st>>>(s.hist, s.bin_base, s.plan, n, 0, 0, 0, nullptr);
  k_force_plan<<<1, 1, 0, st>>>(s.plan, digit, s.lb_state);
  if ((e = launched(2)) != cudaSuccess) return e;
  return launch_pass(s, in, dst, nullptr, n, 0, false, false, st);
}

}  // namespace hsort
