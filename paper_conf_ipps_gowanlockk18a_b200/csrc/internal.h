// internal.h — declarations shared by the library's own translation units (never by oracle/).
#pragma once
#include <cuda_runtime.h>

#include <atomic>
#include <cstdint>

namespace hsort {

// Kernels launched by the library since load (hsort_get_launch_count): every launch site returns
// launched(k) in place of cudaGetLastError() after its k launches.
extern std::atomic<unsigned long long> g_kernel_launches;
inline cudaError_t launched(unsigned k = 1) {
  g_kernel_launches.fetch_add(k, std::memory_order_relaxed);
  return cudaGetLastError();
}

// ---- radix sort (radix.cu) -----------------------------------------------------------------
// Device pass plan written by K2 (k_scan_plan) and read by every K3 launch, so the whole sort is
// stream-ordered with no host round trip (trivial digits are skipped on the device).
// Buffer ids: 0 = in, 1 = out, 2 = tmp.
struct RadixPlan {
  int32_t num_active;   // P_eff: number of non-trivial digits
  int32_t digit[8];     // active digits, ascending (LSD order)
  int32_t src[8];       // buffer id read by pass p
  int32_t dst[8];       // buffer id written by pass p
  int32_t copy_src;     // -1: no final copy; else buffer id copied to out (with conversion)
  int32_t copy_in_f64;  // conversion of the final copy: source is float64 bits
  int32_t copy_out_f64; // conversion of the final copy: destination is float64 bits
  int32_t match_mask;   // bit p: pass p ranks with MATCH.ANY (few distinct digits per warp),
                        // else with the 8-ballot multisplit
  int32_t lb_parity;    // 32-bit look-back mode: status array of pass p is (lb_parity + p) & 1
  // Dominant-digit elision: the top active digit L has one value v held by all but
  // n_out <= cap keys.  Its pass is dropped; pass dde_pass (the new last pass, digit P) diverts the
  // n_out outliers to a side buffer and places the others by digit P alone; the outliers are
  // sorted separately and written to out[0, n_less) and out[n - (n_out - n_less), n).
  int32_t dde;          // 1: active
  int32_t dde_digit;    // L
  uint32_t dde_value;   // v
  int32_t dde_pass;     // index of the diverting pass (num_active - 1)
  uint64_t dde_n_out;   // outliers (n - count of v)
  uint64_t dde_n_less;  // outliers whose digit L is below v
  int32_t dde_k1;       // 1: K1 already counted the outliers' digit-P histogram (L = 7, P = 6)
  // Descending float64 (S§8(f) #4), fused: the passes sort key(u) ^ key_xor (~0 descending, 0
  // ascending); the first pass applies it on load, the last pass removes it on the inverse store.
  // K1 counts ascending digits; K2 reads digit value v at 255 - v when descending.
  uint64_t key_xor;
};

// Device state of the dominant-digit elision, zeroed per sort.
struct DdeState {
  uint32_t n_out;           // outliers diverted so far (append counter of the side buffer)
  uint32_t guess;           // K1: top digit of the first key (the dominant value's guess)
  uint32_t hist_out[256];   // digit-P histogram of the outliers, counted by pass 0
  uint32_t hist_k1[256];    // K1's count: digit 6 of the keys whose top digit != guess (used when
                            // the plan's dde_k1 says the guess was v, L = 7 and P = 6)
};

struct RadixScratch {
  // small block (one allocation, zeroed per sort): hist[8*256] | bin_base[8*256] | plan |
  // tile counters[8]
  void* small = nullptr;
  uint64_t* hist = nullptr;
  uint64_t* bin_base = nullptr;
  RadixPlan* plan = nullptr;
  uint32_t* tile_ctr = nullptr;
  size_t small_zero_bytes = 0;  // bytes of `small` zeroed per sort (hist + plan + counters)
  // decoupled look-back status words, [max_tiles][256] uint64 (flag | epoch | count)
  uint64_t* lookback = nullptr;
  uint64_t max_tiles = 0;
  uint32_t epoch = 0;
  uint32_t* lb_state = nullptr;  // device word: running count of 32-bit-mode passes (parity)
  int lb_mode = 0;               // 0 unused/zeroed, 1 64-bit epoch words, 2 32-bit words
  uint64_t lb_rows = 0;          // 32-bit mode: rows possibly used since the last full clear
  int device = -1;
  // host-pinned mirror of the plan, read back for statistics
  RadixPlan* h_plan = nullptr;
  // optional per-kernel CUDA events (hsort_set_option("kernel_timing", 1)):
  // ev[0] before K1, ev[1] after K1, ev[2] after K2, ev[3+p] after pass p, ev[11] after copy
  bool timing = false;
  cudaEvent_t ev[12] = {};
  // dominant-digit elision: state + side buffer (2 x side_cap keys: outliers and sort scratch)
  DdeState* dde = nullptr;
  uint64_t* side = nullptr;
  uint64_t side_cap = 0;
  RadixScratch* sub = nullptr;  // scratch of the outlier sort (its own look-back rows and plan)
};
constexpr int kNumKernelEvents = 12;

constexpr int kRadixTile = 4096;  // keys per onesweep tile (THREADS x ITEMS), see radix.cu
#ifndef HSORT_KV_CT
#define HSORT_KV_CT 320    // key/value pass: compute threads (10 warps) ...
#endif
#ifndef HSORT_KV_ITEMS
#define HSORT_KV_ITEMS 13  // ... x pairs per thread: 4160-pair tiles, 3 stages of keys + values = 200 KB
#endif                     // (A/B over 10 shapes: 576x7 80.4 ms, 320x13 71.3 ms per 2^30 pairs)
constexpr int kKvTile = HSORT_KV_CT * HSORT_KV_ITEMS;  // pairs per key/value onesweep tile

// dominant-digit elision on/off (option "dde", default on)
extern bool g_dde_enabled;
extern uint64_t g_dde_min_n;
cudaError_t radix_scratch_reserve(RadixScratch& s, uint64_t n);
cudaError_t radix_set_timing(RadixScratch& s, bool on);
// durations (ms) of [K1, K2, pass0..pass7, final copy] of the last timed sort; returns count
int radix_kernel_times(RadixScratch& s, float* ms, int max);
void radix_scratch_release(RadixScratch& s);

// GPUSort of n keys: out = sorted(in).  tmp: n-element scratch (must differ from in and out).
// in == out allowed.  in_f64: input holds float64 bits (key transform fused into the first
// pass).  out_f64: store float64 bits (inverse transform fused into the last pass).
cudaError_t radix_sort(RadixScratch& s, const uint64_t* in, uint64_t* out, uint64_t* tmp,
                       uint64_t n, bool in_f64, bool out_f64, cudaStream_t st);
// Descending float64 GPUSort with the reverse transform fused into the first and last pass
// (warp-specialised pass only: 16-byte aligned buffers, 2^20 <= n <= 2^30; returns
// cudaErrorNotSupported otherwise, and the caller takes the codec path).
cudaError_t radix_sort_desc_f64(RadixScratch& s, const uint64_t* in, uint64_t* out, uint64_t* tmp,
                                uint64_t n, cudaStream_t st);
// Native 32-bit GPUSort (S§8(f) #4): out = sorted(in) over 32-bit keys (float32 bits under IEEE
// totalOrder when in_f32/out_f32, descending when desc; else uint32 ascending); K1 for 4 digits,
// up to 4 warp-specialised passes with 4-byte keys.  Needs 16-byte aligned buffers, n <= 2^30,
// tmp an n-element scratch; returns cudaErrorNotSupported otherwise (caller: codec path).
cudaError_t radix_sort32(RadixScratch& s, const uint32_t* in, uint32_t* out, uint32_t* tmp,
                         uint64_t n, bool in_f32, bool out_f32, bool desc, cudaStream_t st);
// Key/value GPUSort (S§8(f) #3): (out, vout) = (in, vin) stably sorted by key; n <= 2^30, every
// buffer 16-byte aligned, tmp/vtmp n-element scratch; in == out iff vin == vout.  The values are
// opaque 64-bit payloads (e.g. indices: argsort).
cudaError_t radix_sort_pairs(RadixScratch& s, const uint64_t* in, const uint64_t* vin, uint64_t* out,
                             uint64_t* vout, uint64_t* tmp, uint64_t* vtmp, uint64_t n, bool in_f64,
                             bool out_f64, cudaStream_t st);
// K1 only (hist zeroed first); d_hist receives 8*256 counts.
cudaError_t radix_histograms(RadixScratch& s, const uint64_t* in, uint64_t n, bool in_f64,
                             uint64_t* d_hist, cudaStream_t st);
// K1 + K2 + one K3 pass by `digit` over raw uint64 keys, src -> dst.
cudaError_t radix_one_pass(RadixScratch& s, const uint64_t* src, uint64_t* dst, uint64_t n,
                           int digit, cudaStream_t st);

// ---- GPU merge (merge.cu) ------------------------------------------------------------------
#ifndef HSORT_MERGE_TILE
#define HSORT_MERGE_TILE 4096
#endif
constexpr int kMergeTile = HSORT_MERGE_TILE;  // output keys per merge CTA
constexpr int kMaxMergeRuns = 1024;

// Runs of a merge: run j has len_j = d_off[j + 1] - d_off[j] keys (device offsets) and starts at
// keys + d_off[j] (runs back to back in one buffer) or, when rp != nullptr, at rp[j] (a device
// table of run pointers: the runs may live anywhere, including other GPUs' HBM read over
// NVLink with peer access enabled -- the multi-GPU merge).
//
// K4: ranks[b*k + j] for b in [0, n_bounds): co-ranks of o = min((bound_begin + b)*step, total).
// scratch: merge_corank_scratch_elems(...) uint64 of device scratch for the coarse level of the
// two-level search (nullptr / too small: single level).
uint64_t merge_corank_scratch_elems(int k, uint64_t total, uint64_t step, uint64_t bound_begin,
                                    uint64_t n_bounds);
cudaError_t merge_corank(const uint64_t* keys, const uint64_t* const* rp, const uint64_t* d_off,
                         int k, uint64_t total, uint64_t step, uint64_t bound_begin,
                         uint64_t n_bounds, uint64_t* ranks, uint64_t* scratch,
                         uint64_t scratch_elems, cudaStream_t st);
// K5: merge tiles [tile_begin, tile_begin + tile_count) (tile t = output [t*kMergeTile, ...)),
// given co-ranks of boundaries t = rank_tile0, rank_tile0 + 1, ... (row t - rank_tile0 of
// `ranks`, step kMergeTile); writes out[o - out_origin].
// With vout != nullptr the runs carry 64-bit values (vkeys + d_off[j] or vrp[j], same offsets),
// moved with their keys into vout (key/value merge: stable given stably sorted runs).
cudaError_t merge_tiles(const uint64_t* keys, const uint64_t* const* rp, const uint64_t* d_off,
                        int k, uint64_t total, const uint64_t* ranks, uint64_t rank_tile0,
                        uint64_t tile_begin, uint64_t tile_count, uint64_t* out,
                        uint64_t out_origin, bool out_f64, cudaStream_t st,
                        const uint64_t* vkeys = nullptr, const uint64_t* const* vrp = nullptr,
                        uint64_t* vout = nullptr);

// ---- MSD-first split (msd.cu, S§8(f) #2) ---------------------------------------------------------
constexpr int kMaxBuckets = 1024;
// bucket r of a key k = #{splitters < k} (R - 1 sorted splitters): bucket r = (s_{r-1}, s_r].
// counts: bucket_count_elems(n, R) uint32 of scratch; totals[R] receives the batch's bucket sizes;
// out (n keys, transformed if in_f64) holds the batch in bucket order (bucket r at
// sum_{r' < r} totals[r']).  Stream-ordered.
uint64_t bucket_count_elems(uint64_t n, int R);
cudaError_t bucket_partition(const uint64_t* in, uint64_t n, bool in_f64, const uint64_t* d_spl,
                             int R, uint32_t* counts, uint32_t* totals, uint64_t* out,
                             cudaStream_t st);
// dst[seg.dst_off + i] = seg.src[i] for every segment (sources anywhere, incl. peer HBM).
struct GatherSeg {
  const uint64_t* src;
  uint64_t len;
  uint64_t dst_off;
};
uint64_t gather_pieces(uint64_t len);  // CTAs one segment of len keys needs
// d_piece_start[s] = sum_{s' < s} gather_pieces(len_s'); pieces = the total
cudaError_t gather_segments(const GatherSeg* d_segs, const uint64_t* d_piece_start, int nseg,
                            uint64_t pieces, uint64_t* dst, cudaStream_t st);

// ---- key codecs (codec.cu, S§8(f) #4) ---------------------------------------------------------
constexpr int kKeyF64 = 0;
constexpr int kKeyF32 = 1;
// in (n float64 or float32 bits) -> out (n internal uint64 keys, ascending = the requested
// order); 16-byte aligned buffers.  decode is the inverse.
cudaError_t key_encode(const void* in, uint64_t* out, uint64_t n, int key_type, bool desc,
                       cudaStream_t st);
cudaError_t key_decode(const uint64_t* in, void* out, uint64_t n, int key_type, bool desc,
                       cudaStream_t st);

// out[i] = #keys <= values[i] in the sorted run keys[0, n) (device pointers).
cudaError_t upper_bounds(const uint64_t* keys, uint64_t n, const uint64_t* values, uint64_t m,
                         uint64_t* out, cudaStream_t st);

}  // namespace hsort
