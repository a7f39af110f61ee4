// api.cpp — the C ABI (include/hsort.h), planner (A1), staging ring (A2/A8), stream pipeline
// (A3/A7/A9) and the three sort modes, for the B200-native heterogeneous sort.
//
// Paper workflows (§III-D):
//   BLINE       A -> HtoD -> GPUSort -> DtoH -> B
//   BLINEMULTI  A -> HtoD -> GPUSort -> DtoH -> W -> Merge -> B, blocking
//   PIPEDATA    A -> Stage -> HtoD -> GPUSort -> DtoH -> Stage -> W -> Merge -> B on n_s streams
//               with pinned buffers of p_s elements
//   PARMEMCPY   the Stage MCpy done by several host threads
// B200 design: per GPU an uploader thread (Stage+HtoD, then the sort is enqueued on
// the compute stream) and a downloader thread (DtoH+Stage into W), so HtoD, GPUSort and DtoH of
// consecutive batches overlap on three streams; pinned inputs/outputs skip the staging copy; when
// all runs fit in HBM they stay resident and are merged by the GPU (merge.cu) with the merged
// chunks' DtoH overlapped with the merge.
#include <cuda_runtime.h>
#include <nvtx3/nvToolsExt.h>  // header-only NVTX v3: no-ops unless a profiler attaches
#include <sys/mman.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <condition_variable>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <deque>
#include <map>
#include <mutex>
#include <stdexcept>
#include <string>
#include <thread>
#include <vector>

#include "../../include/hsort.h"
#include "internal.h"
#include "pool.h"

namespace hsort {
void host_corank(const uint64_t* keys, const uint64_t* off, int k, uint64_t o, uint64_t* ranks);
void host_merge(const uint64_t* keys, const uint64_t* off, int k, uint64_t* out, bool out_f64,
                int threads);
void host_merge_range(const uint64_t* keys, const uint64_t* off, int k, uint64_t o_lo,
                      uint64_t o_hi, uint64_t* out, bool out_f64, int threads);
void host_corank_runs(const uint64_t* const* run, const uint64_t* len, int k, uint64_t o,
                      uint64_t* ranks);
void host_merge_runs_range(const uint64_t* const* run, const uint64_t* len, int k, uint64_t o_lo,
                           uint64_t o_hi, uint64_t* out, bool out_f64, int threads,
                           ThreadPool* pool);
}  // namespace hsort

using namespace hsort;

std::atomic<unsigned long long> hsort::g_kernel_launches{0};

namespace {

using Clock = std::chrono::steady_clock;
inline double secs_since(Clock::time_point t0) {
  return std::chrono::duration<double>(Clock::now() - t0).count();
}

thread_local std::string g_err = "";

// NVTX range over a scope (the Fig. 2-style overlap timeline of Stage / HtoD / GPUSort /
// DtoH / Merge under nsys or ncu --nvtx)
struct Nvtx {
  explicit Nvtx(const char* name) { nvtxRangePushA(name); }
  ~Nvtx() { nvtxRangePop(); }
  Nvtx(const Nvtx&) = delete;
  Nvtx& operator=(const Nvtx&) = delete;
};

struct HsortError : std::runtime_error {
  int code;
  HsortError(int c, const std::string& m) : std::runtime_error(m), code(c) {}
};

#define CK(expr)                                                                              \
  do {                                                                                        \
    cudaError_t _e = (expr);                                                                  \
    if (_e != cudaSuccess) {                                                                  \
      throw HsortError(_e == cudaErrorMemoryAllocation ? HSORT_ERR_DEVICE_OOM : HSORT_ERR_CUDA, \
                       std::string(#expr) + ": " + cudaGetErrorString(_e));                  \
    }                                                                                         \
  } while (0)

struct DevBuf {
  void* p = nullptr;
  size_t cap = 0;
  void reserve(size_t bytes) {
    if (bytes <= cap) return;
    if (p) cudaFree(p);
    p = nullptr;
    cap = 0;
    if (bytes == 0) return;
    cudaError_t e = cudaMalloc(&p, bytes);
    if (e != cudaSuccess) {
      cudaGetLastError();
      p = nullptr;
      throw HsortError(HSORT_ERR_DEVICE_OOM, "cudaMalloc(" + std::to_string(bytes) + ") failed: " +
                                                 cudaGetErrorString(e));
    }
    cap = bytes;
  }
  void release() {
    if (p) cudaFree(p);
    p = nullptr;
    cap = 0;
  }
  uint64_t* u64() const { return (uint64_t*)p; }
};

struct Options {
  std::map<std::string, int64_t> v = {
      {"n_s", 3},                    // device batch slots per GPU (default 3, see DESIGN)
      {"p_s", 64ll << 20},           // pinned staging chunk bytes (reading A-6)
      {"n_ring", 3},                 // pinned chunks per direction per GPU
      {"memcpy_threads", 0},         // PARMEMCPY threads (0 = all host threads; 1 = serial MCpy)
      {"merge_threads", 0},          // CPU merge threads (0 = all)
      {"resident", -1},              // -1 auto, 0 force STREAM, 1 force RESIDENT
      {"merge_gpu_permille", -1},    // A12 share f (per mille) of merge output on GPUs; -1 auto
      {"pipeline", 1},               // 1 PIPEDATA overlap, 0 blocking BLINEMULTI ablation
      {"pipemerge", 0},              // STREAM: 1 = pair-wise merges during the sort phase (PIPEMERGE)
      {"pipemerge_threads", 0},      // threads for those merges (0 = half the hardware threads)
      {"merge_chunk", 1ll << 26},    // GPU merge output chunk (keys)
      {"device_reserve_mb", 2048},   // HBM kept free for the runtime / other tenants
      {"kernel_timing", 0},          // 1: CUDA events around every radix kernel (bench roofline)
      {"defer_out_drain", 1},        // STREAM GPU merge share: staged DtoH copy-outs drained lazily
      {"dde", 1},                    // 1: dominant-digit elision in the GPUSort
      {"dde_min_n", 1ll << 22},      // smallest n the elision is tried at
      {"memcpy_nt", 1},              // PARMEMCPY staging copies with non-temporal stores
      {"auto_pipeline_min", 1ll << 24},  // auto plan: pipelined RESIDENT schedule from this n (0 = off)
      {"pin_w", -1},                 // STREAM W: 1 page-locked, 0 pageable, -1 locked if <= pin_w_max_mb
      {"pin_w_max_mb", 1ll << 20},   // auto page-locking limit of W (MB)
      {"w_cache", 1},                // keep W (allocated, prefaulted, locked) across calls
      {"merge_stage_threads", 8},    // STREAM merge: host threads per GPU reserved for staging the
                                     // GPU share's DtoH into a pageable B

      {"virtual_gpus", 0},           // > 0 (set before hsort_init): that many GPU contexts mapped
                                     // round-robin onto the visible devices (multi-GPU scheduler,
                                     // exchange and merge testable on one GPU)
      {"msd", 0},                    // 1: RESIDENT plans run the MSD-first split (S§8(f) #2):
                                     // splitter partition per batch, bucket gather (peer loads),
                                     // one LSD sort per bucket, no merge
      {"msd_bucket_keys", 1ll << 24},  // target bucket size (keys) of the MSD-first split
      {"register_host", 0},          // 1: page-lock pageable A/B for the call (cudaHostRegister) and
                                     // DMA them directly instead of staging through the ring
  };
  int64_t get(const char* k) const { return v.at(k); }
};

struct GpuCtx {
  int dev = -1;
  cudaStream_t s_h2d = nullptr, s_comp = nullptr, s_d2h = nullptr;
  RadixScratch rs;
  DevBuf runs, alt, mout, min, ranks, off;
  DevBuf coarse;       // K4's coarse-level co-rank table (two-level search)
  DevBuf rptr;         // multi-GPU merge: device table of run pointers (peer HBM)
  DevBuf part, bcnt, btot, bspl, bseg;  // MSD-first split: partitioned batches, tile counts,
                                        // batch bucket totals, splitters, gather segment table
  DevBuf vruns, valt;  // key/value sorts: values and their ping-pong scratch
  DevBuf vmout, vrptr; // key/value merge: merged value chunks, value run-pointer table
  DevBuf tmp3;         // typed sorts: third key buffer, so the GPUSort runs out of place (elision)
  std::vector<char*> ring_in, ring_out;
  uint64_t ring_bytes = 0;
  std::vector<cudaEvent_t> ev_in, ev_out;
  uint64_t in_next = 0;
  // staged downloads: out-ring slots whose DMA is enqueued but whose copy-out into the host
  // destination is still pending (dst, bytes); with defer_out set, download() returns without
  // draining them, so the next download's DMAs keep the link busy (flush_out drains the rest)
  uint64_t out_next = 0;
  std::vector<std::pair<char*, uint64_t>> out_pend;
  bool defer_out = false;
};

struct State {
  std::mutex m;
  bool inited = false;
  bool poisoned = false;
  std::vector<GpuCtx> gpus;
  Options opt;
  double t_init = 0;
  // pinned working memory W (STREAM mode), allocated once and reused: pinning is expensive
  // so it is cached like the staging ring
  void* w_base = nullptr;       // mmap'd, prefaulted; page-locked (cudaHostRegister) if w_pinned
  size_t w_bytes = 0;
  bool w_pinned = false;
  double r_cpu_merge = 0;  // last measured CPU merge rate (keys/s), for the A12 split
  bool peer_ok = true;     // every pair of devices in use can read each other's HBM
  // plan of the last call, reused by an identical call (same n, b_s, n_GPU, options): the HBM
  // query behind the plan (cudaMemGetInfo) measured 0.1-62 ms on the B200 box
  // (profiles/r02l_setup.txt), which made repeated calls jitter by tens of ms
  uint64_t opt_version = 0;
  struct PlanCache {
    bool valid = false;
    uint64_t n = 0, b = 0;
    int ng = -1;
    uint64_t opt = 0;
    hsort_plan_t plan{};
  };
  PlanCache pc[65];  // [0]: calls over GPUs [0, n_gpus); [1 + l]: calls on lane l
  // concurrency: a regular call owns every GPU context; lane calls (hsort_sort_lane) own one
  // context each and may run concurrently on different lanes
  std::mutex busy_m;
  bool global_busy = false;
  int lanes_active = 0;
  bool lane_busy[64] = {};
  int n_physical = 0;      // visible CUDA devices
};
State& S() {
  static State s;
  return s;
}

// stats of the calling thread's last successful sort (lanes sort concurrently)
thread_local hsort_stats t_last{};

struct BusyGuard {
  bool ok = false;
  int lane;
  explicit BusyGuard(int l = -1) : lane(l) {
    std::lock_guard<std::mutex> g(S().busy_m);
    if (lane < 0) {
      ok = !S().global_busy && S().lanes_active == 0;
      if (ok) S().global_busy = true;
    } else {
      ok = !S().global_busy && !S().lane_busy[lane];
      if (ok) {
        S().lane_busy[lane] = true;
        ++S().lanes_active;
      }
    }
  }
  ~BusyGuard() {
    if (!ok) return;
    std::lock_guard<std::mutex> g(S().busy_m);
    if (lane < 0) {
      S().global_busy = false;
    } else {
      S().lane_busy[lane] = false;
      --S().lanes_active;
    }
  }
};

template <class F>
int guarded(F f) {
  try {
    return f();
  } catch (const HsortError& e) {
    g_err = e.what();
    if (e.code == HSORT_ERR_CUDA) S().poisoned = true;
    return e.code;
  } catch (const std::bad_alloc&) {
    g_err = "host allocation failed";
    return HSORT_ERR_HOST_OOM;
  } catch (const std::exception& e) {
    g_err = e.what();
    return HSORT_ERR_INTERNAL;
  } catch (...) {
    g_err = "unknown exception";
    return HSORT_ERR_INTERNAL;
  }
}

bool is_pinned(const void* p, uint64_t bytes) {
  if (!p || bytes == 0) return false;
  auto one = [](const void* q) {
    cudaPointerAttributes a;
    cudaError_t e = cudaPointerGetAttributes(&a, q);
    if (e != cudaSuccess) {
      cudaGetLastError();
      return false;
    }
    return a.type == cudaMemoryTypeHost;
  };
  return one(p) && one((const char*)p + bytes - 1);
}

// ---- working memory W (STREAM mode) ------------------------------------------------------------
// W holds the sorted runs between the sort phase and the merge.  Allocating
// and pinning host memory is expensive (cudaHostAlloc ran at ~2.3 GB/s on the B200
// box, profiles/r02a_host_probe.jsonl), so W is allocated once and cached like the staging ring:
// an anonymous mapping (transparent huge pages), prefaulted by all host threads in parallel,
// then page-locked with cudaHostRegister (~46 GB/s on prefaulted pages) so the runs are DMA'd
// straight into W and the GPU merge share streams straight out of it.  t_host_alloc reports the
// cost in the call that paid it.
void release_w() {
  if (!S().w_base) return;
  if (S().w_pinned) {
    cudaHostUnregister(S().w_base);
    cudaGetLastError();
  }
  munmap(S().w_base, S().w_bytes);
  S().w_base = nullptr;
  S().w_bytes = 0;
  S().w_pinned = false;
}

uint64_t* acquire_w(uint64_t bytes, bool* direct, double* t_alloc) {
  Nvtx nv("W alloc");
  const int64_t pin_w = S().opt.get("pin_w");
  const bool want_pin = pin_w == 1 ||
                        (pin_w == -1 && bytes <= ((uint64_t)S().opt.get("pin_w_max_mb") << 20));
  auto ta = Clock::now();
  if (S().w_base && S().w_bytes < bytes) release_w();
  if (!S().w_base) {
    void* p = mmap(nullptr, bytes, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
    if (p == MAP_FAILED) throw HsortError(HSORT_ERR_HOST_OOM, "mmap W failed");
    madvise(p, bytes, MADV_HUGEPAGE);
    const uint64_t chunk = 64ull << 20;
    host_pool().parallel_for((int64_t)((bytes + chunk - 1) / chunk), host_threads(), [&](int64_t i) {
      volatile char* q = (volatile char*)p + (uint64_t)i * chunk;
      const uint64_t len = std::min(chunk, bytes - (uint64_t)i * chunk);
      for (uint64_t o = 0; o < len; o += 4096) q[o] = 0;  // first touch: fault the page in
    });
    S().w_base = p;
    S().w_bytes = bytes;
    S().w_pinned = false;
  }
  if (want_pin && !S().w_pinned) {
    if (cudaHostRegister(S().w_base, S().w_bytes, cudaHostRegisterDefault) == cudaSuccess)
      S().w_pinned = true;
    else
      cudaGetLastError();  // not lockable (limits): W stays pageable and is staged
  } else if (!want_pin && S().w_pinned) {
    cudaHostUnregister(S().w_base);
    cudaGetLastError();
    S().w_pinned = false;
  }
  *t_alloc += secs_since(ta);
  *direct = S().w_pinned;
  return (uint64_t*)S().w_base;
}

// ---- staging ring (A2/A3, A7/A8) -------------------------------------------------------------
struct Acc {  // per-thread stage accumulators
  double t_stage = 0;
  uint64_t h2d = 0, d2h = 0;
};

// Host -> device, through the pinned ring (PIPEDATA Stage + PARMEMCPY) unless direct.
void upload(GpuCtx& g, void* d_dst, const void* h_src, uint64_t bytes, cudaStream_t st, bool direct,
            int threads, Acc& acc) {
  Nvtx r(direct ? "HtoD" : "Stage+HtoD");
  acc.h2d += bytes;
  if (bytes == 0) return;
  if (direct) {
    CK(cudaMemcpyAsync(d_dst, h_src, bytes, cudaMemcpyHostToDevice, st));
    return;
  }
  const uint64_t R = g.ring_in.size(), C = g.ring_bytes;
  for (uint64_t o = 0; o < bytes; o += C) {
    uint64_t len = std::min(C, bytes - o);
    uint64_t s = g.in_next++ % R;
    CK(cudaEventSynchronize(g.ev_in[s]));
    auto t0 = Clock::now();
    par_memcpy(g.ring_in[s], (const char*)h_src + o, len, threads);
    acc.t_stage += secs_since(t0);
    CK(cudaMemcpyAsync((char*)d_dst + o, g.ring_in[s], len, cudaMemcpyHostToDevice, st));
    CK(cudaEventRecord(g.ev_in[s], st));
  }
}

// Staged downloads: copy the out-ring slot s (DMA complete) into its pending host destination.
void drain_out(GpuCtx& g, uint64_t s, int threads, Acc& acc) {
  CK(cudaEventSynchronize(g.ev_out[s]));
  auto t0 = Clock::now();
  par_memcpy(g.out_pend[s].first, g.ring_out[s], g.out_pend[s].second, threads);
  acc.t_stage += secs_since(t0);
  g.out_pend[s] = {nullptr, 0};
}
// ... every pending slot, oldest first
void flush_out(GpuCtx& g, int threads, Acc& acc) {
  const uint64_t R = g.out_pend.size();
  for (uint64_t i = 0; i < R; ++i) {
    const uint64_t s = (g.out_next + i) % R;
    if (g.out_pend[s].first) drain_out(g, s, threads, acc);
  }
}
// Device -> host.  Direct: enqueued only (caller synchronises st).  Staged: returns when every
// byte is in h_dst (DMA of chunk c overlaps the host copy-out of chunk c-1), unless g.defer_out:
// then the last ring slots stay pending until a later download needs them or flush_out.
void download(GpuCtx& g, void* h_dst, const void* d_src, uint64_t bytes, cudaStream_t st,
              bool direct, int threads, Acc& acc) {
  Nvtx r(direct ? "DtoH" : "DtoH+Stage");
  acc.d2h += bytes;
  if (bytes == 0) return;
  if (direct) {
    CK(cudaMemcpyAsync(h_dst, d_src, bytes, cudaMemcpyDeviceToHost, st));
    return;
  }
  const uint64_t R = g.ring_out.size(), C = g.ring_bytes;
  if (g.out_pend.size() != R) g.out_pend.assign(R, {nullptr, 0});
  for (uint64_t o = 0; o < bytes; o += C) {
    const uint64_t len = std::min(C, bytes - o);
    const uint64_t s = g.out_next++ % R;
    if (g.out_pend[s].first) drain_out(g, s, threads, acc);  // the slot's previous chunk
    CK(cudaMemcpyAsync(g.ring_out[s], (const char*)d_src + o, len, cudaMemcpyDeviceToHost, st));
    CK(cudaEventRecord(g.ev_out[s], st));
    g.out_pend[s] = {(char*)h_dst + o, len};
  }
  if (!g.defer_out) flush_out(g, threads, acc);
}

struct EvPair {
  cudaEvent_t a = nullptr, b = nullptr;
  void make() {
    CK(cudaEventCreate(&a));
    CK(cudaEventCreate(&b));
  }
  void destroy() {
    if (a) cudaEventDestroy(a);
    if (b) cudaEventDestroy(b);
    a = b = nullptr;
  }
  double ms() const {
    float t = 0;
    if (cudaEventElapsedTime(&t, a, b) != cudaSuccess) {
      cudaGetLastError();
      return 0;
    }
    return t;
  }
};

// ---- planner (A1) --------------------------------------------------------------------------
constexpr double kLookbackBytesPerKey = 256.0 * 8.0 / kRadixTile;  // 0.5 B/key

// Batch boundaries (A1).  schedule 0: uniform b_s with a ragged last batch (A-12).
// schedule 1 (auto RESIDENT): b_s-sized batches, then a halving tail, so the last batch — whose
// sort is the only one no HtoD can hide — is small (~n/256).
std::vector<uint64_t> batch_offsets(uint64_t n, uint64_t b_s, int schedule) {
  std::vector<uint64_t> offs{0};
  if (n == 0) return offs;
  if (schedule == 0) {
    for (uint64_t o = b_s; o < n; o += b_s) offs.push_back(o);
    offs.push_back(n);
    return offs;
  }
  const uint64_t min_b = std::max<uint64_t>(kRadixTile, (n / 256) & ~(uint64_t)(kRadixTile - 1));
  uint64_t rem = n;
  while (rem > 0) {
    uint64_t sz;
    if (rem > 2 * b_s) sz = b_s;
    else if (rem > 2 * min_b) sz = ((rem / 2) + kRadixTile - 1) & ~(uint64_t)(kRadixTile - 1);
    else sz = rem;
    offs.push_back(offs.back() + sz);
    rem -= sz;
  }
  return offs;
}

// Cut [0, n) into N contiguous parts whose inner bounds are multiples of `align` (shards of A
// per GPU, output ranges of B per GPU).
std::vector<uint64_t> shard_bounds(uint64_t n, int N, uint64_t align) {
  std::vector<uint64_t> b(N + 1, 0);
  for (int g = 1; g < N; ++g) {
    const uint64_t x = (uint64_t)((unsigned __int128)n * (unsigned)g / (unsigned)N);
    b[g] = std::max(b[g - 1], x - x % align);
  }
  b[N] = n;
  return b;
}

// Batches of a RESIDENT plan over N GPUs: shard g of A (shard_bounds, tile-aligned) is cut by
// batch_offsets(shard, b_s, schedule); the run count is the sum over the shards.
uint64_t resident_runs(uint64_t n, int N, uint64_t b_s, int schedule, uint64_t* shard_max) {
  const std::vector<uint64_t> sh = shard_bounds(n, N, kRadixTile);
  uint64_t runs = 0, mx = 0;
  for (int g = 0; g < N; ++g) {
    const uint64_t m = sh[g + 1] - sh[g];
    if (schedule == 0 || m / std::max<uint64_t>(b_s, 1) > 4 * (uint64_t)kMaxMergeRuns)
      runs += (m + b_s - 1) / std::max<uint64_t>(b_s, 1);  // closed form (no schedule vector)
    else
      runs += batch_offsets(m, b_s, schedule).size() - 1;
    mx = std::max(mx, sh[g + 1] - sh[g]);
  }
  if (shard_max) *shard_max = mx;
  return runs;
}

// A1.  device_bytes = usable HBM per GPU; multi_ok = the GPUs can read each other's HBM (peer
// access; required by the multi-GPU RESIDENT merge).
hsort_plan_t make_plan(uint64_t n, uint64_t batch_elems, int n_gpus, uint64_t device_bytes,
                       const Options& opt, bool multi_ok = true) {
  hsort_plan_t p{};
  p.n = n;
  p.n_gpus = n_gpus;
  int n_s = (int)std::max<int64_t>(1, opt.get("n_s"));
  uint64_t reserve = (uint64_t)std::max<int64_t>(0, opt.get("device_reserve_mb")) << 20;
  const uint64_t mchunk = (uint64_t)opt.get("merge_chunk");
  uint64_t merge_buf = 2ull * mchunk * 8;
  uint64_t budget = device_bytes > reserve ? device_bytes - reserve : 0;
  // single batch footprint: keys + alt + look-back
  auto bline_bytes = [&](uint64_t b) { return (uint64_t)(b * (16.0 + kLookbackBytesPerKey)); };
  int64_t res = opt.get("resident");
  const uint64_t host_ring = 2ull * (uint64_t)opt.get("n_ring") * (uint64_t)opt.get("p_s");
  // RESIDENT footprint per GPU: its shard's runs + one batch of radix scratch + the merge slots,
  // co-rank rows and coarse table (k runs)
  const uint64_t msd = opt.get("msd") == 1 ? 1 : 0;  // MSD-first split: + the partitioned copy
  auto resident_bytes = [&](uint64_t shard, uint64_t b, uint64_t k) {
    return shard * 8 * (1 + msd) + (uint64_t)(b * (8.0 + kLookbackBytesPerKey)) + merge_buf +
           4 * (mchunk / kMergeTile + 2) * std::max<uint64_t>(k, 1) * 8 + k * 16;
  };
  auto set_resident = [&](uint64_t b, int schedule, int N, uint64_t runs, uint64_t bytes) {
    p.b_s = b;
    p.schedule = schedule;
    p.n_b = runs;
    const std::vector<uint64_t> sh = shard_bounds(n, N, kRadixTile);
    const std::vector<uint64_t> offs = batch_offsets(sh[N] - sh[N - 1], b, schedule);
    p.last_batch = offs.size() > 1 ? offs[offs.size() - 1] - offs[offs.size() - 2] : 0;
    p.n_s = 1;
    p.n_gpus = N;
    p.mode = HSORT_MODE_RESIDENT;
    p.device_bytes_per_gpu = bytes;
    p.host_bytes = host_ring * (uint64_t)N;
    p.batches_per_stream = (double)runs / N;
    return p;
  };
  // Pipelined RESIDENT plan (the auto plan for arrays whose runs fit in HBM, on one or N GPUs):
  // 2^27-key batches + a halving tail per shard, so HtoD of batch i+1 overlaps the sort of batch i
  // and the merge overlaps the DtoH.  With an explicit batch_elems the shards are
  // cut into uniform b_s batches instead (schedule 0).
  const uint64_t auto_min = (uint64_t)std::max<int64_t>(0, opt.get("auto_pipeline_min"));
  const int N = std::max(1, n_gpus);
  const bool multi = N > 1 && multi_ok;
  if (n > 0 && res != 0 && (N == 1 || multi)) {
    uint64_t smax = 0;  // largest shard
    const std::vector<uint64_t> sh = shard_bounds(n, N, kRadixTile);
    for (int g = 0; g < N; ++g) smax = std::max(smax, sh[g + 1] - sh[g]);
    if (batch_elems == 0 && auto_min && n >= auto_min) {
      uint64_t b0 = std::min<uint64_t>(1ull << 27, std::max<uint64_t>(smax / 8, kRadixTile));
      b0 -= b0 % kRadixTile;
      const uint64_t runs = resident_runs(n, N, b0, 1, nullptr);
      const uint64_t rb = resident_bytes(smax, b0, runs);
      if (runs <= (uint64_t)kMaxMergeRuns && rb <= budget) return set_resident(b0, 1, N, runs, rb);
    } else if (multi && batch_elems > 0 && batch_elems < n) {
      const uint64_t b = std::min<uint64_t>(batch_elems, std::max<uint64_t>(smax, 1));
      const uint64_t runs = resident_runs(n, N, b, 0, nullptr);
      const uint64_t rb = resident_bytes(smax, b, runs);
      if (runs <= (uint64_t)kMaxMergeRuns && (res == 1 || rb <= budget))
        return set_resident(b, 0, N, runs, rb);
    }
  }
  uint64_t b_s;
  if (batch_elems == 0) {
    if (bline_bytes(n) <= budget) {
      b_s = n;
    } else {
      // n_s resident slots + one shared alt buffer (b_s chosen to fill global memory)
      double per = 8.0 * (n_s + 1) + kLookbackBytesPerKey;
      b_s = (uint64_t)((double)budget / per);
      b_s -= b_s % kRadixTile;
      if (b_s == 0) b_s = kRadixTile;
      b_s = std::min<uint64_t>(b_s, 1ull << 30);  // the fast onesweep pass handles n <= 2^30
    }
  } else {
    b_s = std::min<uint64_t>(batch_elems, n ? n : 1);
  }
  if (b_s == 0) b_s = 1;
  p.b_s = b_s;
  p.n_b = n ? (n + b_s - 1) / b_s : 0;
  p.last_batch = n ? n - (p.n_b - 1) * b_s : 0;
  p.n_s = p.n_b <= 1 ? 1 : (int)std::min<uint64_t>((uint64_t)n_s, p.n_b);
  const uint64_t rb1 = resident_bytes(n, b_s, std::min<uint64_t>(p.n_b, kMaxMergeRuns));
  if (p.n_b <= 1) {
    p.mode = HSORT_MODE_BLINE;
    p.device_bytes_per_gpu = bline_bytes(n);
    p.n_gpus = 1;
  } else if (N == 1 && p.n_b <= (uint64_t)kMaxMergeRuns &&
             (res == 1 || (res == -1 && rb1 <= budget))) {
    p.mode = HSORT_MODE_RESIDENT;
    p.device_bytes_per_gpu = rb1;
    p.n_gpus = 1;
  } else {
    p.mode = HSORT_MODE_STREAM;
    p.n_gpus = (int)std::min<uint64_t>((uint64_t)N, p.n_b);
    p.device_bytes_per_gpu = (uint64_t)(b_s * (8.0 * (p.n_s + 1) + kLookbackBytesPerKey));
  }
  p.host_bytes = (p.mode == HSORT_MODE_STREAM ? n * 8 : 0) + host_ring * (uint64_t)std::max(1, p.n_gpus);
  p.batches_per_stream = p.n_b ? (double)p.n_b / ((double)p.n_s * std::max(1, p.n_gpus)) : 0.0;
  return p;
}

// ---- mode drivers --------------------------------------------------------------------------
struct CallCtx {
  const void* A;
  void* B;
  uint64_t n;
  bool f64;  // keys are float64 bits (transform on the GPU) vs raw uint64
  hsort_plan_t plan;
  bool direct_in, direct_out;
  int mc_threads, merge_threads;
  hsort_stats* st;
  // key/value calls (S§8(f) #3): the values V (host, n) and VB; nullptr for keys-only calls
  const uint64_t* V = nullptr;
  uint64_t* VB = nullptr;
  bool direct_vin = false, direct_vout = false;
};

void sort_bline(GpuCtx& g, CallCtx& c) {
  CK(cudaSetDevice(g.dev));
  const uint64_t n = c.n;
  g.runs.reserve(n * 8);
  g.alt.reserve(n * 8);
  Acc acc;
  EvPair eh, es, ed;
  eh.make();
  es.make();
  ed.make();
  auto t0 = Clock::now();
  CK(cudaEventRecord(eh.a, g.s_h2d));
  upload(g, g.runs.p, c.A, n * 8, g.s_h2d, c.direct_in, c.mc_threads, acc);
  CK(cudaEventRecord(eh.b, g.s_h2d));
  CK(cudaStreamWaitEvent(g.s_comp, eh.b, 0));
  CK(cudaEventRecord(es.a, g.s_comp));
  CK(radix_sort(g.rs, g.runs.u64(), g.runs.u64(), g.alt.u64(), n, c.f64, c.f64, g.s_comp));
  CK(cudaEventRecord(es.b, g.s_comp));
  CK(cudaStreamWaitEvent(g.s_d2h, es.b, 0));
  CK(cudaEventRecord(ed.a, g.s_d2h));
  download(g, c.B, g.runs.p, n * 8, g.s_d2h, c.direct_out, c.mc_threads, acc);
  CK(cudaEventRecord(ed.b, g.s_d2h));
  CK(cudaStreamSynchronize(g.s_d2h));
  c.st->t_sort_phase = secs_since(t0);
  c.st->t_h2d = eh.ms() / 1e3;
  c.st->t_gpu_sort = es.ms() / 1e3;
  c.st->t_d2h = ed.ms() / 1e3;
  c.st->t_stage = acc.t_stage;
  c.st->bytes_h2d = acc.h2d;
  c.st->bytes_d2h = acc.d2h;
  c.st->passes_run = g.rs.h_plan->num_active;
  c.st->passes_skipped = 8 - g.rs.h_plan->num_active;
  eh.destroy();
  es.destroy();
  ed.destroy();
}

// Per-GPU accumulators of one call (each GPU's host thread owns one; summed into hsort_stats).
struct PhaseTimes {
  Acc acc;
  double t_h2d = 0, t_sort = 0, t_d2h = 0, t_merge = 0;
  int passes = 0;
};

// Run fn(i) for i in [0, N) on N host threads (inline when N == 1); the first failure is
// rethrown after every thread has joined.
template <class F>
void run_per_gpu(size_t N, F fn) {
  if (N == 1) {
    fn(0);
    return;
  }
  std::mutex m;
  int code = 0;
  std::string msg;
  std::vector<std::thread> th;
  for (size_t i = 0; i < N; ++i)
    th.emplace_back([&, i] {
      auto fail = [&](int c, const std::string& w) {
        std::lock_guard<std::mutex> g(m);
        if (!code) {
          code = c;
          msg = w;
        }
      };
      try {
        fn(i);
      } catch (const HsortError& e) {
        fail(e.code, e.what());
      } catch (const std::bad_alloc&) {
        fail(HSORT_ERR_HOST_OOM, "host allocation failed");
      } catch (const std::exception& e) {
        fail(HSORT_ERR_INTERNAL, e.what());
      } catch (...) {
        fail(HSORT_ERR_INTERNAL, "unknown exception");
      }
    });
  for (auto& t : th) t.join();
  if (code) throw HsortError(code, msg);
}

// K4 on g.s_comp with the library-owned coarse-level scratch of this GPU context.
void corank_on(GpuCtx& g, const uint64_t* keys, const uint64_t* const* rp, const uint64_t* d_off,
               int k, uint64_t total, uint64_t step, uint64_t b0, uint64_t nb, uint64_t* ranks,
               cudaStream_t st) {
  const uint64_t need = merge_corank_scratch_elems(k, total, step, b0, nb);
  if (need * 8 > g.coarse.cap) {
    CK(cudaStreamSynchronize(st));  // the buffer may still be read by an earlier K4 on st
    g.coarse.reserve(need * 8);
  }
  CK(merge_corank(keys, rp, d_off, k, total, step, b0, nb, ranks, g.coarse.u64(), g.coarse.cap / 8, st));
}

// GPU merge (K4 + K5) of the k runs (keys | rp, d_off; `total` keys) -- output positions
// [o_lo, o_hi) into B + o_lo, chunk by chunk: the co-ranks of chunk c are computed just before
// its merge, and the DtoH of chunk c overlaps the merge of chunk c+1 (two output slots), so the
// first bytes leave the GPU one chunk after the last batch is sorted.  o_lo is a multiple of
// kMergeTile (a merge tile boundary); o_hi is one too, or total.  With rp the runs are read where
// they lie, including other GPUs' HBM over NVLink (peer access): the multi-GPU exchange is fused
// into K4/K5's loads.
void gpu_merge_to_host(GpuCtx& g, CallCtx& c, const uint64_t* d_keys, const uint64_t* const* d_rp,
                       const uint64_t* d_off, int k, uint64_t total, uint64_t o_lo, uint64_t o_hi,
                       PhaseTimes& pt, const uint64_t* d_vkeys = nullptr,
                       const uint64_t* const* d_vrp = nullptr) {
  const bool kv = c.VB != nullptr;
  if (o_hi <= o_lo) return;
  Nvtx nv("GPU merge -> B");
  const uint64_t t_lo = o_lo / kMergeTile;
  const uint64_t t_hi = (o_hi + kMergeTile - 1) / kMergeTile;
  const uint64_t tiles = t_hi - t_lo;
  const uint64_t ctiles = std::max<uint64_t>(1, (uint64_t)S().opt.get("merge_chunk") / kMergeTile);
  const uint64_t chunk = ctiles * kMergeTile;
  const uint64_t nch = (tiles + ctiles - 1) / ctiles;
  const uint64_t slots = nch > 1 ? 2 : 1;
  g.mout.reserve(slots * chunk * 8);
  if (kv) g.vmout.reserve(slots * chunk * 8);
  g.ranks.reserve(slots * (ctiles + 1) * (uint64_t)k * 8);
  std::vector<cudaEvent_t> ev_done(slots), ev_free(slots);
  std::vector<EvPair> em(nch), ed(nch);
  for (uint64_t s = 0; s < slots; ++s) {
    CK(cudaEventCreateWithFlags(&ev_done[s], cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&ev_free[s], cudaEventDisableTiming));
    CK(cudaEventRecord(ev_free[s], g.s_d2h));
  }
  for (uint64_t ch = 0; ch < nch; ++ch) {
    em[ch].make();
    ed[ch].make();
  }
  char* B = (char*)c.B;
  auto enqueue_merge = [&](uint64_t ch) {
    const uint64_t s = ch % slots;
    const uint64_t tb = t_lo + ch * ctiles, tc = std::min(ctiles, t_hi - tb);
    uint64_t* rk = g.ranks.u64() + s * (ctiles + 1) * (uint64_t)k;
    CK(cudaStreamWaitEvent(g.s_comp, ev_free[s], 0));
    CK(cudaEventRecord(em[ch].a, g.s_comp));
    corank_on(g, d_keys, d_rp, d_off, k, total, kMergeTile, tb, tc + 1, rk, g.s_comp);
    CK(merge_tiles(d_keys, d_rp, d_off, k, total, rk, tb, tb, tc, g.mout.u64() + s * chunk,
                   tb * kMergeTile, c.f64, g.s_comp, d_vkeys, d_vrp,
                   kv ? g.vmout.u64() + s * chunk : nullptr));
    CK(cudaEventRecord(em[ch].b, g.s_comp));
    CK(cudaEventRecord(ev_done[s], g.s_comp));
  };
  enqueue_merge(0);
  for (uint64_t ch = 0; ch < nch; ++ch) {
    if (ch + 1 < nch) enqueue_merge(ch + 1);
    const uint64_t s = ch % slots;
    const uint64_t o = (t_lo + ch * ctiles) * kMergeTile, len = std::min(chunk, o_hi - o);
    CK(cudaStreamWaitEvent(g.s_d2h, ev_done[s], 0));
    CK(cudaEventRecord(ed[ch].a, g.s_d2h));
    download(g, B + o * 8, g.mout.u64() + s * chunk, len * 8, g.s_d2h, c.direct_out, c.mc_threads,
             pt.acc);
    if (kv)
      download(g, c.VB + o, g.vmout.u64() + s * chunk, len * 8, g.s_d2h, c.direct_vout, c.mc_threads,
               pt.acc);
    CK(cudaEventRecord(ed[ch].b, g.s_d2h));
    CK(cudaEventRecord(ev_free[s], g.s_d2h));
  }
  CK(cudaStreamSynchronize(g.s_d2h));
  CK(cudaStreamSynchronize(g.s_comp));
  for (uint64_t ch = 0; ch < nch; ++ch) {
    pt.t_merge += em[ch].ms() / 1e3;
    pt.t_d2h += ed[ch].ms() / 1e3;
    em[ch].destroy();
    ed[ch].destroy();
  }
  for (uint64_t s = 0; s < slots; ++s) {
    cudaEventDestroy(ev_done[s]);
    cudaEventDestroy(ev_free[s]);
  }
}

// Sort phase of the RESIDENT mode on one GPU: the batches [h_off[i], h_off[i+1]) of the shard
// A + a0 are HtoD'd into g.runs at the same offsets and sorted in place (runs stay in HBM, in key
// form); the HtoD of batch i+1 overlaps the sort of batch i.
void resident_sort_phase(GpuCtx& g, CallCtx& c, uint64_t a0, const std::vector<uint64_t>& h_off,
                         PhaseTimes& pt) {
  CK(cudaSetDevice(g.dev));
  const uint64_t nb = h_off.size() - 1, shard = h_off[nb];
  if (shard == 0) return;
  Nvtx nv("sort phase (resident)");
  uint64_t bmax = 0;
  for (uint64_t i = 0; i < nb; ++i) bmax = std::max(bmax, h_off[i + 1] - h_off[i]);
  const bool kv = c.V != nullptr;
  g.runs.reserve(shard * 8);
  g.alt.reserve(bmax * 8);
  if (kv) {
    g.vruns.reserve(shard * 8);
    g.valt.reserve(bmax * 8);
  }
  std::vector<EvPair> eh(nb), es(nb);
  for (auto& e : eh) e.make();
  for (auto& e : es) e.make();
  for (uint64_t i = 0; i < nb; ++i) {
    const uint64_t o = h_off[i], len = h_off[i + 1] - h_off[i];
    CK(cudaEventRecord(eh[i].a, g.s_h2d));
    upload(g, g.runs.u64() + o, (const char*)c.A + (a0 + o) * 8, len * 8, g.s_h2d, c.direct_in,
           c.mc_threads, pt.acc);
    if (kv)
      upload(g, g.vruns.u64() + o, c.V + a0 + o, len * 8, g.s_h2d, c.direct_vin, c.mc_threads, pt.acc);
    CK(cudaEventRecord(eh[i].b, g.s_h2d));
    CK(cudaStreamWaitEvent(g.s_comp, eh[i].b, 0));
    CK(cudaEventRecord(es[i].a, g.s_comp));
    if (kv)  // stable key/value GPUSort of the batch, in place; keys stay transformed for the merge
      CK(radix_sort_pairs(g.rs, g.runs.u64() + o, g.vruns.u64() + o, g.runs.u64() + o,
                          g.vruns.u64() + o, g.alt.u64(), g.valt.u64(), len, c.f64, false, g.s_comp));
    else
      CK(radix_sort(g.rs, g.runs.u64() + o, g.runs.u64() + o, g.alt.u64(), len, c.f64, false, g.s_comp));
    CK(cudaEventRecord(es[i].b, g.s_comp));
  }
  CK(cudaStreamSynchronize(g.s_comp));
  pt.passes = g.rs.h_plan->num_active;  // plan of the last batch
  for (uint64_t i = 0; i < nb; ++i) {
    pt.t_h2d += eh[i].ms() / 1e3;
    pt.t_sort += es[i].ms() / 1e3;
  }
  for (auto& e : eh) e.destroy();
  for (auto& e : es) e.destroy();
}

// RESIDENT mode over N >= 1 GPUs (A1 picks it when the runs fit in N x HBM):
//  1. A is cut into N contiguous shards; GPU g sorts shard g as batches that stay resident
//     (n_b/(n_s n_GPU) batches per stream), every GPU on its own host thread;
//  2. the output B is cut into N ranges at merge-tile boundaries; GPU g merges its range from ALL
//     runs (K4 co-ranks + K5 tiles reading the other GPUs' runs by peer loads: the splitter
//     exchange, S§8(a) A13, fused into the merge) and DMAs it straight to B[o_g, o_{g+1}).
// With N = 1 this is the single-GPU RESIDENT schedule (runs back to back in g.runs, no table).
void sort_resident(std::vector<GpuCtx*>& gs, CallCtx& c) {
  const size_t N = gs.size();
  const uint64_t n = c.n;
  const std::vector<uint64_t> shard = shard_bounds(n, (int)N, kRadixTile);
  std::vector<std::vector<uint64_t>> h_off(N);
  uint64_t n_runs = 0;
  for (size_t g = 0; g < N; ++g) {
    h_off[g] = batch_offsets(shard[g + 1] - shard[g], c.plan.b_s, c.plan.schedule);
    n_runs += h_off[g].size() - 1;
  }
  if (n_runs != c.plan.n_b) throw HsortError(HSORT_ERR_INTERNAL, "batch schedule mismatch");
  std::vector<PhaseTimes> pt(N);
  auto t0 = Clock::now();
  run_per_gpu(N, [&](size_t g) { resident_sort_phase(*gs[g], c, shard[g], h_off[g], pt[g]); });
  c.st->t_sort_phase = secs_since(t0);
  // the global run table (run order: GPU-major, then batch): device pointers and offsets
  std::vector<const uint64_t*> rp, vrp;
  std::vector<uint64_t> goff{0};
  for (size_t g = 0; g < N; ++g)
    for (size_t i = 0; i + 1 < h_off[g].size(); ++i) {
      rp.push_back(gs[g]->runs.u64() + h_off[g][i]);
      if (c.V) vrp.push_back(gs[g]->vruns.u64() + h_off[g][i]);
      goff.push_back(goff.back() + h_off[g][i + 1] - h_off[g][i]);
    }
  const int k = (int)rp.size();
  const std::vector<uint64_t> orng = shard_bounds(n, (int)N, kMergeTile);
  auto t1 = Clock::now();
  run_per_gpu(N, [&](size_t gi) {
    GpuCtx& g = *gs[gi];
    CK(cudaSetDevice(g.dev));
    g.off.reserve((k + 1) * 8);
    CK(cudaMemcpyAsync(g.off.p, goff.data(), (k + 1) * 8, cudaMemcpyHostToDevice, g.s_comp));
    if (N == 1) {
      gpu_merge_to_host(g, c, g.runs.u64(), nullptr, g.off.u64(), k, n, 0, n, pt[gi],
                        c.V ? g.vruns.u64() : nullptr, nullptr);
    } else {
      g.rptr.reserve(k * sizeof(void*));
      CK(cudaMemcpyAsync(g.rptr.p, rp.data(), k * sizeof(void*), cudaMemcpyHostToDevice, g.s_comp));
      const uint64_t* const* d_vrp = nullptr;
      if (c.V) {
        g.vrptr.reserve(k * sizeof(void*));
        CK(cudaMemcpyAsync(g.vrptr.p, vrp.data(), k * sizeof(void*), cudaMemcpyHostToDevice, g.s_comp));
        d_vrp = (const uint64_t* const*)g.vrptr.p;
      }
      gpu_merge_to_host(g, c, nullptr, (const uint64_t* const*)g.rptr.p, g.off.u64(), k, n,
                        orng[gi], orng[gi + 1], pt[gi], nullptr, d_vrp);
    }
  });
  c.st->t_merge_phase = secs_since(t1);
  c.st->merge_gpu_fraction = 1.0;
  for (auto& P : pt) {
    c.st->t_h2d += P.t_h2d;
    c.st->t_gpu_sort += P.t_sort;
    c.st->t_merge_gpu += P.t_merge;
    c.st->t_d2h += P.t_d2h;
    c.st->t_stage += P.acc.t_stage;
    c.st->bytes_h2d += P.acc.h2d;
    c.st->bytes_d2h += P.acc.d2h;
    c.st->passes_run = std::max(c.st->passes_run, P.passes);
  }
  c.st->passes_skipped = 8 - c.st->passes_run;
}

// ---- N2: MSD-first split (S§8(f) #2, option "msd") --------------------------------------------
inline uint64_t host_key(uint64_t u) { return u ^ ((uint64_t)((int64_t)u >> 63) | (1ull << 63)); }
inline uint64_t mix64(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}

// R - 1 splitters (key space) at the quantiles of S regularly hashed samples of A: bucket r =
// (s_{r-1}, s_r].  Only the load balance depends on them, never the result.
std::vector<uint64_t> sample_splitters(const void* A, uint64_t n, bool f64, int R) {
  const uint64_t S = std::min<uint64_t>(n, std::max<uint64_t>(64ull * R, 1ull << 16));
  std::vector<uint64_t> smp(S);
  const uint64_t* a = (const uint64_t*)A;
  for (uint64_t i = 0; i < S; ++i) {
    const uint64_t u = a[mix64(i) % n];
    smp[i] = f64 ? host_key(u) : u;
  }
  std::sort(smp.begin(), smp.end());
  std::vector<uint64_t> spl(std::max(R - 1, 0));
  for (int r = 0; r + 1 < R; ++r) spl[r] = smp[(uint64_t)(r + 1) * S / R - 1];
  return spl;
}

// The MSD-first split over N >= 1 GPUs (replaces the merge of sort_resident):
//  1. GPU g uploads its shard of A batch by batch; each batch is partitioned into R buckets by
//     the sampled splitters (K6a-c) while the next one uploads;
//  2. the host sums the bucket sizes, gives every GPU a contiguous run of buckets (~n/N keys) and
//     places bucket r at B[sum_{r' < r} T_r'];
//  3. GPU g gathers its buckets' segments from every GPU's partitioned batches (K6d: peer loads
//     over NVLink = the exchange), LSD-sorts each bucket in place (inverse transform fused into the
//     last pass; high digits constant inside a bucket are skipped by K2) and DMAs it to B while
//     the next bucket sorts.
void sort_msd(std::vector<GpuCtx*>& gs, CallCtx& c) {
  const size_t N = gs.size();
  const uint64_t n = c.n;
  const std::vector<uint64_t> shard = shard_bounds(n, (int)N, kRadixTile);
  std::vector<std::vector<uint64_t>> h_off(N);
  for (size_t g = 0; g < N; ++g) h_off[g] = batch_offsets(shard[g + 1] - shard[g], c.plan.b_s, c.plan.schedule);
  const uint64_t bk = (uint64_t)std::max<int64_t>(1 << 16, S().opt.get("msd_bucket_keys"));
  int R = (int)std::min<uint64_t>(kMaxBuckets, std::max<uint64_t>(4 * N, n / bk));
  R -= R % (int)N;
  std::vector<uint64_t> spl;
  std::mutex spl_m;
  std::condition_variable spl_cv;
  bool spl_ready = false;
  bool spl_failed = false;
  std::thread sampler([&] {
    std::vector<uint64_t> v;
    bool ok = true;
    try {
      v = sample_splitters(c.A, n, c.f64, R);
    } catch (...) {
      ok = false;
    }
    {
      std::lock_guard<std::mutex> lk(spl_m);
      spl = std::move(v);
      spl_failed = !ok;
      spl_ready = true;
    }
    spl_cv.notify_all();
  });
  struct SamplerJoin {
    std::thread& t;
    ~SamplerJoin() {
      if (t.joinable()) t.join();
    }
  } sj{sampler};
  std::vector<std::vector<uint32_t>> tot(N);  // [batch][R] bucket sizes per GPU
  std::vector<PhaseTimes> pt(N);
  auto t0 = Clock::now();
  run_per_gpu(N, [&](size_t gi) {
    GpuCtx& g = *gs[gi];
    CK(cudaSetDevice(g.dev));
    const std::vector<uint64_t>& off = h_off[gi];
    const uint64_t nb = off.size() - 1, sh = off[nb];
    if (sh == 0) return;
    uint64_t bmax = 0;
    for (uint64_t i = 0; i < nb; ++i) bmax = std::max(bmax, off[i + 1] - off[i]);
    g.runs.reserve(sh * 8);
    g.part.reserve(sh * 8);
    g.bcnt.reserve(bucket_count_elems(bmax, R) * 4);
    g.btot.reserve(nb * R * 4);
    g.bspl.reserve(R * 8);
    std::vector<EvPair> eh(nb), es(nb);
    for (auto& e : eh) e.make();
    for (auto& e : es) e.make();
    for (uint64_t i = 0; i < nb; ++i) {
      const uint64_t o = off[i], len = off[i + 1] - off[i];
      CK(cudaEventRecord(eh[i].a, g.s_h2d));
      upload(g, g.runs.u64() + o, (const char*)c.A + (shard[gi] + o) * 8, len * 8, g.s_h2d,
             c.direct_in, c.mc_threads, pt[gi].acc);
      CK(cudaEventRecord(eh[i].b, g.s_h2d));
      if (i == 0) {  // the splitters are sampled while the first batch uploads
        std::unique_lock<std::mutex> lk(spl_m);
        spl_cv.wait(lk, [&] { return spl_ready; });
        if (spl_failed) throw HsortError(HSORT_ERR_HOST_OOM, "splitter sampling failed");
        if (R > 1)
          CK(cudaMemcpyAsync(g.bspl.p, spl.data(), (R - 1) * 8, cudaMemcpyHostToDevice, g.s_comp));
      }
      CK(cudaStreamWaitEvent(g.s_comp, eh[i].b, 0));
      CK(cudaEventRecord(es[i].a, g.s_comp));
      CK(bucket_partition(g.runs.u64() + o, len, c.f64, g.bspl.u64(), R, (uint32_t*)g.bcnt.p,
                          (uint32_t*)g.btot.p + i * R, g.part.u64() + o, g.s_comp));
      CK(cudaEventRecord(es[i].b, g.s_comp));
    }
    tot[gi].resize(nb * R);
    CK(cudaMemcpyAsync(tot[gi].data(), g.btot.p, nb * R * 4, cudaMemcpyDeviceToHost, g.s_comp));
    CK(cudaStreamSynchronize(g.s_comp));
    for (uint64_t i = 0; i < nb; ++i) {
      pt[gi].t_h2d += eh[i].ms() / 1e3;
      pt[gi].t_sort += es[i].ms() / 1e3;
    }
    for (auto& e : eh) e.destroy();
    for (auto& e : es) e.destroy();
  });
  c.st->t_sort_phase = secs_since(t0);
  // bucket sizes, owners (contiguous bucket runs of ~n/N keys), places in B and in the owner's
  // receive buffer (bucket starts kept 16-byte aligned for the TMA passes)
  std::vector<uint64_t> T(R, 0), G(R + 1, 0);
  for (size_t h = 0; h < N; ++h)
    for (size_t i = 0; i < tot[h].size(); ++i) T[i % R] += tot[h][i];
  for (int r = 0; r < R; ++r) G[r + 1] = G[r] + T[r];
  if (G[R] != n) throw HsortError(HSORT_ERR_INTERNAL, "bucket sizes do not add up to n");
  std::vector<int> first(N + 1, R);
  first[0] = 0;
  {
    size_t g = 1;
    for (int r = 0; r < R && g < N; ++r)
      while (g < N && G[r + 1] > (uint64_t)((unsigned __int128)n * g / N)) first[g++] = r + 1;
    for (; g < N; ++g) first[g] = R;
    for (size_t q = 1; q < N; ++q) first[q] = std::max(first[q], first[q - 1]);
  }
  auto t1 = Clock::now();
  run_per_gpu(N, [&](size_t gi) {
    GpuCtx& g = *gs[gi];
    CK(cudaSetDevice(g.dev));
    const int r0 = first[gi], r1 = first[gi + 1];
    if (r1 <= r0) return;
    std::vector<GatherSeg> segs;
    std::vector<uint64_t> pstart{0}, roff(r1 - r0 + 1, 0);
    uint64_t cap = 0, tmax = 0;
    for (int r = r0; r < r1; ++r) {
      roff[r - r0] = cap;
      for (size_t h = 0; h < N; ++h) {
        const uint64_t nb = h_off[h].size() - 1;
        for (uint64_t i = 0; i < nb; ++i) {
          const uint32_t* tb = &tot[h][i * R];
          const uint64_t len = tb[r];
          if (!len) continue;
          uint64_t bb = 0;  // start of bucket r inside batch i of GPU h
          for (int q = 0; q < r; ++q) bb += tb[q];
          segs.push_back({gs[h]->part.u64() + h_off[h][i] + bb, len, cap});
          cap += len;
          pstart.push_back(pstart.back() + gather_pieces(len));
        }
      }
      tmax = std::max(tmax, T[r]);
      cap += cap & 1;  // next bucket 16-byte aligned
    }
    roff[r1 - r0] = cap;
    if (segs.empty()) return;
    pstart.pop_back();
    const uint64_t pieces = pstart.back() + gather_pieces(segs.back().len);
    g.runs.reserve(std::max<uint64_t>(cap, 2) * 8);  // this GPU's raw batches are partitioned: free
    g.alt.reserve(std::max<uint64_t>(tmax, 2) * 8);
    const size_t tb_bytes = segs.size() * sizeof(GatherSeg);
    g.bseg.reserve(tb_bytes + pstart.size() * 8);
    CK(cudaMemcpyAsync(g.bseg.p, segs.data(), tb_bytes, cudaMemcpyHostToDevice, g.s_comp));
    CK(cudaMemcpyAsync((char*)g.bseg.p + tb_bytes, pstart.data(), pstart.size() * 8,
                       cudaMemcpyHostToDevice, g.s_comp));
    EvPair eg;
    eg.make();
    CK(cudaEventRecord(eg.a, g.s_comp));
    CK(gather_segments((const GatherSeg*)g.bseg.p, (const uint64_t*)((char*)g.bseg.p + tb_bytes),
                       (int)segs.size(), pieces, g.runs.u64(), g.s_comp));
    CK(cudaEventRecord(eg.b, g.s_comp));
    const int nr = r1 - r0;
    std::vector<EvPair> es(nr), ed(nr);
    for (int q = 0; q < nr; ++q) {
      es[q].make();
      ed[q].make();
    }
    // every bucket's sort is enqueued first (one compute stream), then the DtoH of bucket q waits
    // for its sort only, so sorts and DtoH overlap
    for (int q = 0; q < nr; ++q) {
      CK(cudaEventRecord(es[q].a, g.s_comp));
      if (T[r0 + q])
        CK(radix_sort(g.rs, g.runs.u64() + roff[q], g.runs.u64() + roff[q], g.alt.u64(), T[r0 + q],
                      false, c.f64, g.s_comp));
      CK(cudaEventRecord(es[q].b, g.s_comp));
    }
    for (int q = 0; q < nr; ++q) {
      CK(cudaStreamWaitEvent(g.s_d2h, es[q].b, 0));
      CK(cudaEventRecord(ed[q].a, g.s_d2h));
      download(g, (char*)c.B + G[r0 + q] * 8, g.runs.u64() + roff[q], T[r0 + q] * 8, g.s_d2h,
               c.direct_out, c.mc_threads, pt[gi].acc);
      CK(cudaEventRecord(ed[q].b, g.s_d2h));
    }
    CK(cudaStreamSynchronize(g.s_d2h));
    CK(cudaStreamSynchronize(g.s_comp));
    pt[gi].t_merge += eg.ms() / 1e3;  // the exchange (gather) takes the merge's place
    for (int q = 0; q < nr; ++q) {
      pt[gi].t_sort += es[q].ms() / 1e3;
      pt[gi].t_d2h += ed[q].ms() / 1e3;
      es[q].destroy();
      ed[q].destroy();
    }
    eg.destroy();
    pt[gi].passes = g.rs.h_plan->num_active;
  });
  c.st->t_merge_phase = secs_since(t1);
  c.st->merge_gpu_fraction = 1.0;
  c.st->msd_buckets = R;
  for (auto& P : pt) {
    c.st->t_h2d += P.t_h2d;
    c.st->t_gpu_sort += P.t_sort;
    c.st->t_merge_gpu += P.t_merge;
    c.st->t_d2h += P.t_d2h;
    c.st->t_stage += P.acc.t_stage;
    c.st->bytes_h2d += P.acc.h2d;
    c.st->bytes_d2h += P.acc.d2h;
    c.st->passes_run = std::max(c.st->passes_run, P.passes);
  }
  c.st->passes_skipped = 8 - c.st->passes_run;
}

// GPU share of the STREAM merge: output positions [o_lo, o_hi) of the merge of the k runs in
// host memory W, in chunks of `merge_chunk` keys: exact co-ranks on the host, HtoD of the k
// slices (direct from pinned W), K4/K5 on the GPU, DtoH into B.  Two slots: the HtoD of chunk c+1
// overlaps the merge and DtoH of chunk c.
void gpu_merge_from_host(GpuCtx& g, CallCtx& c, const std::vector<const uint64_t*>& run,
                         const std::vector<uint64_t>& rlen, uint64_t o_lo, uint64_t o_hi,
                         bool w_direct, double* t_gpu) {
  Nvtx nv("GPU merge share W -> B");
  CK(cudaSetDevice(g.dev));
  const int k = (int)run.size();
  const uint64_t C = std::max<uint64_t>(
      kMergeTile, ((uint64_t)S().opt.get("merge_chunk") / kMergeTile) * kMergeTile);
  const uint64_t nch = (o_hi - o_lo + C - 1) / C;
  const uint64_t tiles_c = C / kMergeTile;
  g.min.reserve(2 * C * 8);
  g.mout.reserve(2 * C * 8);
  g.ranks.reserve(2 * (tiles_c + 1) * (uint64_t)k * 8);
  g.off.reserve(2 * (k + 1) * 8);
  std::vector<uint64_t> cr((nch + 1) * (size_t)k);
  host_pool().parallel_for((int64_t)nch + 1, host_threads(), [&](int64_t i) {
    const uint64_t p = std::min(o_lo + (uint64_t)i * C, o_hi);
    host_corank_runs(run.data(), rlen.data(), k, p, &cr[(size_t)i * k]);
  });
  cudaEvent_t in_ready[2], in_free[2], merged[2], out_free[2];
  for (int s = 0; s < 2; ++s) {
    CK(cudaEventCreateWithFlags(&in_ready[s], cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&in_free[s], cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&merged[s], cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&out_free[s], cudaEventDisableTiming));
    CK(cudaEventRecord(in_free[s], g.s_comp));
    CK(cudaEventRecord(out_free[s], g.s_d2h));
  }
  EvPair em;
  em.make();
  std::vector<uint64_t> hoff(2 * (size_t)(k + 1));
  Acc acc;
  // a staged (pageable B) download of chunk ch leaves its last ring slots pending, so chunk ch+1's
  // DMAs start at once instead of after the copy-out tail (HSORT option defer_out_drain)
  struct DeferGuard {
    GpuCtx& g;
    ~DeferGuard() {
      g.defer_out = false;
      std::fill(g.out_pend.begin(), g.out_pend.end(), std::make_pair((char*)nullptr, (uint64_t)0));
    }
  } dg{g};
  g.defer_out = S().opt.get("defer_out_drain") == 1;
  CK(cudaEventRecord(em.a, g.s_h2d));
  // Chunk ch+1's HtoD + K4/K5 are enqueued before chunk ch's (possibly staged, blocking) DtoH, so
  // the two link directions overlap (duplex); two slots per buffer.
  std::vector<uint64_t> totals(nch, 0);
  auto enqueue = [&](uint64_t ch) {
    const int s = (int)(ch & 1);
    const uint64_t* r0 = &cr[(size_t)ch * k];
    const uint64_t* r1 = &cr[(size_t)(ch + 1) * k];
    uint64_t* din = g.min.u64() + (uint64_t)s * C;
    uint64_t* ho = &hoff[(size_t)s * (k + 1)];
    if (ch >= 2) CK(cudaEventSynchronize(in_ready[s]));  // chunk ch-2's offsets copy read ho
    ho[0] = 0;
    CK(cudaStreamWaitEvent(g.s_h2d, in_free[s], 0));
    for (int j = 0; j < k; ++j) {
      const uint64_t len = r1[j] - r0[j];
      ho[j + 1] = ho[j] + len;
      if (len) upload(g, din + ho[j], run[j] + r0[j], len * 8, g.s_h2d, w_direct, c.mc_threads, acc);
    }
    uint64_t* doff = g.off.u64() + (size_t)s * (k + 1);
    CK(cudaMemcpyAsync(doff, ho, (k + 1) * 8, cudaMemcpyHostToDevice, g.s_h2d));
    CK(cudaEventRecord(in_ready[s], g.s_h2d));
    const uint64_t total = ho[k];
    totals[ch] = total;
    const uint64_t tiles = (total + kMergeTile - 1) / kMergeTile;
    uint64_t* rk = g.ranks.u64() + (uint64_t)s * (tiles_c + 1) * k;
    uint64_t* dout = g.mout.u64() + (uint64_t)s * C;
    CK(cudaStreamWaitEvent(g.s_comp, in_ready[s], 0));
    CK(cudaStreamWaitEvent(g.s_comp, out_free[s], 0));
    corank_on(g, din, nullptr, doff, k, total, kMergeTile, 0, tiles + 1, rk, g.s_comp);
    CK(merge_tiles(din, nullptr, doff, k, total, rk, 0, 0, tiles, dout, 0, c.f64, g.s_comp));
    CK(cudaEventRecord(in_free[s], g.s_comp));
    CK(cudaEventRecord(merged[s], g.s_comp));
  };
  if (nch) enqueue(0);
  for (uint64_t ch = 0; ch < nch; ++ch) {
    const int s = (int)(ch & 1);
    if (ch + 1 < nch) enqueue(ch + 1);
    CK(cudaStreamWaitEvent(g.s_d2h, merged[s], 0));
    const uint64_t p0 = o_lo + ch * C;
    download(g, (uint64_t*)c.B + p0, g.mout.u64() + (uint64_t)s * C, totals[ch] * 8, g.s_d2h,
             c.direct_out, (int)S().opt.get("merge_stage_threads"), acc);
    CK(cudaEventRecord(out_free[s], g.s_d2h));
  }
  flush_out(g, (int)S().opt.get("merge_stage_threads"), acc);
  CK(cudaEventRecord(em.b, g.s_d2h));
  CK(cudaStreamSynchronize(g.s_d2h));
  CK(cudaStreamSynchronize(g.s_comp));
  *t_gpu = em.ms() / 1e3;
  em.destroy();
  for (int s = 0; s < 2; ++s) {
    cudaEventDestroy(in_ready[s]);
    cudaEventDestroy(in_free[s]);
    cudaEventDestroy(merged[s]);
    cudaEventDestroy(out_free[s]);
  }
}

// STREAM mode: batches -> W (host) through per-GPU uploader/downloader threads, then the CPU
// multiway merge W -> B.
void sort_stream(std::vector<GpuCtx*>& gs, CallCtx& c) {
  const uint64_t n = c.n, b_s = c.plan.b_s, n_b = c.plan.n_b;
  const int n_s = std::max(1, c.plan.n_s);
  const bool pipelined = S().opt.get("pipeline") != 0;
  // PIPEMERGE: m pair-wise merges of sorted batches (2j, 2j+1), j < m, run on the
  // host threads while the GPUs are still sorting; m = hsort_pipemerge_count (reading A-9), so the
  // last pair (n_b even) or the last batch (n_b odd) is never pre-merged, only full b_s batches
  // are paired, and merged outputs are never merged again.
  const uint64_t m_pipe = (pipelined && S().opt.get("pipemerge") != 0 && n_b >= 3)
                              ? hsort_pipemerge_count(n_b, (int)gs.size()) : 0;
  // W: working memory for the sorted sublists; transformed uint64 keys.
  // Pinned and cached across calls when possible (runs then DMA straight into W and the GPU merge
  // share streams straight out of it); pageable mmap otherwise.  With PIPEMERGE, W has a 2 b_s
  // spare region in front: batch i lands at Wb + i b_s (Wb = W + 2 b_s) and pair merge j writes
  // W[2j b_s, (2j+2) b_s) — the spare for j = 0, else the inputs of pair j-1, already consumed
  // because the pair merges run one after another.
  const uint64_t spare = m_pipe ? 2 * b_s : 0;
  const uint64_t wn = n + spare;
  bool w_direct = false;
  uint64_t* W = acquire_w(wn * 8, &w_direct, &c.st->t_host_alloc);
  struct WRelease {
    ~WRelease() {
      if (S().opt.get("w_cache") == 0) release_w();
    }
  } w_release;
  uint64_t* const Wb = W + spare;

  std::atomic<uint64_t> next_batch{0};
  std::mutex err_m;
  std::string err_msg;
  int err_code = 0;
  std::atomic<bool> failed{false};
  std::mutex pm_m;  // PIPEMERGE: which batches have landed in W
  std::condition_variable pm_cv;
  std::vector<uint8_t> landed(m_pipe ? n_b : 0, 0);
  auto fail = [&](int code, const std::string& m) {
    {
      std::lock_guard<std::mutex> gd(err_m);
      if (!err_code) {
        err_code = code;
        err_msg = m;
      }
      failed = true;
    }
    { std::lock_guard<std::mutex> gd(pm_m); }
    pm_cv.notify_all();
  };
  auto mark_landed = [&](uint64_t i) {
    if (!m_pipe) return;
    {
      std::lock_guard<std::mutex> gd(pm_m);
      landed[i] = 1;
    }
    pm_cv.notify_all();
  };
  struct PerGpu {
    Acc up, down;
    double t_h2d = 0, t_sort = 0, t_d2h = 0;
    int passes = 0;
  };
  std::vector<PerGpu> pg(gs.size());
  auto t0 = Clock::now();

  auto gpu_main = [&](size_t gi) {
    GpuCtx& g = *gs[gi];
    PerGpu& P = pg[gi];
    try {
      CK(cudaSetDevice(g.dev));
      g.runs.reserve((uint64_t)n_s * b_s * 8);
      g.alt.reserve(b_s * 8);
      std::vector<cudaEvent_t> ev_up(n_s), ev_sorted(n_s);
      for (int s = 0; s < n_s; ++s) {
        CK(cudaEventCreateWithFlags(&ev_up[s], cudaEventDisableTiming));
        CK(cudaEventCreateWithFlags(&ev_sorted[s], cudaEventDisableTiming));
      }
      struct Item {
        uint64_t batch;
        int slot;
        EvPair eh, es, ed;
      };
      std::deque<Item*> fifo;
      std::vector<Item*> all;
      std::mutex m;
      std::condition_variable cv;
      bool up_done = false;
      std::vector<int> slot_busy(n_s, 0);
      if (!pipelined) {
        // BLINEMULTI: blocking, one stream, no overlap
        while (!failed) {
          uint64_t i = next_batch.fetch_add(1);
          if (i >= n_b) break;
          uint64_t o = i * b_s, len = std::min(b_s, n - o);
          Item* it = new Item{i, 0, {}, {}, {}};
          all.push_back(it);
          it->eh.make();
          it->es.make();
          it->ed.make();
          CK(cudaEventRecord(it->eh.a, g.s_comp));
          upload(g, g.runs.p, (const char*)c.A + o * 8, len * 8, g.s_comp, c.direct_in, c.mc_threads, P.up);
          CK(cudaEventRecord(it->eh.b, g.s_comp));
          CK(cudaEventRecord(it->es.a, g.s_comp));
          CK(radix_sort(g.rs, g.runs.u64(), g.runs.u64(), g.alt.u64(), len, c.f64, false, g.s_comp));
          CK(cudaEventRecord(it->es.b, g.s_comp));
          CK(cudaEventRecord(it->ed.a, g.s_comp));
          download(g, Wb + o, g.runs.p, len * 8, g.s_comp, w_direct, c.mc_threads, P.down);
          CK(cudaEventRecord(it->ed.b, g.s_comp));
          CK(cudaStreamSynchronize(g.s_comp));
          P.passes += g.rs.h_plan->num_active;
        }
      } else {
        std::thread downloader([&] {
          try {
            CK(cudaSetDevice(g.dev));
            while (true) {
              Item* it;
              {
                std::unique_lock<std::mutex> lk(m);
                cv.wait(lk, [&] { return !fifo.empty() || up_done || failed; });
                if (fifo.empty()) break;
                it = fifo.front();
                fifo.pop_front();
              }
              uint64_t o = it->batch * b_s, len = std::min(b_s, n - o);
              CK(cudaStreamWaitEvent(g.s_d2h, ev_sorted[it->slot], 0));
              CK(cudaEventRecord(it->ed.a, g.s_d2h));
              download(g, Wb + o, g.runs.u64() + (uint64_t)it->slot * b_s, len * 8, g.s_d2h, w_direct,
                       c.mc_threads, P.down);
              CK(cudaEventRecord(it->ed.b, g.s_d2h));
              CK(cudaEventSynchronize(it->ed.b));
              mark_landed(it->batch);
              {
                std::lock_guard<std::mutex> gd(m);
                slot_busy[it->slot] = 0;
              }
              cv.notify_all();
            }
          } catch (const HsortError& e) {
            fail(e.code, e.what());
          } catch (const std::exception& e) {
            fail(HSORT_ERR_INTERNAL, e.what());
          } catch (...) {
            fail(HSORT_ERR_INTERNAL, "unknown exception in the downloader");
          }
          // `failed` is set; take m before notifying so an uploader between its predicate check
          // and its wait cannot miss the wakeup
          { std::lock_guard<std::mutex> gd(m); }
          cv.notify_all();
        });
        uint64_t local = 0;
        try {
          while (!failed) {
            uint64_t i = next_batch.fetch_add(1);
            if (i >= n_b) break;
            int s = (int)(local++ % n_s);
            {
              std::unique_lock<std::mutex> lk(m);
              cv.wait(lk, [&] { return !slot_busy[s] || failed; });
              if (failed) break;
              slot_busy[s] = 1;
            }
            uint64_t o = i * b_s, len = std::min(b_s, n - o);
            Item* it = new Item{i, s, {}, {}, {}};
            all.push_back(it);
            it->eh.make();
            it->es.make();
            it->ed.make();
            uint64_t* dslot = g.runs.u64() + (uint64_t)s * b_s;
            CK(cudaEventRecord(it->eh.a, g.s_h2d));
            upload(g, dslot, (const char*)c.A + o * 8, len * 8, g.s_h2d, c.direct_in, c.mc_threads, P.up);
            CK(cudaEventRecord(it->eh.b, g.s_h2d));
            CK(cudaStreamWaitEvent(g.s_comp, it->eh.b, 0));
            CK(cudaEventRecord(it->es.a, g.s_comp));
            CK(radix_sort(g.rs, dslot, dslot, g.alt.u64(), len, c.f64, false, g.s_comp));
            CK(cudaEventRecord(it->es.b, g.s_comp));
            CK(cudaEventRecord(ev_sorted[s], g.s_comp));
            {
              std::lock_guard<std::mutex> gd(m);
              fifo.push_back(it);
            }
            cv.notify_all();
          }
        } catch (const HsortError& e) {
          fail(e.code, e.what());
        } catch (const std::exception& e) {
          fail(HSORT_ERR_INTERNAL, e.what());
        } catch (...) {
          fail(HSORT_ERR_INTERNAL, "unknown exception in the uploader");
        }
        {
          std::lock_guard<std::mutex> gd(m);
          up_done = true;
        }
        cv.notify_all();
        downloader.join();
        CK(cudaStreamSynchronize(g.s_comp));
        P.passes += g.rs.h_plan->num_active;
      }
      CK(cudaDeviceSynchronize());
      for (Item* it : all) {
        P.t_h2d += it->eh.ms() / 1e3;
        P.t_sort += it->es.ms() / 1e3;
        P.t_d2h += it->ed.ms() / 1e3;
        it->eh.destroy();
        it->es.destroy();
        it->ed.destroy();
        delete it;
      }
      for (int s = 0; s < n_s; ++s) {
        cudaEventDestroy(ev_up[s]);
        cudaEventDestroy(ev_sorted[s]);
      }
    } catch (const HsortError& e) {
      fail(e.code, e.what());
    } catch (const std::exception& e) {
      fail(HSORT_ERR_INTERNAL, e.what());
    } catch (...) {
      fail(HSORT_ERR_INTERNAL, "unknown exception in a GPU worker");
    }
  };
  // PIPEMERGE worker: pair j as soon as batches 2j and 2j+1 are in W, one pair at a time, each
  // merge spread over the merge threads by exact co-ranks (the output stays in key form).
  double t_pipe = 0;
  uint64_t pipe_done = 0;
  const int pm_threads = (int)std::max<int64_t>(
      1, std::min<int64_t>(S().opt.get("pipemerge_threads") > 0 ? S().opt.get("pipemerge_threads")
                                                                : host_threads() / 2,
                           pipe_pool().size() + 1));
  std::thread merger;
  if (m_pipe) {
    merger = std::thread([&] {
      try {
        for (uint64_t j = 0; j < m_pipe; ++j) {
          {
            std::unique_lock<std::mutex> lk(pm_m);
            pm_cv.wait(lk, [&] { return failed.load() || (landed[2 * j] && landed[2 * j + 1]); });
            if (failed) return;
          }
          auto tm = Clock::now();
          const uint64_t* rp[2] = {Wb + 2 * j * b_s, Wb + (2 * j + 1) * b_s};
          const uint64_t rl[2] = {b_s, b_s};
          host_merge_runs_range(rp, rl, 2, 0, 2 * b_s, W + 2 * j * b_s, false, pm_threads, &pipe_pool());
          t_pipe += secs_since(tm);
          ++pipe_done;
        }
      } catch (const std::exception& e) {
        fail(HSORT_ERR_INTERNAL, e.what());
      } catch (...) {
        fail(HSORT_ERR_INTERNAL, "unknown exception in the PIPEMERGE worker");
      }
    });
  }
  if (gs.size() == 1) {
    gpu_main(0);
  } else {
    std::vector<std::thread> th;
    for (size_t gi = 0; gi < gs.size(); ++gi) th.emplace_back(gpu_main, gi);
    for (auto& t : th) t.join();
  }
  c.st->t_sort_phase = secs_since(t0);
  if (merger.joinable()) merger.join();
  if (failed) throw HsortError(err_code ? err_code : HSORT_ERR_INTERNAL, err_msg);
  c.st->pipe_merges = pipe_done;
  c.st->t_pipemerge = t_pipe;
  c.st->t_pipemerge_wait = secs_since(t0) - c.st->t_sort_phase;
  for (auto& P : pg) {
    c.st->t_h2d += P.t_h2d;
    c.st->t_gpu_sort += P.t_sort;
    c.st->t_d2h += P.t_d2h;
    c.st->t_stage += P.up.t_stage + P.down.t_stage;
    c.st->bytes_h2d += P.up.h2d;
    c.st->bytes_d2h += P.down.d2h;
    c.st->passes_run += P.passes;
  }
  // Merge with the CPU/GPU split of A12: the GPU merges output positions [0, o_f)
  // by streaming co-ranked slices of W through HBM (K4/K5), while the host threads merge
  // [o_f, n) with loser trees; f balances the two measured rates (the split cannot be
  // derived asymptotically, it must be measured).
  auto t1 = Clock::now();
  // the sublists of the final merge: m merged pairs, then the batches 2m .. n_b-1
  std::vector<const uint64_t*> run;
  std::vector<uint64_t> rlen;
  for (uint64_t j = 0; j < m_pipe; ++j) {
    run.push_back(W + 2 * j * b_s);
    rlen.push_back(2 * b_s);
  }
  for (uint64_t i = 2 * m_pipe; i < n_b; ++i) {
    run.push_back(Wb + i * b_s);
    rlen.push_back(std::min(b_s, n - i * b_s));
  }
  const int k = (int)run.size();
  c.st->merge_k = k;
  double f = 0.0;
  const int64_t fp = S().opt.get("merge_gpu_permille");
  if (k <= kMaxMergeRuns && !gs.empty()) {
    if (fp >= 0) {
      f = fp / 1000.0;
    } else {
      // GPU share is link-bound (HtoD in, DtoH out, duplex); CPU rate from the last STREAM call
      const double bw_in = c.st->t_h2d > 0 ? c.st->bytes_h2d / c.st->t_h2d : 50e9;
      const double bw_out = c.st->t_d2h > 0 ? c.st->bytes_d2h / c.st->t_d2h : 50e9;
      // The GPU share's rate from the link (0.85 of the slower direction per GPU).  Balancing
      // with the GPU share's *measured* rate of the last call was tried and converged to
      // f = 0.56 at n = 4.3e9 (2.83 s) against 2.72 s at this estimate's f = 0.8: the rates are
      // not independent -- while the CPU merge runs it slows the staging of a pageable B, so the
      // GPU share measured under contention looks slower than it is (profiles/r02p_ooc_split.txt)
      const double r_gpu = 0.85 * std::min(bw_in, bw_out) / 8.0 * gs.size();
      const double r_cpu = S().r_cpu_merge > 0 ? S().r_cpu_merge : 4e7 * host_threads();
      f = r_gpu / (r_gpu + r_cpu);
    }
  }
  const uint64_t o_f = std::min<uint64_t>(n, (uint64_t)((double)n * f));
  double t_cpu = 0;
  int cpu_code = 0;
  std::string cpu_err;
  std::thread cpu_part([&] {
    try {
      Nvtx nv("CPU merge W -> B");
      auto tc = Clock::now();
      // the CPU share runs on its own pool; while the GPU share stages DtoH chunks into a
      // pageable B it keeps `merge_stage_threads` cores free for that staging
      int mt = c.merge_threads > 0 ? c.merge_threads : host_threads();
      if (o_f > 0 && !c.direct_out)
        mt = std::max<int>(1, mt - (int)S().opt.get("merge_stage_threads") * (int)gs.size());
      host_merge_runs_range(run.data(), rlen.data(), k, o_f, n, (uint64_t*)c.B + o_f, c.f64, mt,
                            &merge_pool());
      t_cpu = secs_since(tc);
    } catch (const std::exception& e) {
      cpu_code = HSORT_ERR_INTERNAL;
      cpu_err = e.what();
    } catch (...) {
      cpu_code = HSORT_ERR_INTERNAL;
      cpu_err = "unknown exception in the CPU merge";
    }
  });
  // the GPU share [0, o_f) is cut into one range per GPU, each streamed through its own GPU
  std::vector<double> t_gpu(gs.size(), 0.0);
  std::string gpu_err;
  int gpu_code = 0;
  if (o_f > 0) {
    const std::vector<uint64_t> gr = shard_bounds(o_f, (int)gs.size(), 1);
    try {
      run_per_gpu(gs.size(), [&](size_t gi) {
        if (gr[gi + 1] > gr[gi])
          gpu_merge_from_host(*gs[gi], c, run, rlen, gr[gi], gr[gi + 1], w_direct, &t_gpu[gi]);
      });
    } catch (const HsortError& e) {
      gpu_code = e.code;
      gpu_err = e.what();
    }
  }
  cpu_part.join();
  if (gpu_code) throw HsortError(gpu_code, gpu_err);
  if (cpu_code) throw HsortError(cpu_code, cpu_err);
  if (n > o_f + (1u << 20) && t_cpu > 0) S().r_cpu_merge = (double)(n - o_f) / t_cpu;
  c.st->t_merge_cpu = t_cpu;
  c.st->t_merge_gpu = *std::max_element(t_gpu.begin(), t_gpu.end());
  c.st->t_merge_phase = secs_since(t1);
  c.st->merge_gpu_fraction = (double)o_f / (double)n;
}

void ctx_create(GpuCtx& g, int dev, const Options& opt) {
  g.dev = dev;
  CK(cudaSetDevice(dev));
  CK(cudaStreamCreateWithFlags(&g.s_h2d, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&g.s_comp, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&g.s_d2h, cudaStreamNonBlocking));
  int R = (int)std::max<int64_t>(2, opt.get("n_ring"));
  g.ring_bytes = (uint64_t)std::max<int64_t>(1 << 20, opt.get("p_s"));
  g.ring_bytes = (g.ring_bytes + 4095) & ~4095ull;
  for (int i = 0; i < R; ++i) {
    void* p = nullptr;
    CK(cudaHostAlloc(&p, g.ring_bytes, cudaHostAllocDefault));
    g.ring_in.push_back((char*)p);
    CK(cudaHostAlloc(&p, g.ring_bytes, cudaHostAllocDefault));
    g.ring_out.push_back((char*)p);
    cudaEvent_t e;
    CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    g.ev_in.push_back(e);
    CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    g.ev_out.push_back(e);
  }
  CK(radix_scratch_reserve(g.rs, kRadixTile));
}

void ctx_destroy(GpuCtx& g) {
  if (g.dev < 0) return;
  cudaSetDevice(g.dev);
  cudaDeviceSynchronize();
  for (auto p : g.ring_in) cudaFreeHost(p);
  for (auto p : g.ring_out) cudaFreeHost(p);
  for (auto e : g.ev_in) cudaEventDestroy(e);
  for (auto e : g.ev_out) cudaEventDestroy(e);
  g.runs.release();
  g.alt.release();
  g.tmp3.release();
  g.vruns.release();
  g.valt.release();
  g.vmout.release();
  g.vrptr.release();
  g.mout.release();
  g.min.release();
  g.ranks.release();
  g.off.release();
  g.coarse.release();
  g.rptr.release();
  g.part.release();
  g.bcnt.release();
  g.btot.release();
  g.bspl.release();
  g.bseg.release();
  radix_scratch_release(g.rs);
  if (g.s_h2d) cudaStreamDestroy(g.s_h2d);
  if (g.s_comp) cudaStreamDestroy(g.s_comp);
  if (g.s_d2h) cudaStreamDestroy(g.s_d2h);
  g = GpuCtx();
}

// Usable HBM per GPU context for a call on the first n_gpus contexts: free memory of its device
// shared by the call's contexts on that device (virtual GPUs, option "virtual_gpus"), plus what
// the context already holds; the minimum over the contexts.
uint64_t device_budget(const std::vector<int>& ctx) {
  uint64_t best = ~0ull;
  std::map<int, int> per_dev;
  for (int i : ctx) per_dev[S().gpus[i].dev]++;
  std::map<int, uint64_t> free_of;
  for (auto& kv : per_dev) {
    CK(cudaSetDevice(kv.first));
    size_t fr = 0, tot = 0;
    CK(cudaMemGetInfo(&fr, &tot));
    free_of[kv.first] = fr;
  }
  for (int i : ctx) {
    const GpuCtx& g = S().gpus[i];
    const uint64_t held = g.runs.cap + g.alt.cap + g.mout.cap + g.ranks.cap + g.min.cap + g.coarse.cap;
    best = std::min<uint64_t>(best, free_of[g.dev] / per_dev[g.dev] + held);
  }
  return best == ~0ull ? 0 : best;
}
uint64_t device_budget(int n_gpus) {
  std::vector<int> ctx;
  for (int i = 0; i < n_gpus; ++i) ctx.push_back(i);
  return device_budget(ctx);
}

GpuCtx& current_ctx() {
  int dev = 0;
  CK(cudaGetDevice(&dev));
  for (auto& g : S().gpus)
    if (g.dev == dev) return g;
  throw HsortError(HSORT_ERR_INVALID, "current device not managed by hsort_init");
}

int check_ready() {
  if (!S().inited) {
    g_err = "hsort_init() has not been called";
    return HSORT_ERR_NOT_INITIALIZED;
  }
  if (S().poisoned) {
    g_err = "library poisoned by an earlier CUDA error; call hsort_finalize()";
    return HSORT_ERR_CUDA;
  }
  return HSORT_OK;
}

int do_sort(const void* A, void* B, uint64_t n, uint64_t batch_elems, int n_gpus, bool f64,
            int lane = -1) {
  int rc = check_ready();
  if (rc) return rc;
  if (lane >= (int)S().gpus.size() || lane >= 64) {
    g_err = "lane must be in [0, GPU contexts)";
    return HSORT_ERR_INVALID;
  }
  BusyGuard busy(lane);
  if (!busy.ok) {
    g_err = "hsort_sort already running";
    return HSORT_ERR_BUSY;
  }
  if (n == 0) {
    t_last = hsort_stats{};
    return HSORT_OK;
  }
  if (!A || !B) {
    g_err = "null A or B with n > 0";
    return HSORT_ERR_INVALID;
  }
  if (((uintptr_t)A & 7) || ((uintptr_t)B & 7)) {
    g_err = "A and B must be 8-byte aligned";
    return HSORT_ERR_INVALID;
  }
  const uintptr_t a0 = (uintptr_t)A, b0 = (uintptr_t)B, bytes = n * 8;
  if (A != B && a0 < b0 + bytes && b0 < a0 + bytes) {
    g_err = "A and B partially overlap";
    return HSORT_ERR_INVALID;
  }
  const int vis = (int)S().gpus.size();
  if (n_gpus < 0 || n_gpus > vis) {
    g_err = "n_gpus must be in [0, " + std::to_string(vis) + "]";
    return HSORT_ERR_INVALID;
  }
  if (n_gpus == 0) n_gpus = vis;
  if (lane >= 0) n_gpus = 1;
  return guarded([&]() -> int {
    Nvtx nv("hsort_sort");
    auto t0 = Clock::now();
    std::vector<int> ctx;  // the GPU contexts this call owns
    if (lane >= 0) ctx.push_back(lane);
    else
      for (int i = 0; i < n_gpus; ++i) ctx.push_back(i);
    GpuCtx& g0 = S().gpus[ctx[0]];
    State::PlanCache& pc = S().pc[lane + 1];
    hsort_plan_t plan;
    if (pc.valid && pc.n == n && pc.b == batch_elems && pc.ng == n_gpus && pc.opt == S().opt_version) {
      plan = pc.plan;  // the buffers it needs are already held
    } else {
      const uint64_t budget = device_budget(ctx);
      plan = make_plan(n, batch_elems, n_gpus, budget, S().opt, S().peer_ok);
      pc.valid = false;
    }
    if (lane >= 0 && plan.mode == HSORT_MODE_STREAM)
      throw HsortError(HSORT_ERR_INVALID, "lane sorts keep their runs in HBM (RESIDENT/BLINE); "
                                          "STREAM (host working memory W) is not per lane");
    CK(cudaSetDevice(g0.dev));
    hsort_stats st{};
    st.n = n;
    st.b_s = plan.b_s;
    st.n_b = plan.n_b;
    st.n_gpus = plan.n_gpus;
    st.n_s = plan.n_s;
    st.mode = plan.mode;
    st.merge_k = (int)plan.n_b;
    st.t_init = S().t_init;
    CallCtx c;
    c.A = A;
    c.B = B;
    c.n = n;
    c.f64 = f64;
    c.plan = plan;
    c.direct_in = is_pinned(A, bytes);
    c.direct_out = is_pinned(B, bytes);
    // option register_host: page-lock pageable A / B for this call and DMA them directly
    // (measured ~46 GB/s to lock + ~58 GB/s to unlock prefaulted memory: slower than staging
    // through the ring unless the caller reuses its buffers -- off by default)
    struct HostReg {
      std::vector<void*> p;
      ~HostReg() {
        for (void* q : p) cudaHostUnregister(q);
        if (!p.empty()) cudaGetLastError();
      }
    } hreg;
    if (S().opt.get("register_host") == 1) {
      auto ta = Clock::now();
      auto reg = [&](const void* q, unsigned flags) {
        if (cudaHostRegister(const_cast<void*>(q), bytes, flags) == cudaSuccess) {
          hreg.p.push_back(const_cast<void*>(q));
          return true;
        }
        cudaGetLastError();
        return false;
      };
      if (!c.direct_in) c.direct_in = reg(A, A == B ? cudaHostRegisterDefault : cudaHostRegisterReadOnly);
      if (!c.direct_out) c.direct_out = A == B ? c.direct_in : reg(B, cudaHostRegisterDefault);
      st.t_host_alloc += secs_since(ta);
    }
    c.mc_threads = (int)S().opt.get("memcpy_threads");
    c.merge_threads = (int)S().opt.get("merge_threads");
    c.st = &st;
    st.direct_in = c.direct_in;
    st.direct_out = c.direct_out;
    st.t_setup = secs_since(t0);
    if (plan.mode == HSORT_MODE_BLINE) {
      sort_bline(g0, c);
    } else if (plan.mode == HSORT_MODE_RESIDENT) {
      std::vector<GpuCtx*> gs;
      for (int i = 0; i < plan.n_gpus; ++i) gs.push_back(&S().gpus[ctx[i]]);
      if (S().opt.get("msd") == 1) sort_msd(gs, c);
      else sort_resident(gs, c);
    } else {
      // in-place (B == A) is safe: W holds the runs, B is written only by the merge
      std::vector<GpuCtx*> gs;
      for (int i = 0; i < plan.n_gpus; ++i) gs.push_back(&S().gpus[i]);
      sort_stream(gs, c);
    }
    st.t_total = secs_since(t0);
    t_last = st;
    pc.plan = plan;  // succeeded: its buffers are allocated
    pc.n = n;
    pc.b = batch_elems;
    pc.ng = n_gpus;
    pc.opt = S().opt_version;
    pc.valid = true;
    return HSORT_OK;
  });
}

// Key/value host->host sort (S§8(f) #3, the [5] workload of P:743-761): BLINE on one GPU --
// HtoD of keys and values, the key/value GPUSort in place, DtoH of both.  Out-of-core pairs (a
// merge that carries values) are not built: n must fit one GPU (32 B/pair + look-back).
int do_sort_pairs(const void* A, const uint64_t* V, void* B, uint64_t* VB, uint64_t n, bool f64,
                  uint64_t batch_elems = 0, int n_gpus = 1) {
  int rc = check_ready();
  if (rc) return rc;
  BusyGuard busy;
  if (!busy.ok) {
    g_err = "hsort_sort already running";
    return HSORT_ERR_BUSY;
  }
  if (n == 0) {
    t_last = hsort_stats{};
    return HSORT_OK;
  }
  if (!A || !B || !V || !VB) {
    g_err = "null A, V, B or VB with n > 0";
    return HSORT_ERR_INVALID;
  }
  if ((((uintptr_t)A | (uintptr_t)B | (uintptr_t)V | (uintptr_t)VB) & 7) != 0) {
    g_err = "A, V, B, VB must be 8-byte aligned";
    return HSORT_ERR_INVALID;
  }
  const uint64_t bytes = n * 8;
  auto overlap = [&](const void* x, const void* y) {
    const uintptr_t a0 = (uintptr_t)x, b0 = (uintptr_t)y;
    return x != y && a0 < b0 + bytes && b0 < a0 + bytes;
  };
  if (overlap(A, B) || overlap(V, VB) || overlap(A, V) || overlap(A, VB) || overlap(B, V) ||
      overlap(B, VB) || (const void*)A == (const void*)V || (const void*)B == (const void*)VB ||
      (const void*)A == (const void*)VB || (const void*)B == (const void*)V) {
    g_err = "key and value arrays must not overlap (B == A and VB == V are allowed)";
    return HSORT_ERR_INVALID;
  }
  const int vis = (int)S().gpus.size();
  if (n_gpus < 0 || n_gpus > vis) {
    g_err = "n_gpus must be in [0, " + std::to_string(vis) + "]";
    return HSORT_ERR_INVALID;
  }
  if (n_gpus == 0) n_gpus = vis;
  if (!S().peer_ok) n_gpus = 1;
  const uint64_t auto_min = (uint64_t)std::max<int64_t>(0, S().opt.get("auto_pipeline_min"));
  const bool batched = (batch_elems > 0 && batch_elems < n) || n_gpus > 1 || n > (1ull << 30) ||
                       (batch_elems == 0 && auto_min && n >= auto_min);
  if (batched) {
    // RESIDENT key/value plan over n_gpus GPUs (S§8(f) #3 widened out of core): every batch of a
    // GPU's shard is sorted stably in HBM, then each GPU merges one range of B/VB from all runs
    // with K4 + the key/value K5 (ties in run order = input order, so the result is the unique
    // stable sort).  The runs must fit in HBM (16 B/pair); a streamed pair merge is not built.
    return guarded([&]() -> int {
      Nvtx nv("hsort_sort_pairs (resident)");
      auto t0 = Clock::now();
      const int N = n_gpus;
      const std::vector<uint64_t> sh = shard_bounds(n, N, kRadixTile);
      uint64_t smax = 0;
      for (int g = 0; g < N; ++g) smax = std::max(smax, sh[g + 1] - sh[g]);
      uint64_t b;
      int schedule;
      if (batch_elems > 0 && batch_elems < n) {
        b = std::min<uint64_t>(batch_elems, 1ull << 30);
        b += b & 1;  // 16-byte aligned batch starts (TMA tile loads of the pair sort)
        schedule = 0;
      } else {
        b = std::min<uint64_t>(1ull << 27, std::max<uint64_t>(smax / 8, kRadixTile));
        b -= b % kRadixTile;
        schedule = 1;
      }
      const uint64_t runs = resident_runs(n, N, b, schedule, nullptr);
      if (runs > (uint64_t)kMaxMergeRuns)
        throw HsortError(HSORT_ERR_INVALID, "key/value sort: more than 1024 runs; use larger batches");
      const uint64_t need = smax * 16 + b * (16 + (uint64_t)kLookbackBytesPerKey + 1) +
                            4 * (uint64_t)S().opt.get("merge_chunk") * 8 +
                            ((uint64_t)S().opt.get("device_reserve_mb") << 20);
      if (need > device_budget(N))
        throw HsortError(HSORT_ERR_INVALID,
                         "key/value sort: the runs do not fit in HBM (16 B/pair per GPU shard); "
                         "a streamed key/value merge is not built");
      hsort_stats st{};
      st.n = n;
      st.b_s = b;
      st.n_b = runs;
      st.n_gpus = N;
      st.n_s = 1;
      st.mode = HSORT_MODE_RESIDENT;
      st.merge_k = (int)runs;
      st.t_init = S().t_init;
      CallCtx c;
      c.A = A;
      c.B = B;
      c.n = n;
      c.f64 = f64;
      c.plan = hsort_plan_t{};
      c.plan.n = n;
      c.plan.b_s = b;
      c.plan.n_b = runs;
      c.plan.n_gpus = N;
      c.plan.schedule = schedule;
      c.plan.mode = HSORT_MODE_RESIDENT;
      c.direct_in = is_pinned(A, bytes);
      c.direct_out = is_pinned(B, bytes);
      c.V = V;
      c.VB = VB;
      c.direct_vin = is_pinned(V, bytes);
      c.direct_vout = is_pinned(VB, bytes);
      c.mc_threads = (int)S().opt.get("memcpy_threads");
      c.merge_threads = (int)S().opt.get("merge_threads");
      c.st = &st;
      st.direct_in = c.direct_in && c.direct_vin;
      st.direct_out = c.direct_out && c.direct_vout;
      st.t_setup = secs_since(t0);
      std::vector<GpuCtx*> gs;
      for (int i = 0; i < N; ++i) gs.push_back(&S().gpus[i]);
      sort_resident(gs, c);
      st.t_total = secs_since(t0);
      t_last = st;
      return HSORT_OK;
    });
  }
  return guarded([&]() -> int {
    auto t0 = Clock::now();
    GpuCtx& g = S().gpus[0];
    CK(cudaSetDevice(g.dev));
    hsort_stats st{};
    st.n = n;
    st.b_s = n;
    st.n_b = 1;
    st.n_gpus = 1;
    st.n_s = 1;
    st.mode = HSORT_MODE_BLINE;
    st.merge_k = 1;
    st.t_init = S().t_init;
    const bool din = is_pinned(A, bytes) && is_pinned(V, bytes);
    const bool dout = is_pinned(B, bytes) && is_pinned(VB, bytes);
    const int mc = (int)S().opt.get("memcpy_threads");
    st.direct_in = din;
    st.direct_out = dout;
    g.runs.reserve(bytes);
    g.alt.reserve(bytes);
    g.vruns.reserve(bytes);
    g.valt.reserve(bytes);
    Acc acc;
    EvPair eh, es, ed;
    eh.make();
    es.make();
    ed.make();
    CK(cudaEventRecord(eh.a, g.s_h2d));
    upload(g, g.runs.p, A, bytes, g.s_h2d, din, mc, acc);
    upload(g, g.vruns.p, V, bytes, g.s_h2d, din, mc, acc);
    CK(cudaEventRecord(eh.b, g.s_h2d));
    CK(cudaStreamWaitEvent(g.s_comp, eh.b, 0));
    CK(cudaEventRecord(es.a, g.s_comp));
    CK(radix_sort_pairs(g.rs, g.runs.u64(), g.vruns.u64(), g.runs.u64(), g.vruns.u64(), g.alt.u64(),
                        g.valt.u64(), n, f64, f64, g.s_comp));
    CK(cudaEventRecord(es.b, g.s_comp));
    CK(cudaStreamWaitEvent(g.s_d2h, es.b, 0));
    CK(cudaEventRecord(ed.a, g.s_d2h));
    download(g, B, g.runs.p, bytes, g.s_d2h, dout, mc, acc);
    download(g, VB, g.vruns.p, bytes, g.s_d2h, dout, mc, acc);
    CK(cudaEventRecord(ed.b, g.s_d2h));
    CK(cudaStreamSynchronize(g.s_d2h));
    st.t_sort_phase = secs_since(t0);
    st.t_h2d = eh.ms() / 1e3;
    st.t_gpu_sort = es.ms() / 1e3;
    st.t_d2h = ed.ms() / 1e3;
    st.t_stage = acc.t_stage;
    st.bytes_h2d = acc.h2d;
    st.bytes_d2h = acc.d2h;
    st.passes_run = g.rs.h_plan->num_active;
    st.passes_skipped = 8 - g.rs.h_plan->num_active;
    eh.destroy();
    es.destroy();
    ed.destroy();
    st.t_total = secs_since(t0);
    t_last = st;
    return HSORT_OK;
  });
}

// Other key types / orders (S§8(f) #4), host -> host on one GPU (BLINE): HtoD of the raw keys,
// encode into internal uint64 keys, the GPUSort on those, decode, DtoH.  float64 ascending keeps
// the fused path (do_sort, every mode).
int do_sort_typed(const void* A, void* B, uint64_t n, int key_type, int desc) {
  if (key_type == HSORT_KEY_F64 && !desc) return do_sort(A, B, n, 0, 1, true);
  int rc = check_ready();
  if (rc) return rc;
  if (key_type != HSORT_KEY_F64 && key_type != HSORT_KEY_F32)
    return g_err = "key_type must be HSORT_KEY_F64 or HSORT_KEY_F32", HSORT_ERR_INVALID;
  BusyGuard busy;
  if (!busy.ok) {
    g_err = "hsort_sort already running";
    return HSORT_ERR_BUSY;
  }
  if (n == 0) {
    t_last = hsort_stats{};
    return HSORT_OK;
  }
  const uint64_t es = key_type == HSORT_KEY_F64 ? 8 : 4;
  if (!A || !B) return g_err = "null A or B with n > 0", HSORT_ERR_INVALID;
  if ((((uintptr_t)A) | ((uintptr_t)B)) & (es - 1))
    return g_err = "A and B must be aligned to the key size", HSORT_ERR_INVALID;
  const uint64_t bytes = n * es;
  const uintptr_t a0 = (uintptr_t)A, b0 = (uintptr_t)B;
  if (A != B && a0 < b0 + bytes && b0 < a0 + bytes)
    return g_err = "A and B partially overlap", HSORT_ERR_INVALID;
  return guarded([&]() -> int {
    auto t0 = Clock::now();
    GpuCtx& g = S().gpus[0];
    CK(cudaSetDevice(g.dev));
    size_t fr = 0, tot = 0;
    CK(cudaMemGetInfo(&fr, &tot));
    const uint64_t held = g.runs.cap + g.alt.cap + g.mout.cap + g.tmp3.cap;
    const uint64_t need = n * 8 * 3 + ((bytes + 15) & ~15ull) + n / 2 +
                          (uint64_t)S().opt.get("device_reserve_mb") * (1ull << 20);
    if (need > fr + held)
      throw HsortError(HSORT_ERR_INVALID, "typed sort: n does not fit one GPU (BLINE only)");
    hsort_stats st{};
    st.n = n;
    st.b_s = n;
    st.n_b = 1;
    st.n_gpus = 1;
    st.n_s = 1;
    st.mode = HSORT_MODE_BLINE;
    st.merge_k = 1;
    st.t_init = S().t_init;
    const bool din = is_pinned(A, bytes), dout = is_pinned(B, bytes);
    const int mc = (int)S().opt.get("memcpy_threads");
    st.direct_in = din;
    st.direct_out = dout;
    g.runs.reserve(n * 8);
    g.alt.reserve(n * 8);
    g.tmp3.reserve(n * 8);
    g.mout.reserve((bytes + 15) & ~15ull);
    Acc acc;
    EvPair eh, es_, ed;
    eh.make();
    es_.make();
    ed.make();
    CK(cudaEventRecord(eh.a, g.s_h2d));
    upload(g, g.mout.p, A, bytes, g.s_h2d, din, mc, acc);
    CK(cudaEventRecord(eh.b, g.s_h2d));
    CK(cudaStreamWaitEvent(g.s_comp, eh.b, 0));
    CK(cudaEventRecord(es_.a, g.s_comp));
    // float64 descending: the reverse transform fused into the GPUSort (mout -> runs); else the
    // codec passes around the ascending GPUSort of internal keys
    // float32: the native 32-bit GPUSort (4-byte keys, transform fused into its first and last
    // pass); float64 descending: the reverse transform fused into the 64-bit GPUSort
    const cudaError_t fe =
        key_type == HSORT_KEY_F32
            ? radix_sort32(g.rs, (const uint32_t*)g.mout.p, (uint32_t*)g.runs.p, (uint32_t*)g.alt.p, n,
                           true, true, desc != 0, g.s_comp)
        : desc ? radix_sort_desc_f64(g.rs, g.mout.u64(), g.runs.u64(), g.alt.u64(), n, g.s_comp)
               : cudaErrorNotSupported;
    if (fe == cudaErrorNotSupported) {
      cudaGetLastError();
      CK(key_encode(g.mout.p, g.runs.u64(), n, key_type, desc != 0, g.s_comp));
      CK(radix_sort(g.rs, g.runs.u64(), g.alt.u64(), g.tmp3.u64(), n, false, false, g.s_comp));
      CK(key_decode(g.alt.u64(), g.mout.p, n, key_type, desc != 0, g.s_comp));
    } else {
      CK(fe);
    }
    const void* result = fe == cudaErrorNotSupported ? g.mout.p : g.runs.p;
    CK(cudaEventRecord(es_.b, g.s_comp));
    CK(cudaStreamWaitEvent(g.s_d2h, es_.b, 0));
    CK(cudaEventRecord(ed.a, g.s_d2h));
    download(g, B, result, bytes, g.s_d2h, dout, mc, acc);
    CK(cudaEventRecord(ed.b, g.s_d2h));
    CK(cudaStreamSynchronize(g.s_d2h));
    st.t_sort_phase = secs_since(t0);
    st.t_h2d = eh.ms() / 1e3;
    st.t_gpu_sort = es_.ms() / 1e3;
    st.t_d2h = ed.ms() / 1e3;
    st.t_stage = acc.t_stage;
    st.bytes_h2d = acc.h2d;
    st.bytes_d2h = acc.d2h;
    st.passes_run = g.rs.h_plan->num_active;
    st.passes_skipped = 8 - g.rs.h_plan->num_active;
    eh.destroy();
    es_.destroy();
    ed.destroy();
    st.t_total = secs_since(t0);
    t_last = st;
    return HSORT_OK;
  });
}

}  // namespace

// =============================================================================================
extern "C" {

const char* hsort_last_error(void) { return g_err.c_str(); }
const char* hsort_version(void) { return "hsort-b200 0.1 (sm_100a)"; }

int hsort_device_count(void) {
  int n = 0;
  if (cudaGetDeviceCount(&n) != cudaSuccess) {
    cudaGetLastError();
    return 0;
  }
  return n;
}

int hsort_init(void) {
  std::lock_guard<std::mutex> lk(S().m);
  if (S().inited) {
    g_err = "hsort_init called twice";
    return HSORT_ERR_BUSY;
  }
  return guarded([&]() -> int {
    auto t0 = Clock::now();
    int n = 0;
    cudaError_t e = cudaGetDeviceCount(&n);
    if (e != cudaSuccess || n == 0) {
      cudaGetLastError();
      throw HsortError(HSORT_ERR_CUDA, std::string("no CUDA device: ") + cudaGetErrorString(e));
    }
    S().n_physical = n;
    const int nv = (int)S().opt.get("virtual_gpus");
    const int nctx = nv > 0 ? nv : n;
    S().gpus.resize(nctx);
    try {
      for (int i = 0; i < nctx; ++i) ctx_create(S().gpus[i], i % n, S().opt);
      // the multi-GPU merge reads the other GPUs' runs by peer loads (NVLink): enable peer access
      // between every pair of distinct devices
      S().peer_ok = true;
      for (int a = 0; a < std::min(n, nctx); ++a)
        for (int b = 0; b < std::min(n, nctx); ++b) {
          if (a == b) continue;
          int can = 0;
          CK(cudaDeviceCanAccessPeer(&can, a, b));
          if (!can) {
            S().peer_ok = false;
            continue;
          }
          CK(cudaSetDevice(a));
          cudaError_t e = cudaDeviceEnablePeerAccess(b, 0);
          if (e == cudaErrorPeerAccessAlreadyEnabled) cudaGetLastError();
          else CK(e);
        }
    } catch (...) {
      for (auto& g : S().gpus) ctx_destroy(g);
      S().gpus.clear();
      throw;
    }
    host_pool();
    if (S().opt.get("kernel_timing"))
      for (auto& g : S().gpus) {
        CK(cudaSetDevice(g.dev));
        CK(radix_set_timing(g.rs, true));
      }
    S().inited = true;
    S().poisoned = false;
    S().t_init = secs_since(t0);
    return HSORT_OK;
  });
}

int hsort_finalize(void) {
  std::lock_guard<std::mutex> lk(S().m);
  release_w();
  for (auto& p : S().pc) p.valid = false;
  for (auto& g : S().gpus) ctx_destroy(g);
  S().gpus.clear();
  S().inited = false;
  S().poisoned = false;
  return HSORT_OK;
}

int hsort_sort(const double* A_host, double* B_host, uint64_t n, uint64_t batch_elems, int n_gpus) {
  return do_sort(A_host, B_host, n, batch_elems, n_gpus, true);
}

int hsort_sort_u64(const uint64_t* A_host, uint64_t* B_host, uint64_t n, uint64_t batch_elems,
                   int n_gpus) {
  return do_sort(A_host, B_host, n, batch_elems, n_gpus, false);
}

int hsort_sort_lane(int lane, const double* A_host, double* B_host, uint64_t n,
                    uint64_t batch_elems) {
  if (lane < 0) return g_err = "lane must be >= 0", HSORT_ERR_INVALID;
  return do_sort(A_host, B_host, n, batch_elems, 1, true, lane);
}

int hsort_sort_typed(const void* A_host, void* B_host, uint64_t n, int key_type, int descending) {
  return do_sort_typed(A_host, B_host, n, key_type, descending);
}

int hsort_sort_pairs(const double* A_host, const uint64_t* V_host, double* B_host, uint64_t* VB_host,
                     uint64_t n) {
  return do_sort_pairs(A_host, V_host, B_host, VB_host, n, true);
}

int hsort_sort_pairs_u64(const uint64_t* A_host, const uint64_t* V_host, uint64_t* B_host,
                         uint64_t* VB_host, uint64_t n) {
  return do_sort_pairs(A_host, V_host, B_host, VB_host, n, false);
}

int hsort_sort_pairs_ex(const void* A_host, const uint64_t* V_host, void* B_host, uint64_t* VB_host,
                        uint64_t n, uint64_t batch_elems, int n_gpus, int keys_f64) {
  return do_sort_pairs(A_host, V_host, B_host, VB_host, n, keys_f64 != 0, batch_elems, n_gpus);
}

int hsort_set_option(const char* key, int64_t value) {
  if (!key || !S().opt.v.count(key)) {
    g_err = std::string("unknown option ") + (key ? key : "(null)");
    return HSORT_ERR_INVALID;
  }
  std::string k = key;
  if (k == "virtual_gpus" && (value < 0 || value > 64))
    return g_err = "virtual_gpus in [0, 64]", HSORT_ERR_INVALID;
  if ((k == "n_s" || k == "n_ring") && value < 1) return g_err = k + " must be >= 1", HSORT_ERR_INVALID;
  if (k == "p_s" && value < (1 << 20)) return g_err = "p_s must be >= 1 MiB", HSORT_ERR_INVALID;
  if (k == "merge_chunk" && value < kMergeTile) return g_err = "merge_chunk too small", HSORT_ERR_INVALID;
  if (k == "merge_gpu_permille" && (value < -1 || value > 1000)) return g_err = "bad permille", HSORT_ERR_INVALID;
  if (k == "resident" && (value < -1 || value > 1)) return g_err = "resident in {-1,0,1}", HSORT_ERR_INVALID;
  if (k == "pin_w" && (value < -1 || value > 1)) return g_err = "pin_w in {-1,0,1}", HSORT_ERR_INVALID;
  if (S().inited && (k == "p_s" || k == "n_ring" || k == "virtual_gpus")) {
    g_err = k + " must be set before hsort_init";
    return HSORT_ERR_BUSY;
  }
  S().opt.v[k] = value;
  ++S().opt_version;
  if (k == "dde") g_dde_enabled = value != 0;
  if (k == "dde_min_n") g_dde_min_n = (uint64_t)(value < 1 ? 1 : value);
  if (k == "memcpy_nt") g_memcpy_nt = value != 0;
  if (k == "kernel_timing") {
    return guarded([&]() -> int {
      for (auto& g : S().gpus) {
        CK(cudaSetDevice(g.dev));
        CK(radix_set_timing(g.rs, value != 0));
      }
      return HSORT_OK;
    });
  }
  return HSORT_OK;
}

int hsort_get_kernel_times(float* ms, int max_entries, int* num_active_passes) {
  int rc = check_ready();
  if (rc) return rc;
  if (!ms || max_entries < 0) return g_err = "bad arguments", HSORT_ERR_INVALID;
  return guarded([&]() -> int {
    GpuCtx& g = current_ctx();
    if (num_active_passes) *num_active_passes = g.rs.h_plan ? g.rs.h_plan->num_active : 0;
    return radix_kernel_times(g.rs, ms, max_entries);
  });
}

int hsort_get_last_plan(int* num_active_passes, int* elided, uint64_t* n_outliers) {
  int rc = check_ready();
  if (rc) return rc;
  return guarded([&]() -> int {
    GpuCtx& g = current_ctx();
    const RadixPlan* P = g.rs.h_plan;
    if (num_active_passes) *num_active_passes = P ? P->num_active : 0;
    if (elided) *elided = P ? P->dde : 0;
    if (n_outliers) *n_outliers = P && P->dde ? P->dde_n_out : 0;
    return HSORT_OK;
  });
}

int hsort_get_option(const char* key, int64_t* value) {
  if (!key || !value || !S().opt.v.count(key)) {
    g_err = "unknown option";
    return HSORT_ERR_INVALID;
  }
  *value = S().opt.v[key];
  return HSORT_OK;
}

int hsort_get_stats(hsort_stats* out) {
  if (!out) return HSORT_ERR_INVALID;
  *out = t_last;
  return HSORT_OK;
}

int hsort_plan(uint64_t n, uint64_t batch_elems, int n_gpus, uint64_t device_bytes,
               hsort_plan_t* out) {
  if (!out || n_gpus < 0) {
    g_err = "bad arguments";
    return HSORT_ERR_INVALID;
  }
  return guarded([&]() -> int {
    uint64_t db = device_bytes;
    int ng = n_gpus;
    if (db == 0 || ng == 0) {
      int cnt = hsort_device_count();
      if (cnt == 0) throw HsortError(HSORT_ERR_CUDA, "no CUDA device to query");
      if (ng == 0) ng = cnt;
      if (db == 0) {
        size_t fr = 0, tot = 0;
        CK(cudaMemGetInfo(&fr, &tot));
        db = fr;
      }
    }
    *out = make_plan(n, batch_elems, ng, db, S().opt);
    return HSORT_OK;
  });
}

int hsort_sort_device(const double* d_in, double* d_out, uint64_t n, void* stream) {
  return hsort_sort_device_keys((const uint64_t*)d_in, (uint64_t*)d_out, n, 1, 1, stream);
}

int hsort_sort_device_keys(const uint64_t* d_in, uint64_t* d_out, uint64_t n, int in_f64,
                           int out_f64, void* stream) {
  int rc = check_ready();
  if (rc) return rc;
  if (n && (!d_in || !d_out)) return g_err = "null device pointer", HSORT_ERR_INVALID;
  return guarded([&]() -> int {
    GpuCtx& g = current_ctx();
    g.alt.reserve(n * 8);
    CK(radix_sort(g.rs, d_in, d_out, g.alt.u64(), n, in_f64 != 0, out_f64 != 0,
                  (cudaStream_t)stream));
    return HSORT_OK;
  });
}

int hsort_sort_device_typed(const void* d_in, void* d_out, uint64_t n, int key_type,
                            int descending, void* stream) {
  int rc = check_ready();
  if (rc) return rc;
  if (key_type != HSORT_KEY_F64 && key_type != HSORT_KEY_F32)
    return g_err = "key_type must be HSORT_KEY_F64 or HSORT_KEY_F32", HSORT_ERR_INVALID;
  if (n && (!d_in || !d_out)) return g_err = "null device pointer", HSORT_ERR_INVALID;
  if (key_type == HSORT_KEY_F64 && !descending)
    return hsort_sort_device_keys((const uint64_t*)d_in, (uint64_t*)d_out, n, 1, 1, stream);
  if ((((uintptr_t)d_in) | ((uintptr_t)d_out)) & 15)
    return g_err = "typed sort: device buffers must be 16-byte aligned", HSORT_ERR_INVALID;
  return guarded([&]() -> int {
    GpuCtx& g = current_ctx();
    cudaStream_t st = (cudaStream_t)stream;
    g.runs.reserve(n * 8);
    g.alt.reserve(n * 8);
    if (key_type == HSORT_KEY_F32) {
      // native 32-bit GPUSort; the codec path below when it does not apply
      const cudaError_t fe = radix_sort32(g.rs, (const uint32_t*)d_in, (uint32_t*)d_out,
                                          (uint32_t*)g.alt.p, n, true, true, descending != 0, st);
      if (fe != cudaErrorNotSupported) {
        CK(fe);
        return HSORT_OK;
      }
      cudaGetLastError();
    }
    if (key_type == HSORT_KEY_F64 && descending && d_in != d_out) {
      // reverse transform fused into the GPUSort's first and last pass
      const cudaError_t fe = radix_sort_desc_f64(g.rs, (const uint64_t*)d_in, (uint64_t*)d_out,
                                                 g.alt.u64(), n, st);
      if (fe != cudaErrorNotSupported) {
        CK(fe);
        return HSORT_OK;
      }
      cudaGetLastError();
    }
    g.tmp3.reserve(n * 8);
    CK(key_encode(d_in, g.runs.u64(), n, key_type, descending != 0, st));
    CK(radix_sort(g.rs, g.runs.u64(), g.alt.u64(), g.tmp3.u64(), n, false, false, st));
    CK(key_decode(g.alt.u64(), d_out, n, key_type, descending != 0, st));
    return HSORT_OK;
  });
}

int hsort_sort_device_pairs(const uint64_t* d_keys_in, const uint64_t* d_vals_in,
                            uint64_t* d_keys_out, uint64_t* d_vals_out, uint64_t n, int keys_f64,
                            void* stream) {
  int rc = check_ready();
  if (rc) return rc;
  if (n && (!d_keys_in || !d_vals_in || !d_keys_out || !d_vals_out))
    return g_err = "null device pointer", HSORT_ERR_INVALID;
  if (n > (1ull << 30)) return g_err = "key/value sort: n <= 2^30", HSORT_ERR_INVALID;
  if ((((uintptr_t)d_keys_in | (uintptr_t)d_vals_in | (uintptr_t)d_keys_out |
        (uintptr_t)d_vals_out) & 15) != 0)
    return g_err = "key/value sort: device buffers must be 16-byte aligned", HSORT_ERR_INVALID;
  if ((d_keys_in == d_keys_out) != (d_vals_in == d_vals_out))
    return g_err = "key/value sort: keys and values must both be in place or both not",
           HSORT_ERR_INVALID;
  return guarded([&]() -> int {
    GpuCtx& g = current_ctx();
    g.alt.reserve(n * 8);
    g.valt.reserve(n * 8);
    CK(radix_sort_pairs(g.rs, d_keys_in, d_vals_in, d_keys_out, d_vals_out, g.alt.u64(),
                        g.valt.u64(), n, keys_f64 != 0, keys_f64 != 0, (cudaStream_t)stream));
    return HSORT_OK;
  });
}

int hsort_device_histograms(const uint64_t* d_keys, uint64_t n, int in_f64, uint64_t* d_hist,
                            void* stream) {
  int rc = check_ready();
  if (rc) return rc;
  return guarded([&]() -> int {
    GpuCtx& g = current_ctx();
    CK(radix_histograms(g.rs, d_keys, n, in_f64 != 0, d_hist, (cudaStream_t)stream));
    CK(cudaStreamSynchronize((cudaStream_t)stream));
    return HSORT_OK;
  });
}

int hsort_device_radix_pass(const uint64_t* d_src, uint64_t* d_dst, uint64_t n, int digit,
                            void* stream) {
  int rc = check_ready();
  if (rc) return rc;
  if (digit < 0 || digit > 7) return g_err = "digit must be 0..7", HSORT_ERR_INVALID;
  if (d_src == d_dst && n) return g_err = "src and dst must differ", HSORT_ERR_INVALID;
  return guarded([&]() -> int {
    GpuCtx& g = current_ctx();
    CK(radix_one_pass(g.rs, d_src, d_dst, n, digit, (cudaStream_t)stream));
    CK(cudaStreamSynchronize((cudaStream_t)stream));
    return HSORT_OK;
  });
}

int hsort_device_corank(const uint64_t* d_keys, const uint64_t* h_off, int k, uint64_t step,
                        uint64_t n_bounds, uint64_t* d_ranks, void* stream) {
  int rc = check_ready();
  if (rc) return rc;
  if (k < 1 || k > kMaxMergeRuns || !h_off) return g_err = "k must be 1..1024", HSORT_ERR_INVALID;
  return guarded([&]() -> int {
    GpuCtx& g = current_ctx();
    g.off.reserve((k + 1) * 8);
    cudaStream_t st = (cudaStream_t)stream;
    CK(cudaMemcpyAsync(g.off.p, h_off, (k + 1) * 8, cudaMemcpyHostToDevice, st));
    corank_on(g, d_keys, nullptr, g.off.u64(), k, h_off[k] - h_off[0], step, 0, n_bounds, d_ranks, st);
    CK(cudaStreamSynchronize(st));
    return HSORT_OK;
  });
}

int hsort_device_merge(const uint64_t* d_keys, const uint64_t* h_off, int k, uint64_t* d_out,
                       int out_f64, void* stream) {
  int rc = check_ready();
  if (rc) return rc;
  if (k < 1 || k > kMaxMergeRuns || !h_off) return g_err = "k must be 1..1024", HSORT_ERR_INVALID;
  return guarded([&]() -> int {
    GpuCtx& g = current_ctx();
    cudaStream_t st = (cudaStream_t)stream;
    const uint64_t total = h_off[k] - h_off[0];
    if (total == 0) return HSORT_OK;
    g.off.reserve((k + 1) * 8);
    CK(cudaMemcpyAsync(g.off.p, h_off, (k + 1) * 8, cudaMemcpyHostToDevice, st));
    const uint64_t tiles = (total + kMergeTile - 1) / kMergeTile;
    g.ranks.reserve((tiles + 1) * (uint64_t)k * 8);
    corank_on(g, d_keys, nullptr, g.off.u64(), k, total, kMergeTile, 0, tiles + 1, g.ranks.u64(), st);
    CK(merge_tiles(d_keys, nullptr, g.off.u64(), k, total, g.ranks.u64(), 0, 0, tiles, d_out, 0,
                   out_f64 != 0, st));
    CK(cudaStreamSynchronize(st));
    return HSORT_OK;
  });
}

int hsort_device_upper_bounds(const uint64_t* d_keys, uint64_t n, const uint64_t* d_values,
                              uint64_t m, uint64_t* d_out, void* stream) {
  int rc = check_ready();
  if (rc) return rc;
  if (m && (!d_values || !d_out || (n && !d_keys))) return g_err = "null pointer", HSORT_ERR_INVALID;
  return guarded([&]() -> int {
    cudaStream_t st = (cudaStream_t)stream;
    CK(upper_bounds(d_keys, n, d_values, m, d_out, st));
    CK(cudaStreamSynchronize(st));
    return HSORT_OK;
  });
}

int hsort_host_upper_bounds(const uint64_t* keys, uint64_t n, const uint64_t* values, uint64_t m,
                            uint64_t* out) {
  if (m && (!values || !out || (n && !keys))) return g_err = "null pointer", HSORT_ERR_INVALID;
  for (uint64_t i = 0; i < m; ++i) {
    uint64_t lo = 0, hi = n;
    while (lo < hi) {
      const uint64_t mid = lo + ((hi - lo) >> 1);
      if (keys[mid] <= values[i]) lo = mid + 1;
      else hi = mid;
    }
    out[i] = lo;
  }
  return HSORT_OK;
}

int hsort_par_memcpy(void* dst, const void* src, uint64_t bytes, int threads) {
  if (bytes && (!dst || !src)) return g_err = "null pointer", HSORT_ERR_INVALID;
  return guarded([&]() -> int {
    par_memcpy(dst, src, bytes, threads > 0 ? threads : (int)S().opt.get("memcpy_threads"));
    return HSORT_OK;
  });
}

int hsort_host_merge(const uint64_t* keys, const uint64_t* off, int k, uint64_t* out, int out_f64,
                     int threads) {
  if (k < 1 || !off || (off[k] > off[0] && (!keys || !out)))
    return g_err = "bad arguments", HSORT_ERR_INVALID;
  for (int j = 0; j < k; ++j)
    if (off[j + 1] < off[j]) return g_err = "offsets must be non-decreasing", HSORT_ERR_INVALID;
  return guarded([&]() -> int {
    host_merge(keys, off, k, out, out_f64 != 0, threads > 0 ? threads : (int)S().opt.get("merge_threads"));
    return HSORT_OK;
  });
}

int hsort_host_corank(const uint64_t* keys, const uint64_t* off, int k, uint64_t o,
                      uint64_t* ranks) {
  if (k < 1 || !off || !ranks) return g_err = "bad arguments", HSORT_ERR_INVALID;
  return guarded([&]() -> int {
    std::vector<uint64_t> o2(k + 1);
    for (int j = 0; j <= k; ++j) o2[j] = off[j] - off[0];
    host_corank(keys + off[0], o2.data(), k, o, ranks);
    return HSORT_OK;
  });
}

uint64_t hsort_get_launch_count(void) { return g_kernel_launches.load(); }

int hsort_sample_positions(uint64_t n, uint64_t s, uint64_t* pos) {
  // regular samples of a sorted run of n keys: positions (i + 1) n / (s + 1), i < s (A13)
  if (s && !pos) return g_err = "null pos", HSORT_ERR_INVALID;
  if (n == 0) return s ? (g_err = "n = 0 has no samples", HSORT_ERR_INVALID) : HSORT_OK;
  for (uint64_t i = 0; i < s; ++i) {
    const uint64_t p = (uint64_t)((unsigned __int128)(i + 1) * n / (s + 1));
    pos[i] = p < n ? p : n - 1;
  }
  return HSORT_OK;
}

int hsort_select_splitters(const uint64_t* samples, uint64_t m, int P, uint64_t* spl) {
  // P - 1 splitters at the P-quantiles of the m merged samples: spl[r - 1] = samples[r m / P]
  if (P < 1 || (P > 1 && (!spl || (m && !samples)))) return g_err = "bad arguments", HSORT_ERR_INVALID;
  for (int r = 1; r < P; ++r)
    spl[r - 1] = m ? samples[(uint64_t)((unsigned __int128)r * m / (unsigned)P)] : 0;
  return HSORT_OK;
}

uint64_t hsort_pipemerge_count(uint64_t n_b, int n_gpus) {
  // P:430-454 (reading A-9): one GPU -> floor((n_b-1)/2); two or more -> floor(n_b/(2 n_GPU))
  if (n_b == 0) return 0;
  if (n_gpus <= 1) return (n_b - 1) / 2;
  return n_b / (2 * (uint64_t)n_gpus);
}

}  // extern "C"
