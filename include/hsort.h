/* include/hsort.h — C ABI of the B200-native heterogeneous float64 sort.
 *
 * The problem (§I): "given an unsorted input list, A, of n elements in main
 * memory, generate a sorted output list, B, using the CPUs and GPU(s) on the platform".
 * The method (§III): split A into n_b batches of b_s elements, sort each
 * batch on the GPU, merge the sorted batches with a multiway merge,
 * pipelining transfers through pinned staging buffers on CUDA streams (PIPEDATA) with
 * parallel host copies (PARMEMCPY).  Table I names the parameters
 * n, n_b, n_GPU, n_s, b_s, p_s used below.
 *
 * Result contract (readings A-1..A-4): B holds A's 64-bit patterns permuted into
 * ascending IEEE 754 totalOrder (-NaNs < -inf < ... < -0 < +0 < ... < +inf < +NaNs).  No
 * floating-point arithmetic touches a key; NaN payloads and the sign of zero are preserved.
 * Equal keys are bit-identical, so the output is unique and checked bit-exactly.
 *
 * Conventions
 *  - Every function returns HSORT_OK (0) or a negative hsort_status; none throws.
 *  - hsort_last_error() returns a thread-local message for the last failing call.
 *  - After a CUDA error the library is poisoned: later calls return HSORT_ERR_CUDA until
 *    hsort_finalize().  B's contents are unspecified after an error; A is never written
 *    unless B == A.
 *  - The library is not re-entrant: a concurrent hsort_sort returns HSORT_ERR_BUSY (except
 *    hsort_sort_lane calls on different lanes, which may run concurrently).
 *  - "host" pointers may be pageable or pinned (cudaHostAlloc / cudaHostRegister); pinned
 *    buffers are DMA'd directly, pageable ones go through the pinned staging ring (Stage, MCpy).
 *  - "device" pointers are CUDA global memory on the CURRENT device; "stream" is a cudaStream_t
 *    (NULL = legacy default stream).  Device entry points are asynchronous on that stream
 *    unless stated otherwise.
 */
#ifndef HSORT_H_
#define HSORT_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  HSORT_OK = 0,
  HSORT_ERR_INVALID = -1,          /* bad argument (null with n > 0, partial overlap, n_gpus) */
  HSORT_ERR_NOT_INITIALIZED = -2,  /* hsort_init() not called */
  HSORT_ERR_HOST_OOM = -3,         /* host allocation (W, pinned ring) failed */
  HSORT_ERR_DEVICE_OOM = -4,       /* device allocation failed */
  HSORT_ERR_CUDA = -5,             /* CUDA runtime error (library poisoned until finalize) */
  HSORT_ERR_NCCL = -6,             /* reserved, never returned: the in-library multi-GPU exchange
                                      uses peer loads over NVLink, not NCCL */
  HSORT_ERR_BUSY = -7,             /* concurrent call, or hsort_init twice */
  HSORT_ERR_INTERNAL = -8          /* invariant violated inside the library */
} hsort_status;

/* Merge/placement mode chosen by the planner (A1) for one hsort_sort call. */
typedef enum {
  HSORT_MODE_BLINE = 0,     /* n_b = 1: A -> HtoD -> GPUSort -> DtoH -> B */
  HSORT_MODE_RESIDENT = 1,  /* n_b > 1, sorted runs stay in HBM, GPU merge-path merge, DtoH of
                               merged chunks overlapped with the merge (B200 design) */
  HSORT_MODE_STREAM = 2     /* n_b > 1, runs go to host working memory W, multiway merge on the
                               CPU (+ optional GPU share f): PIPEDATA / BLINEMULTI */
} hsort_mode;

/* Per-call statistics (the paper reports per-component response times). Seconds are
 * host wall-clock (steady_clock) unless marked "device". */
typedef struct hsort_stats {
  uint64_t n;              /* keys sorted */
  uint64_t b_s;            /* batch size (elements) */
  uint64_t n_b;            /* number of batches = ceil(n / b_s) */
  int32_t n_gpus;          /* GPUs used */
  int32_t n_s;             /* batch slots in flight per GPU (streams) */
  int32_t mode;            /* hsort_mode */
  int32_t passes_run;      /* radix digit passes run, summed over batches */
  int32_t passes_skipped;  /* trivial digit passes skipped (one non-empty bin), summed */
  int32_t direct_in;       /* 1 if A was DMA'd directly (pinned), 0 if staged */
  int32_t direct_out;      /* 1 if B was written directly by DMA (pinned), 0 if staged */
  int32_t merge_k;         /* runs merged (= n_b) */
  double merge_gpu_fraction; /* share f of merge output produced by GPUs (A12) */
  double t_total;          /* whole hsort_sort call */
  double t_sort_phase;     /* from first HtoD to last run sorted (and, STREAM, landed in W) */
  double t_merge_phase;    /* merge (+ its DtoH) after the sort phase */
  double t_gpu_sort;       /* device: sum of GPUSort (K1+K2+K3) over batches (CUDA events) */
  double t_h2d;            /* device: sum of HtoD copy time (CUDA events) */
  double t_d2h;            /* device: sum of DtoH copy time (CUDA events) */
  double t_stage;          /* host: sum of MCpy time into/out of pinned staging */
  double t_merge_cpu;      /* host: CPU multiway merge time */
  double t_merge_gpu;      /* device: GPU merge kernels (K4+K5) */
  double t_init;           /* hsort_init() duration (pinned + device allocation) */
  uint64_t bytes_h2d;      /* bytes moved host -> device */
  uint64_t bytes_d2h;      /* bytes moved device -> host */
  double t_host_alloc;     /* pinned working-memory (W) allocation in this call (cached after) */
  uint64_t pipe_merges;    /* STREAM PIPEMERGE: pair-wise merges done during the sort phase */
  double t_pipemerge;      /* host: time spent in those pair-wise merges */
  double t_pipemerge_wait; /* host: wait after the sort phase for the last pair merge (P:422-425
                              wants 0: pair merges must not delay the final multiway merge) */
  int32_t msd_buckets;     /* MSD-first split (option "msd"): key-range buckets R; 0 = merge path */
  int32_t reserved0;
  double t_setup;          /* host: planning before the first copy (HBM query, plan, pointer checks) */
} hsort_stats;

/* Planner output (A1).  Pure host arithmetic; see hsort_plan(). */
typedef struct hsort_plan_t {
  uint64_t n, b_s, n_b;
  int32_t n_gpus, n_s, mode;
  uint64_t last_batch;            /* size of the ragged last batch (reading A-12) */
  uint64_t device_bytes_per_gpu;  /* predicted device footprint */
  uint64_t host_bytes;            /* predicted host working memory (W + staging) */
  double batches_per_stream;      /* n_b / (n_s * n_GPU) */
  int32_t schedule;               /* 0: uniform b_s batches; 1: b_s batches + halving tail
                                     (auto RESIDENT plan: the last batch's sort is the only one
                                     not hidden behind an HtoD) */
} hsort_plan_t;

/* ---------------------------------------------------------------------------------------------
 * Lifecycle
 * ------------------------------------------------------------------------------------------- */

/* Enumerate GPUs; create per-GPU streams (H2D / compute / D2H) and the pinned staging ring
 * (n_ring slots of p_s bytes per GPU and direction; P:331-334 — pinned memory is expensive to
 * allocate, so it is done once here).  Device batch buffers are allocated lazily by
 * the first hsort_sort and cached.  A second call before hsort_finalize -> HSORT_ERR_BUSY. */
int hsort_init(void);

/* Free every library-owned resource.  Safe after errors and when not initialised. */
int hsort_finalize(void);

/* ---------------------------------------------------------------------------------------------
 * The sort (host -> host).  Synchronous; retains no pointer.
 *   A_host       n float64, 8-byte aligned host memory, read-only (unless B == A).
 *   B_host       n float64 writable host memory; B == A allowed (in place); partial overlap of
 *                A and B -> HSORT_ERR_INVALID.
 *   n            number of keys; 0 -> HSORT_OK, no-op.
 *   batch_elems  b_s; > n -> clamped to n; n_b = ceil(n / b_s).  0 -> auto: if n >= option
 *                "auto_pipeline_min" (2^24) and the runs fit in HBM, a pipelined RESIDENT
 *                schedule (b_s = min(2^27, n/8) batches + halving tail); else one batch if it
 *                fits (BLINE), else the largest b_s filling HBM.
 *   n_gpus       1..visible devices; 0 -> all visible; > visible -> HSORT_ERR_INVALID.
 * ------------------------------------------------------------------------------------------- */
int hsort_sort(const double* A_host, double* B_host, uint64_t n, uint64_t batch_elems, int n_gpus);

/* Same, on raw uint64 keys (ascending unsigned order; no key transform). */
int hsort_sort_u64(const uint64_t* A_host, uint64_t* B_host, uint64_t n, uint64_t batch_elems,
                   int n_gpus);

/* Concurrent sorts (serving): hsort_sort on GPU context `lane` alone (0 <= lane < contexts: the
 * visible devices, or option "virtual_gpus").  Calls on different lanes may run at the same time
 * from different host threads -- on one GPU their HtoD and DtoH overlap, which one sort cannot do
 * (its first output key depends on its last input key).  The runs must fit in the lane's HBM
 * (RESIDENT or BLINE plans; a STREAM plan -> HSORT_ERR_INVALID).  A call on a busy lane, or while
 * an hsort_sort/hsort_sort_pairs/hsort_sort_typed call runs, -> HSORT_ERR_BUSY (and vice versa).
 * Arguments as hsort_sort. */
int hsort_sort_lane(int lane, const double* A_host, double* B_host, uint64_t n,
                    uint64_t batch_elems);

/* ---------------------------------------------------------------------------------------------
 * Other key types and orders.  key_type HSORT_KEY_F64 (8-byte float64) or
 * HSORT_KEY_F32 (4-byte float32); descending != 0 sorts by the reverse of IEEE totalOrder (the
 * exact reverse of the ascending result: every totalOrder class is one bit pattern).  Keys are
 * sorted as bit patterns (NaN payloads and -0.0 preserved).  float64 ascending is hsort_sort
 * (every mode); every other combination runs on one GPU as one batch (BLINE): float32 on the
 * native 32-bit GPUSort (binary32 key transform fused into its first/last pass, <= 4 passes; the
 * 64-bit codec path below for n > 2^30), float64 descending with the reverse transform fused into
 * the 64-bit GPUSort, else an encode pass to 64-bit internal keys, the GPUSort, a decode pass.
 * n must fit one GPU (24 B/key + the key array), else
 * HSORT_ERR_INVALID.  A and B aligned to the key size; B == A allowed; partial overlap -> INVALID.
 * ------------------------------------------------------------------------------------------- */
#define HSORT_KEY_F64 0
#define HSORT_KEY_F32 1
int hsort_sort_typed(const void* A_host, void* B_host, uint64_t n, int key_type, int descending);

/* ---------------------------------------------------------------------------------------------
 * Key/value sort (the [5] workload of 64-bit keys with 64-bit values,
 * P:743-761).  B/VB = the pairs (A[i], V[i]) ordered by A under IEEE totalOrder, STABLY: pairs
 * with equal keys keep their input order, so the result is unique (V = 0..n-1 gives the stable
 * argsort).  Values are opaque 64-bit payloads, never transformed.  n < 2^24 (option
 * "auto_pipeline_min"): one GPU, one batch (BLINE; 32.5 B/pair of HBM); larger n: the RESIDENT
 * key/value plan of hsort_sort_pairs_ex on GPU 0 (runs in HBM, key/value merge; n beyond one GPU's
 * HBM -> HSORT_ERR_INVALID).  B == A and VB == V allowed together or separately; any
 * other overlap among A, V, B, VB -> HSORT_ERR_INVALID.  Synchronous; retains no pointer.
 * ------------------------------------------------------------------------------------------- */
int hsort_sort_pairs(const double* A_host, const uint64_t* V_host, double* B_host, uint64_t* VB_host,
                     uint64_t n);
/* Same with raw uint64 keys (ascending unsigned). */
int hsort_sort_pairs_u64(const uint64_t* A_host, const uint64_t* V_host, uint64_t* B_host,
                         uint64_t* VB_host, uint64_t n);
/* Key/value sort with the batch size and GPU count of hsort_sort (keys_f64: 1 float64 keys under
 * totalOrder, 0 raw uint64 keys).  batch_elems = 0 and n < option "auto_pipeline_min" (2^24):
 * one batch on one GPU as above; otherwise (or batch_elems < n, n_gpus > 1, n > 2^30) the RESIDENT
 * plan: GPU g stably sorts the batches of its shard of the pairs in HBM (key/value GPUSort) and
 * merges one range of B/VB from all GPUs' runs (K4 on the keys, the key/value K5, equal keys in run
 * order), so the result is the same unique stable sort.  The runs must fit in HBM (16 B/pair per
 * shard + one batch of scratch), else HSORT_ERR_INVALID; a streamed (W) key/value merge is not
 * built.  Aliasing and errors as hsort_sort_pairs. */
int hsort_sort_pairs_ex(const void* A_host, const uint64_t* V_host, void* B_host, uint64_t* VB_host,
                        uint64_t n, uint64_t batch_elems, int n_gpus, int keys_f64);

/* ---------------------------------------------------------------------------------------------
 * Options, statistics, errors
 *   keys: "n_s" (batch slots per GPU, default 3), "p_s" (pinned staging chunk bytes),
 *         "n_ring" (pinned slots per direction), "memcpy_threads" (PARMEMCPY threads; 1 = serial
 *         MCpy), "merge_threads" (CPU merge threads), "resident" (-1 auto, 0 force
 *         STREAM, 1 force RESIDENT), "merge_gpu_permille" (A12 share f in 1/1000; -1 auto),
 *         "pipeline" (1 = overlapped streams PIPEDATA, 0 = blocking BLINEMULTI ablation),
 *         "pipemerge" (STREAM mode with pipeline = 1: 1 = PIPEMERGE pair-wise merges of sorted
 *         batches on the host threads while the GPUs sort, hsort_pipemerge_count(n_b, n_gpus)
 *         of them; 0 = off (default: slower on a B200 box), the final
 *         merge takes all n_b runs), "pipemerge_threads"
 *         (host threads for those pair merges, on their own pool; 0 = half the hardware threads),
 *         "merge_chunk" (GPU merge output chunk elements), "device_reserve_mb" (HBM left free),
 *         "kernel_timing" (1 = CUDA events around each radix kernel, see hsort_get_kernel_times),
 *         "auto_pipeline_min" (smallest n for the auto pipelined RESIDENT plan; 0 = never),
 *         "pin_w" (STREAM-mode W: 1 cached pinned, 0 pageable + staging, -1 auto = pinned up to
 *         "pin_w_max_mb" (default 2^20 MB) or when a large enough pinned W is already cached),
 *         "w_cache" (1 = keep W allocated, prefaulted and locked across calls),
 *         "dde" (1 = dominant-digit elision in the GPUSort: when the top active digit has one
 *         value held by all but a few keys, its LSD pass is dropped and the outliers are sorted
 *         separately; output-invisible; 0 = off), "dde_min_n" (smallest n it is tried at),
 *         "memcpy_nt" (1 = PARMEMCPY with non-temporal stores),
 *         "merge_stage_threads" (STREAM merge: host threads per GPU that stage the GPU share's
 *         DtoH into a pageable B), "defer_out_drain" (1 = those staged copy-outs drained lazily
 *         across merge chunks, so the next chunk's DMA starts at once),
 *         "register_host" (1 = page-lock pageable A / B for the call and DMA them directly),
 *         "msd" (1 = RESIDENT plans use the MSD-first bucket split), "msd_bucket_keys",
 *         "virtual_gpus" (set before hsort_init: that many GPU contexts, mapped round-robin onto
 *         the visible devices; the lanes of hsort_sort_lane and multi-GPU tests on one device).
 * ------------------------------------------------------------------------------------------- */
int hsort_set_option(const char* key, int64_t value);
int hsort_get_option(const char* key, int64_t* value);
int hsort_get_stats(hsort_stats* out);      /* stats of the calling thread's last successful sort */
const char* hsort_last_error(void);          /* thread-local; never NULL */
const char* hsort_version(void);

/* Per-kernel device durations of the last GPUSort on the current device, recorded with CUDA
 * events on the sort's stream when option "kernel_timing" = 1 (used by bench.py for the
 * roofline).  ms[0] = K1 histograms, ms[1] = K2 scan/plan, ms[2+p] = K3 pass p (p = 0..7; passes
 * p >= *num_active_passes are empty launches), ms[10] = final copy.  Returns the number of
 * entries written (>= 0) or a negative hsort_status.  Call after synchronising the stream. */
int hsort_get_kernel_times(float* ms, int max_entries, int* num_active_passes);

/* Plan of the last GPUSort on the current device (after synchronising its stream): active LSD
 * passes run, whether the dominant-digit elision dropped the top digit's pass (option "dde"), and
 * how many outlier keys it sorted separately. */
int hsort_get_last_plan(int* num_active_passes, int* elided, uint64_t* n_outliers);

/* Planner (A1): pure host arithmetic, no GPU needed.  device_bytes = usable HBM per GPU
 * (0 -> query the current device).  Fills *out; HSORT_ERR_INVALID on bad arguments. */
int hsort_plan(uint64_t n, uint64_t batch_elems, int n_gpus, uint64_t device_bytes,
               hsort_plan_t* out);

/* ---------------------------------------------------------------------------------------------
 * Device-resident entry points (current device, library-owned scratch; stream-ordered).
 * The scratch (histograms, plan, look-back words, ping-pong buffers) is one per device: calls on
 * one device must be ordered -- issue them from one thread on one stream, or synchronise between
 * streams.  Concurrent calls on different devices are independent.
 * ------------------------------------------------------------------------------------------- */

/* GPUSort of one batch, device -> device:  d_out = totalOrder-sorted d_in.
 * d_in == d_out allowed.  Runs K1 (digit histograms) + K2 (bin scan / pass plan) + up to 8
 * K3 onesweep passes; trivial digits are skipped on the device.  Requires hsort_init().
 * Stream-ordered, except that an out-of-place sort of n >= 2^22 keys waits once on `stream`
 * after K2 (~10 us) to read the plan: if the top active digit has a dominant value (option
 * "dde"), the host launches one pass fewer plus the outlier sort.  That wait
 * makes such a call not capturable into a CUDA graph: set option "dde" = 0 before capturing. */
int hsort_sort_device(const double* d_in, double* d_out, uint64_t n, void* stream);

/* Same, keys already uint64 (ascending unsigned); in_f64/out_f64 select whether the input is
 * float64 bits (key transform fused into the first pass) and whether the output is stored as
 * float64 bits (inverse transform fused into the last pass). */
int hsort_sort_device_keys(const uint64_t* d_in, uint64_t* d_out, uint64_t n, int in_f64,
                           int out_f64, void* stream);

/* Typed GPUSort, device -> device (current device, stream-ordered): key_type / descending as for
 * hsort_sort_typed.  float64 ascending = hsort_sort_device; otherwise encode -> GPUSort -> decode
 * (16-byte aligned buffers; d_in == d_out allowed; library scratch 24 B/key). */
int hsort_sort_device_typed(const void* d_in, void* d_out, uint64_t n, int key_type,
                            int descending, void* stream);

/* Key/value GPUSort, device -> device (current device, stream-ordered): (d_keys_out,
 * d_vals_out) = the pairs stably sorted by key (float64 totalOrder bits in and out if keys_f64,
 * else ascending uint64).  n <= 2^30; all four buffers 16-byte aligned (TMA tile loads); keys in
 * place iff values in place.  Same K1/K2 as hsort_sort_device, then the key/value onesweep pass
 * (4160-pair tiles) per active digit: 32 HBM bytes per pair per pass. */
int hsort_sort_device_pairs(const uint64_t* d_keys_in, const uint64_t* d_vals_in,
                            uint64_t* d_keys_out, uint64_t* d_vals_out, uint64_t n, int keys_f64,
                            void* stream);

/* K1 alone: d_hist[8*256] (uint64, device) = per-digit histograms of the keys (digit d =
 * bits [8d, 8d+8) of key(x) if in_f64 else of the raw uint64).  Synchronous. */
int hsort_device_histograms(const uint64_t* d_keys, uint64_t n, int in_f64, uint64_t* d_hist,
                            void* stream);

/* K3 alone: one stable LSD counting-sort pass by digit `digit` (0..7) of raw uint64 keys,
 * d_src -> d_dst (must not overlap).  Synchronous. */
int hsort_device_radix_pass(const uint64_t* d_src, uint64_t* d_dst, uint64_t n, int digit,
                            void* stream);

/* K4 alone: exact co-ranks (merge path) of output positions o_b = min(b*step, total)
 * for b = 0..n_bounds-1 over k sorted uint64 runs d_keys[h_off[j] .. h_off[j+1]).  d_ranks is
 * (n_bounds x k) uint64 row-major on the device; h_off is k+1 HOST offsets.  Ties are taken in
 * run order.  Synchronous. */
int hsort_device_corank(const uint64_t* d_keys, const uint64_t* h_off, int k, uint64_t step,
                        uint64_t n_bounds, uint64_t* d_ranks, void* stream);

/* K4+K5: multiway merge of k sorted uint64 runs (layout as above) into d_out
 * (total = h_off[k]-h_off[0] elements); out_f64 = 1 stores inverse-transformed float64 bits.
 * Synchronous. */
int hsort_device_merge(const uint64_t* d_keys, const uint64_t* h_off, int k, uint64_t* d_out,
                       int out_f64, void* stream);

/* Splitter partition of one sorted uint64 run (multi-GPU exchange):
 * d_out[i] = number of keys <= d_values[i] in d_keys[0, n).  Device pointers; synchronous. */
int hsort_device_upper_bounds(const uint64_t* d_keys, uint64_t n, const uint64_t* d_values,
                              uint64_t m, uint64_t* d_out, void* stream);

/* ---------------------------------------------------------------------------------------------
 * Host-native components (no GPU needed)
 * ------------------------------------------------------------------------------------------- */

/* Parallel host memcpy (PARMEMCPY) with `threads` workers (0 = option default). */
int hsort_par_memcpy(void* dst, const void* src, uint64_t bytes, int threads);

/* CPU multiway merge (H2): k sorted uint64 key runs keys[off[j]..off[j+1]) (host)
 * -> out (host, total elements); out_f64 = 1 stores inverse-transformed float64 bits.
 * Output ranges are split by exact co-ranks and merged by `threads` loser trees. */
int hsort_host_merge(const uint64_t* keys, const uint64_t* off, int k, uint64_t* out,
                     int out_f64, int threads);

/* Exact co-ranks of output position o over the k host runs (same definition as K4). */
int hsort_host_corank(const uint64_t* keys, const uint64_t* off, int k, uint64_t o,
                      uint64_t* ranks);

/* Host version of hsort_device_upper_bounds (keys, values, out in host memory). */
int hsort_host_upper_bounds(const uint64_t* keys, uint64_t n, const uint64_t* values, uint64_t m,
                            uint64_t* out);

/* Splitter arithmetic of the multi-process exchange (A13, paper_conf_ipps_gowanlockk18a_b200/dist.py;
 * one process per GPU, torch.distributed moves the data).  hsort_sample_positions: the s regular
 * sample positions of a sorted run of n >= 1 keys, pos[i] = min(n - 1, (i + 1) n / (s + 1)).
 * hsort_select_splitters: from the m merged (sorted) samples of all ranks, the P - 1 splitters
 * spl[r - 1] = samples[r m / P] (r = 1..P-1; all 0 when m = 0); rank r then owns the keys k with
 * spl[r - 1] < k <= spl[r].  Pure host arithmetic; HSORT_ERR_INVALID on bad arguments. */
int hsort_sample_positions(uint64_t n, uint64_t s, uint64_t* pos);
int hsort_select_splitters(const uint64_t* samples, uint64_t m, int P, uint64_t* spl);

/* The PIPEMERGE heuristic (reading A-9): number of pair-wise merges overlapped with
 * GPU sorting; STREAM mode merges pairs (0,1), (2,3), ... of that many (option "pipemerge").
 * Pure arithmetic. */
uint64_t hsort_pipemerge_count(uint64_t n_b, int n_gpus);

/* Kernels the library has launched since it was loaded (all devices; K1, K2, K3 passes, copies,
 * the elision's kernels, K4, K5, codecs): the difference across a region counts the region's
 * launches (bench.py gpu_launches). */
uint64_t hsort_get_launch_count(void);

/* Number of GPUs visible to the library (0 when none; never an error). */
int hsort_device_count(void);

#ifdef __cplusplus
}
#endif
#endif /* HSORT_H_ */
