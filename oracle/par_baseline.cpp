// oracle/par_baseline.cpp — the PARALLEL-CPU BASELINE (BASELINE.md "CPU-baseline plan" item 2;
// SURVEY.md §8(d)): the paper's reference implementation, GNU libstdc++ parallel-mode sort
// (multiway mergesort), on all host cores, under the same IEEE totalOrder as the
// oracle.  TEST / BENCH INFRASTRUCTURE ONLY (bench.py's cpu baseline leg and tests/); the product
// never links it, and it shares no code with the CUDA path.  Built with -fopenmp into its own
// library so the serial oracle stays OpenMP-free.
#include <omp.h>
#include <parallel/algorithm>

#include <compare>
#include <cstdint>
#include <cstring>

extern "C" {

// B = A sorted by totalOrder (std::strong_order<double>), threads = OpenMP threads (0 = default).
void par_sort_f64(const double* A, double* B, uint64_t n, int threads) {
  if (B != A) std::memcpy(B, A, n * sizeof(double));
  if (threads > 0) omp_set_num_threads(threads);
  __gnu_parallel::sort(B, B + n, [](double a, double b) { return std::strong_order(a, b) < 0; },
                       __gnu_parallel::multiway_mergesort_exact_tag());
}

int par_max_threads(void) { return omp_get_max_threads(); }

}  // extern "C"

#include <parallel/multiway_merge.h>

#include <utility>
#include <vector>

extern "C" {

// CPU-merge reference (BASELINE.md plan item 3; the paper's own merge): GNU parallel
// multiway_merge of k sorted uint64 runs keys[off[j], off[j+1]) into out, `threads` OpenMP threads.
void par_multiway_merge_u64(const uint64_t* keys, const uint64_t* off, int k, uint64_t* out,
                            int threads) {
  if (threads > 0) omp_set_num_threads(threads);
  // (libstdc++'s multiway_merge needs mutable iterators; the runs are only read)
  uint64_t* base = const_cast<uint64_t*>(keys);
  std::vector<std::pair<uint64_t*, uint64_t*>> seqs(k);
  for (int j = 0; j < k; ++j) seqs[j] = {base + off[j], base + off[j + 1]};
  const uint64_t total = off[k] - off[0];
  __gnu_parallel::multiway_merge(seqs.begin(), seqs.end(), out, total, std::less<uint64_t>(),
                                 __gnu_parallel::parallel_tag());
}

}  // extern "C"
