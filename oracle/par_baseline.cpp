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
