// oracle/oracle.cpp — the CPU ORACLE for the heterogeneous float64 sort.
//
// TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
// `--impl reference` leg may load this library.  The product path
// (paper_conf_ipps_gowanlockk18a_b200/) never links, imports or calls it, and this file shares
// no code, header, table or constant generator with the CUDA path.
//
// Each function is the plain definition of what the method computes, written serially, with no
// blocking, fusion or reordering; a library primitive (std::sort, std::stable_sort) serves as a
// step where the definition is "sort".  Citations are PAPER.md line ranges (P:a-b).
//
// Parity status (details in DESIGN.md §4 "Oracle pins"):
//   oracle_sort_f64            pinned: brute force (all permutations n<=7, all length-<=4
//                              sequences over the special alphabet) vs an IEEE 754 §5.10
//                              clause-by-clause predicate; numpy.sort on NaN/-0-free data;
//                              closed-form permutation inputs; sortedness + multiset invariants.
//   oracle_key / oracle_key_inv pinned: order-isomorphism with std::strong_order (C++20 library
//                              totalOrder) over the special alphabet x alphabet and 10^6 random
//                              pairs; bijection on random words.
//   oracle_digit_histograms    pinned: closed-form histograms of constructed key sets.
//   oracle_counting_sort_pass  pinned: numpy stable argsort gather; LSD composition theorem.
//   oracle_merge_runs          pinned: heapq.merge; equals oracle_sort of the concatenation.
//   oracle_corank              pinned: co-rank invariants (sum, boundary) + brute force.
//   oracle_pipemerge_count     pinned: Fig. 3 worked example (tests/golden/fig3_pipemerge.txt).
//   oracle_is_sorted_f64 / oracle_multiset_hash: pinned by planted faults.
//   oracle_sort_f32 / oracle_sort_desc_f64 pinned: brute force (all permutations of small
//                              inputs over a binary32 special alphabet) vs a Python restatement
//                              of the IEEE clauses on binary32 bits; numpy.sort on NaN/-0-free
//                              data; descending = reverse of ascending (unique result).
//   oracle_sort_pairs_f64/_u64 pinned: keys = oracle_sort; values = numpy stable argsort on
//                              NaN/-0-free keys; brute force over all permutations of small
//                              duplicate-heavy inputs vs a Python insertion sort (stable by
//                              construction) under the IEEE clause predicate; pair multiset.
#include <algorithm>
#include <compare>
#include <cstdint>
#include <cstring>
#include <vector>

namespace {
inline uint64_t d2u(double d) { uint64_t u; std::memcpy(&u, &d, 8); return u; }
inline double u2d(uint64_t u) { double d; std::memcpy(&d, &u, 8); return d; }
inline bool total_less(double a, double b) { return std::strong_order(a, b) < 0; }
}  // namespace

extern "C" {

// ---------------------------------------------------------------------------------------------
// IEEE 754 totalOrder as a three-way compare, via the C++20 library (std::strong_order is
// specified as ISO/IEC 60559 totalOrder for floating-point types).  Reading A-1..A-3 of
// -0 < +0, NaNs ordered by sign and payload, denormals by value, bits preserved.
int oracle_total_order_cmp(double a, double b) {
  auto c = std::strong_order(a, b);
  return c < 0 ? -1 : (c > 0 ? 1 : 0);
}

// ---------------------------------------------------------------------------------------------
// The problem (§I): given unsorted A of n elements in main memory, produce the sorted
// list B.  B = the multiset {bits(A[i])} in non-decreasing IEEE totalOrder (A-1..A-4).
// The paper's batched sort + multiway merge reaches exactly this result.
void oracle_sort_f64(const double* A, double* B, uint64_t n) {
  if (B != A) std::memcpy(B, A, n * sizeof(double));
  std::sort(B, B + n, total_less);
}

// ---------------------------------------------------------------------------------------------
// Other key types and orders.  float32 keys under binary32 totalOrder
// (std::strong_order<float>), and the descending order (reverse totalOrder) for both types:
// B = A sorted by y precedes x <=> totalOrder(x, y) strictly.
void oracle_sort_f32(const float* A, float* B, uint64_t n, int descending) {
  if (B != A) std::memcpy(B, A, n * sizeof(float));
  if (descending)
    std::sort(B, B + n, [](float a, float b) { return std::strong_order(a, b) > 0; });
  else
    std::sort(B, B + n, [](float a, float b) { return std::strong_order(a, b) < 0; });
}

void oracle_sort_desc_f64(const double* A, double* B, uint64_t n) {
  if (B != A) std::memcpy(B, A, n * sizeof(double));
  std::sort(B, B + n, [](double a, double b) { return std::strong_order(a, b) > 0; });
}

// ---------------------------------------------------------------------------------------------
// Key/value sort (the [5] workload of 64-bit keys with values):
// the pairs (A[i], V[i]) ordered by A under totalOrder, STABLY (equal keys keep input order), so
// the result is unique.  Definition: std::stable_sort of the index sequence 0..n-1 by A[i], then
// gather.
void oracle_sort_pairs_f64(const double* A, const uint64_t* V, double* B, uint64_t* VB, uint64_t n) {
  std::vector<uint64_t> idx(n);
  for (uint64_t i = 0; i < n; ++i) idx[i] = i;
  std::stable_sort(idx.begin(), idx.end(), [&](uint64_t x, uint64_t y) { return total_less(A[x], A[y]); });
  std::vector<double> b(n);
  std::vector<uint64_t> vb(n);
  for (uint64_t i = 0; i < n; ++i) {
    b[i] = A[idx[i]];
    vb[i] = V[idx[i]];
  }
  std::memcpy(B, b.data(), n * sizeof(double));
  std::memcpy(VB, vb.data(), n * sizeof(uint64_t));
}

// Same on raw uint64 keys, ascending unsigned.
void oracle_sort_pairs_u64(const uint64_t* A, const uint64_t* V, uint64_t* B, uint64_t* VB, uint64_t n) {
  std::vector<uint64_t> idx(n);
  for (uint64_t i = 0; i < n; ++i) idx[i] = i;
  std::stable_sort(idx.begin(), idx.end(), [&](uint64_t x, uint64_t y) { return A[x] < A[y]; });
  std::vector<uint64_t> b(n), vb(n);
  for (uint64_t i = 0; i < n; ++i) {
    b[i] = A[idx[i]];
    vb[i] = V[idx[i]];
  }
  std::memcpy(B, b.data(), n * sizeof(uint64_t));
  std::memcpy(VB, vb.data(), n * sizeof(uint64_t));
}

// ---------------------------------------------------------------------------------------------
// Order-preserving map float64 bits -> uint64 (DESIGN.md §2 step A4; not in the paper, whose
// GPU sort hides it inside Thrust):  key(u) = u>>63 ? ~u : u | 2^63.
uint64_t oracle_key(uint64_t u) {
  if (u >> 63) return ~u;
  return u | 0x8000000000000000ULL;
}
uint64_t oracle_key_inv(uint64_t k) {
  if (k >> 63) return k & 0x7FFFFFFFFFFFFFFFULL;
  return ~k;
}
void oracle_keys_from_f64(const double* A, uint64_t* K, uint64_t n) {
  for (uint64_t i = 0; i < n; ++i) K[i] = oracle_key(d2u(A[i]));
}
void oracle_f64_from_keys(const uint64_t* K, double* B, uint64_t n) {
  for (uint64_t i = 0; i < n; ++i) B[i] = u2d(oracle_key_inv(K[i]));
}

// Sort of raw uint64 keys ascending (the "sorted batch" of P:202-204 in key space).
void oracle_sort_u64(const uint64_t* A, uint64_t* B, uint64_t n) {
  if (B != A) std::memcpy(B, A, n * sizeof(uint64_t));
  std::sort(B, B + n);
}

// ---------------------------------------------------------------------------------------------
// LSD radix semantics of the GPU sort (P:253-264 says only "radix sort"; DESIGN.md §2 A5/A6):
// digit d of key k is bits [8d, 8d+8).  hist[d*256 + v] = #{i : digit_d(K[i]) == v}.
void oracle_digit_histograms(const uint64_t* K, uint64_t n, uint64_t* hist) {
  std::memset(hist, 0, 8 * 256 * sizeof(uint64_t));
  for (uint64_t i = 0; i < n; ++i)
    for (int d = 0; d < 8; ++d) hist[d * 256 + ((K[i] >> (8 * d)) & 255)] += 1;
}

// One LSD pass: the stable counting sort of src by digit d (textbook: count, exclusive prefix
// sum, stable scatter in input order).
void oracle_counting_sort_pass(const uint64_t* src, uint64_t* dst, uint64_t n, int d) {
  std::vector<uint64_t> cnt(256, 0);
  for (uint64_t i = 0; i < n; ++i) cnt[(src[i] >> (8 * d)) & 255] += 1;
  uint64_t run = 0;
  for (int v = 0; v < 256; ++v) { uint64_t c = cnt[v]; cnt[v] = run; run += c; }
  for (uint64_t i = 0; i < n; ++i) dst[cnt[(src[i] >> (8 * d)) & 255]++] = src[i];
}

// ---------------------------------------------------------------------------------------------
// Multiway merge of the n_b sorted batches (§III-A): the result is the sorted
// concatenation.  keys holds the k runs back to back; run j is [off[j], off[j+1]).
void oracle_merge_runs(const uint64_t* keys, const uint64_t* off, int k, uint64_t* out) {
  uint64_t n = off[k] - off[0];
  std::memcpy(out, keys + off[0], n * sizeof(uint64_t));
  std::stable_sort(out, out + n);
}

// Co-ranks of output position o (merge path [18]): ranks[j] = how many elements of
// run j are among the first o elements of the merge in which equal keys are taken in run order.
// Definition written out: tag every element with (key, run), stable-sort, count the first o.
void oracle_corank(const uint64_t* keys, const uint64_t* off, int k, uint64_t o, uint64_t* ranks) {
  std::vector<std::pair<uint64_t, int>> all;
  for (int j = 0; j < k; ++j)
    for (uint64_t i = off[j]; i < off[j + 1]; ++i) all.push_back({keys[i], j});
  std::stable_sort(all.begin(), all.end());
  for (int j = 0; j < k; ++j) ranks[j] = 0;
  for (uint64_t i = 0; i < o && i < all.size(); ++i) ranks[all[i].second] += 1;
}

// ---------------------------------------------------------------------------------------------
// PIPEMERGE heuristic (§III-D3; reading A-9): the number of pair-wise merges run
// while the GPU still sorts.  n_GPU = 1: floor((n_b - 1) / 2);  n_GPU >= 2: floor(n_b / (2 n_GPU)).
uint64_t oracle_pipemerge_count(uint64_t n_b, int n_gpu) {
  if (n_b == 0) return 0;
  if (n_gpu <= 1) return (n_b - 1) / 2;
  return n_b / (2 * (uint64_t)n_gpu);
}

// ---------------------------------------------------------------------------------------------
// Verifiers for sizes where a full oracle run is too slow: B is the
// unique answer iff it is sorted under totalOrder and is a permutation of A's bit patterns.
int oracle_is_sorted_f64(const double* B, uint64_t n) {
  for (uint64_t i = 1; i < n; ++i)
    if (total_less(B[i], B[i - 1])) return 0;
  return 1;
}
// Order-independent multiset hash: (sum h1(u), sum h2(u)) mod 2^64 over bit patterns u.
void oracle_multiset_hash(const double* A, uint64_t n, uint64_t* out2) {
  uint64_t s1 = 0, s2 = 0;
  for (uint64_t i = 0; i < n; ++i) {
    uint64_t z = d2u(A[i]) + 0x9E3779B97F4A7C15ULL;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    s1 += z ^ (z >> 31);
    uint64_t y = d2u(A[i]) * 0xD6E8FEB86659FD93ULL;
    y ^= y >> 32;
    y *= 0xD6E8FEB86659FD93ULL;
    y ^= y >> 29;
    s2 += y;
  }
  out2[0] = s1;
  out2[1] = s2;
}

}  // extern "C"
