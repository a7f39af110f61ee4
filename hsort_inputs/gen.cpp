// hsort_inputs/gen.cpp — seeded synthetic float64 workloads (test/bench input generator).
//
// This module holds NONE of the method's arithmetic (no key transform, no ordering, no sort,
// no merge). It only produces input arrays A, shaped like the paper's workloads:
//   * uniform float64            — the paper's only distribution (§IV-A)
//   * normal N(0,1)              — BASELINE.json configs[3] "normal/skewed"
//   * zipf-dup skew              — BASELINE.json configs[3]; heavy exact duplicates
//   * special-value mixes, sorted/reverse/all-equal/few-distinct — edge cases
//   * closed-form permutations   — A[i] = f(pi(i)), f(i) = (double)(i - n/2); the sorted
//                                  result is B[i] = f(i), checkable in O(n)
//
// Random numbers: counter-based splitmix64, r_i = mix(seed + (i+1) * 0x9E3779B97F4A7C15),
// so any element can be produced independently and the generation is parallel and
// bit-reproducible for any thread count.
#include <cmath>
#include <cstdint>
#include <cstring>
#include <thread>
#include <vector>
#include <algorithm>

namespace {

inline uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}
// r(seed, stream, i): independent 64-bit random word for element i of sub-stream `stream`.
inline uint64_t rnd(uint64_t seed, uint64_t stream, uint64_t i) {
  return mix64(seed * 0xD1B54A32D192ED03ULL + stream * 0xABC98388FB8FAC03ULL +
               (i + 1) * 0x9E3779B97F4A7C15ULL);
}
// U[0,1) from the top 53 bits.
inline double u01(uint64_t r) { return (double)(r >> 11) * 0x1.0p-53; }
// (0,1] from the top 53 bits (for logs).
inline double u01_open0(uint64_t r) { return (double)((r >> 11) + 1) * 0x1.0p-53; }

inline double bits2d(uint64_t u) { double d; std::memcpy(&d, &u, 8); return d; }

template <class F>
void par_for(uint64_t n, int threads, F f) {
  if (threads <= 0) {
    unsigned hc = std::thread::hardware_concurrency();
    threads = hc ? (int)hc : 1;
  }
  if (n < (1u << 16) || threads == 1) { f(0, n); return; }
  std::vector<std::thread> ts;
  uint64_t chunk = (n + threads - 1) / threads;
  for (int t = 0; t < threads; ++t) {
    uint64_t lo = t * chunk, hi = std::min<uint64_t>(n, lo + chunk);
    if (lo >= hi) break;
    ts.emplace_back([=] { f(lo, hi); });
  }
  for (auto& t : ts) t.join();
}

inline double normal_at(uint64_t seed, uint64_t i) {
  // Box–Muller, one output per pair of independent uniforms.
  double u1 = u01_open0(rnd(seed, 1, i)), u2 = u01(rnd(seed, 2, i));
  return std::sqrt(-2.0 * std::log(u1)) * std::cos(6.283185307179586 * u2);
}

// The special-value alphabet (15 values + random bit patterns), SURVEY.md §8(c) item 1.
const uint64_t kSpecial[] = {
    0xFFF8000000000000ULL,  // -qNaN
    0xFFF0000000000001ULL,  // -sNaN
    0xFFF0000000000000ULL,  // -inf
    0xFFEFFFFFFFFFFFFFULL,  // -DBL_MAX
    0xBFF0000000000000ULL,  // -1
    0x8000000000000001ULL,  // -DBL_TRUE_MIN
    0x8000000000000000ULL,  // -0
    0x0000000000000000ULL,  // +0
    0x0000000000000001ULL,  // +DBL_TRUE_MIN
    0x3FF0000000000000ULL,  // +1
    0x7FEFFFFFFFFFFFFFULL,  // +DBL_MAX
    0x7FF0000000000000ULL,  // +inf
    0x7FF0000000000001ULL,  // +sNaN
    0x7FF8000000000000ULL,  // +qNaN
    0x7FFFFFFFFFFFFFFFULL,  // +qNaN, max payload
};
constexpr int kNumSpecial = 15;

}  // namespace

extern "C" {

int hsort_inputs_num_special(void) { return kNumSpecial; }
void hsort_inputs_special(uint64_t* out) { std::memcpy(out, kSpecial, sizeof(kSpecial)); }

// dist codes (mirrored in hsort_inputs/__init__.py)
//  0 uniform U[0,1)      1 normal N(0,1)      2 zipf-dup skew      3 special mix
//  4 random bit patterns 5 sorted ascending   6 sorted descending  7 all equal
//  8 few distinct (16)   9 closed-form perm   10 signed-zero / NaN salted uniform (1%)
//  11 uniform U[-1,1)
int hsort_inputs_generate(double* out, uint64_t n, int dist, uint64_t seed, int threads) {
  switch (dist) {
    case 0:
      par_for(n, threads, [&](uint64_t lo, uint64_t hi) {
        for (uint64_t i = lo; i < hi; ++i) out[i] = u01(rnd(seed, 0, i));
      });
      return 0;
    case 1:
      par_for(n, threads, [&](uint64_t lo, uint64_t hi) {
        for (uint64_t i = lo; i < hi; ++i) out[i] = normal_at(seed, i);
      });
      return 0;
    case 2: {
      // zipf-dup: 50% draws from a hot set of 2^16 normal values with Zipf(s=1) weights,
      // 50% fresh normals.
      const int H = 1 << 16;
      std::vector<double> hot(H), cdf(H);
      double acc = 0;
      for (int r = 0; r < H; ++r) {
        hot[r] = normal_at(seed ^ 0x5EED5EEDULL, (uint64_t)r);
        acc += 1.0 / (double)(r + 1);
        cdf[r] = acc;
      }
      for (int r = 0; r < H; ++r) cdf[r] /= acc;
      par_for(n, threads, [&](uint64_t lo, uint64_t hi) {
        for (uint64_t i = lo; i < hi; ++i) {
          uint64_t c = rnd(seed, 3, i);
          if (c & 1) {
            double u = u01(rnd(seed, 4, i));
            int r = (int)(std::lower_bound(cdf.begin(), cdf.end(), u) - cdf.begin());
            if (r >= H) r = H - 1;
            out[i] = hot[r];
          } else {
            out[i] = normal_at(seed, i);
          }
        }
      });
      return 0;
    }
    case 3:
      par_for(n, threads, [&](uint64_t lo, uint64_t hi) {
        for (uint64_t i = lo; i < hi; ++i) {
          uint64_t r = rnd(seed, 5, i);
          uint64_t sel = r % 20;
          out[i] = sel < (uint64_t)kNumSpecial ? bits2d(kSpecial[sel]) : bits2d(rnd(seed, 6, i));
        }
      });
      return 0;
    case 4:
      par_for(n, threads, [&](uint64_t lo, uint64_t hi) {
        for (uint64_t i = lo; i < hi; ++i) out[i] = bits2d(rnd(seed, 7, i));
      });
      return 0;
    case 5:
      par_for(n, threads, [&](uint64_t lo, uint64_t hi) {
        for (uint64_t i = lo; i < hi; ++i) out[i] = (double)i * 0.5 - 1000.0;
      });
      return 0;
    case 6:
      par_for(n, threads, [&](uint64_t lo, uint64_t hi) {
        for (uint64_t i = lo; i < hi; ++i) out[i] = (double)(n - i) * 0.25;
      });
      return 0;
    case 7:
      par_for(n, threads, [&](uint64_t lo, uint64_t hi) {
        double v = u01(rnd(seed, 8, 0));
        for (uint64_t i = lo; i < hi; ++i) out[i] = v;
      });
      return 0;
    case 8:
      par_for(n, threads, [&](uint64_t lo, uint64_t hi) {
        for (uint64_t i = lo; i < hi; ++i) out[i] = (double)(int)(rnd(seed, 9, i) % 16) - 7.5;
      });
      return 0;
    case 9: {
      // A[i] = f(pi(i)), pi(i) = (a*i + c) mod n with gcd(a, n) = 1; f(j) = (double)(j - n/2).
      if (n == 0) return 0;
      auto gcd = [](uint64_t x, uint64_t y) { while (y) { uint64_t t = x % y; x = y; y = t; } return x; };
      uint64_t a = rnd(seed, 10, 0) % n;
      if (a == 0) a = 1;
      while (gcd(a, n) != 1) { if (++a >= n) a = 1; }
      uint64_t c = rnd(seed, 11, 0) % n;
      int64_t half = (int64_t)(n / 2);
      par_for(n, threads, [&](uint64_t lo, uint64_t hi) {
        for (uint64_t i = lo; i < hi; ++i) {
          uint64_t j = (uint64_t)(((__uint128_t)a * i + c) % n);
          out[i] = (double)((int64_t)j - half);
        }
      });
      return 0;
    }
    case 10:
      par_for(n, threads, [&](uint64_t lo, uint64_t hi) {
        for (uint64_t i = lo; i < hi; ++i) {
          uint64_t r = rnd(seed, 12, i);
          uint64_t s = r % 400;
          if (s == 0) out[i] = bits2d(0x8000000000000000ULL);
          else if (s == 1) out[i] = 0.0;
          else if (s == 2) out[i] = bits2d(0x7FF8000000000000ULL | (r >> 20));
          else if (s == 3) out[i] = bits2d(0xFFF8000000000000ULL | (r >> 20));
          else out[i] = u01(rnd(seed, 13, i)) * ((r >> 9) & 1 ? 1.0 : -1.0);
        }
      });
      return 0;
    case 11:
      par_for(n, threads, [&](uint64_t lo, uint64_t hi) {
        for (uint64_t i = lo; i < hi; ++i) out[i] = 2.0 * u01(rnd(seed, 14, i)) - 1.0;
      });
      return 0;
    default:
      return -1;
  }
}

}  // extern "C"
