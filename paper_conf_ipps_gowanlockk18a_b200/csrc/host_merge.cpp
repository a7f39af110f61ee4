// host_merge.cpp — CPU multiway merge of the sorted batches (§III-A: "we use
// the parallel multiway merge from the GNU library ... O(n log n_b) work").
//
// B200 build: the output is cut into ranges by exact co-ranks (merge path [18], P:138-142,
// generalised to k runs: multi-sequence selection with ties taken in run order), and each range
// is merged independently by one thread with a loser tree (ceil(log2 k) compares per key); the
// inverse key transform is fused into the store.  Keys are the order-preserving uint64 view of the
// float64 bits, so compares are plain unsigned compares.
#include <algorithm>
#include <cstdint>
#include <cstring>
#include <vector>

#include "pool.h"

namespace hsort {

namespace {

inline uint64_t from_key(uint64_t k) {
  return k ^ ((uint64_t)((int64_t)(~k) >> 63) | 0x8000000000000000ull);
}

// #elements <= v in a[lo, hi)  (absolute index)
inline uint64_t ub(const uint64_t* a, uint64_t lo, uint64_t hi, uint64_t v) {
  while (lo < hi) {
    uint64_t m = lo + ((hi - lo) >> 1);
    if (a[m] <= v) lo = m + 1;
    else hi = m;
  }
  return lo;
}
inline uint64_t lb(const uint64_t* a, uint64_t lo, uint64_t hi, uint64_t v) {
  while (lo < hi) {
    uint64_t m = lo + ((hi - lo) >> 1);
    if (a[m] < v) lo = m + 1;
    else hi = m;
  }
  return lo;
}

// Loser tree over K (power of two) leaves; dead leaves lose to every live one.
class LoserTree {
 public:
  LoserTree(int k) : k_(k) {
    K_ = 1;
    while (K_ < k) K_ <<= 1;
    key_.assign(K_, ~0ull);
    dead_.assign(K_, 1);
    pos_.assign(K_, 0);
    end_.assign(K_, 0);
    tree_.assign(K_, 0);
  }
  void set_leaf(int j, const uint64_t* p, const uint64_t* e) {
    pos_[j] = p;
    end_[j] = e;
    dead_[j] = (p >= e);
    key_[j] = dead_[j] ? ~0ull : *p;
  }
  void build() {
    // winners bottom-up, storing losers
    std::vector<int> win(2 * K_);
    for (int i = 0; i < K_; ++i) win[K_ + i] = i;
    for (int n = K_ - 1; n >= 1; --n) {
      int a = win[2 * n], b = win[2 * n + 1];
      if (less(b, a)) std::swap(a, b);
      win[n] = a;
      tree_[n] = b;
    }
    tree_[0] = win[1];
  }
  inline bool less(int a, int b) const {
    if (dead_[a]) return false;
    if (dead_[b]) return true;
    return key_[a] < key_[b] || (key_[a] == key_[b] && a < b);
  }
  // pop the minimum (caller guarantees one live leaf)
  inline uint64_t pop() {
    int w = tree_[0];
    uint64_t out = key_[w];
    const uint64_t* p = ++pos_[w];
    if (p < end_[w]) key_[w] = *p;
    else dead_[w] = 1;
    for (int n = (w + K_) >> 1; n >= 1; n >>= 1) {
      int l = tree_[n];
      if (less(l, w)) { tree_[n] = w; w = l; }
    }
    tree_[0] = w;
    return out;
  }

 private:
  int k_, K_;
  std::vector<uint64_t> key_;
  std::vector<uint8_t> dead_;
  std::vector<const uint64_t*> pos_, end_;
  std::vector<int> tree_;
};

}  // namespace

// Exact co-ranks of output position o (ties in run order).  Same definition as K4 (merge.cu).
void host_corank(const uint64_t* keys, const uint64_t* off, int k, uint64_t o, uint64_t* ranks) {
  std::vector<uint64_t> lo(k), hi(k);
  uint64_t total = off[k] - off[0];
  for (int j = 0; j < k; ++j) {
    lo[j] = 0;
    hi[j] = off[j + 1] - off[j];
  }
  if (o >= total) {
    for (int j = 0; j < k; ++j) ranks[j] = hi[j];
    return;
  }
  uint64_t L = 0, H = ~0ull;
  while (true) {
    uint64_t mn = ~0ull, mx = 0;
    for (int j = 0; j < k; ++j)
      if (hi[j] > lo[j]) {
        const uint64_t* r = keys + off[j];
        mn = std::min(mn, r[lo[j]]);
        mx = std::max(mx, r[hi[j] - 1]);
      }
    L = std::max(L, mn);
    H = std::min(H, mx);
    if (L >= H) break;
    uint64_t mid = L + ((H - L) >> 1), s = 0;
    std::vector<uint64_t> u(k);
    for (int j = 0; j < k; ++j) {
      u[j] = ub(keys + off[j], lo[j], hi[j], mid);
      s += u[j];
    }
    if (s > o) { H = mid; hi = u; }
    else { L = mid + 1; lo = u; }
  }
  const uint64_t v = L;
  uint64_t lt = 0;
  std::vector<uint64_t> eq(k);
  for (int j = 0; j < k; ++j) {
    const uint64_t* r = keys + off[j];
    uint64_t a = lb(r, lo[j], hi[j], v);
    uint64_t z = ub(r, a, hi[j], v);
    lo[j] = a;
    eq[j] = z - a;
    lt += a;
  }
  uint64_t rem = o - lt;
  for (int j = 0; j < k; ++j) {
    uint64_t t = std::min(rem, eq[j]);
    ranks[j] = lo[j] + t;
    rem -= t;
  }
}

// Merge output range [o_a, o_b) given its co-ranks ra (at o_a) and rb (at o_b).
static void merge_range(const uint64_t* keys, const uint64_t* off, int k, const uint64_t* ra,
                        const uint64_t* rb, uint64_t* out, bool out_f64) {
  int live = 0, last = -1;
  for (int j = 0; j < k; ++j)
    if (rb[j] > ra[j]) { ++live; last = j; }
  if (live == 0) return;
  if (live == 1) {
    const uint64_t* s = keys + off[last] + ra[last];
    uint64_t len = rb[last] - ra[last];
    if (out_f64)
      for (uint64_t i = 0; i < len; ++i) out[i] = from_key(s[i]);
    else
      std::memcpy(out, s, len * 8);
    return;
  }
  if (live == 2) {
    int a = -1, b = -1;
    for (int j = 0; j < k; ++j)
      if (rb[j] > ra[j]) (a < 0 ? a : b) = j;
    const uint64_t *p = keys + off[a] + ra[a], *pe = keys + off[a] + rb[a];
    const uint64_t *q = keys + off[b] + ra[b], *qe = keys + off[b] + rb[b];
    uint64_t* o = out;
    while (p < pe && q < qe) {
      uint64_t x = *p, y = *q;
      bool takep = x <= y;
      uint64_t v = takep ? x : y;
      p += takep;
      q += !takep;
      *o++ = out_f64 ? from_key(v) : v;
    }
    while (p < pe) { *o++ = out_f64 ? from_key(*p) : *p; ++p; }
    while (q < qe) { *o++ = out_f64 ? from_key(*q) : *q; ++q; }
    return;
  }
  LoserTree lt(k);
  uint64_t total = 0;
  for (int j = 0; j < k; ++j) {
    lt.set_leaf(j, keys + off[j] + ra[j], keys + off[j] + rb[j]);
    total += rb[j] - ra[j];
  }
  lt.build();
  if (out_f64)
    for (uint64_t i = 0; i < total; ++i) out[i] = from_key(lt.pop());
  else
    for (uint64_t i = 0; i < total; ++i) out[i] = lt.pop();
}

void host_merge(const uint64_t* keys, const uint64_t* off, int k, uint64_t* out, bool out_f64,
                int threads) {
  if (threads <= 0) threads = host_threads();
  const uint64_t total = off[k] - off[0];
  if (total == 0) return;
  // normalise offsets to start at 0 relative to keys + off[0]
  std::vector<uint64_t> o2(k + 1);
  for (int j = 0; j <= k; ++j) o2[j] = off[j] - off[0];
  const uint64_t* K = keys + off[0];
  // ranges: ~4 per thread, each at least 64K keys
  int64_t R = std::max<int64_t>(1, std::min<int64_t>((int64_t)threads * 4, (int64_t)(total >> 16)));
  std::vector<uint64_t> ranks((R + 1) * (uint64_t)k);
  host_pool().parallel_for(R + 1, threads, [&](int64_t r) {
    uint64_t o = (uint64_t)((__uint128_t)total * (uint64_t)r / (uint64_t)R);
    host_corank(K, o2.data(), k, o, &ranks[(uint64_t)r * k]);
  });
  host_pool().parallel_for(R, threads, [&](int64_t r) {
    uint64_t o = (uint64_t)((__uint128_t)total * (uint64_t)r / (uint64_t)R);
    merge_range(K, o2.data(), k, &ranks[(uint64_t)r * k], &ranks[(uint64_t)(r + 1) * k], out + o,
                out_f64);
  });
}

}  // namespace hsort
