// host_merge.cpp — CPU multiway merge of the sorted batches (§III-A: "we use
// the parallel multiway merge from the GNU library ... O(n log n_b) work").
//
// B200 build: the output is cut into ranges by exact co-ranks (merge path [18], P:138-142,
// generalised to k runs: multi-sequence selection with ties taken in run order), and each range
// is merged independently by one thread with a loser tree (ceil(log2 k) compares per key); the
// inverse key transform is fused into the store.  Keys are the order-preserving uint64 view of the
// float64 bits, so compares are plain unsigned compares.
#include <emmintrin.h>

#include <algorithm>
#include <cstdint>
#include <cstring>
#include <new>
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

// Loser tree over K (power of two) leaves, branch-free replay.  Each node holds a (key, src)
// pair compared lexicographically; a live leaf has src = leaf index (< K) and an exhausted leaf
// has key = 2^64-1 and src = K + leaf, so it loses to every live key, including a live 2^64-1.
class LoserTree {
 public:
  explicit LoserTree(int k) {
    K_ = 1;
    while (K_ < k) K_ <<= 1;
    tk_.assign(K_, ~0ull);
    ts_.assign(K_, 0);
    cur_.assign(K_, nullptr);
    end_.assign(K_, nullptr);
  }
  void set_leaf(int j, const uint64_t* p, const uint64_t* e) {
    cur_[j] = p;
    end_[j] = e;
  }
  void build() {
    std::vector<uint64_t> wk(2 * K_);
    std::vector<uint32_t> ws(2 * K_);
    for (int i = 0; i < K_; ++i) {
      const bool live = cur_[i] && cur_[i] < end_[i];
      wk[K_ + i] = live ? *cur_[i] : ~0ull;
      ws[K_ + i] = live ? (uint32_t)i : (uint32_t)(K_ + i);
    }
    for (int v = K_ - 1; v >= 1; --v) {
      uint64_t ak = wk[2 * v], bk = wk[2 * v + 1];
      uint32_t as = ws[2 * v], bs = ws[2 * v + 1];
      const bool bwins = (bk < ak) | ((bk == ak) & (bs < as));
      wk[v] = bwins ? bk : ak;
      ws[v] = bwins ? bs : as;
      tk_[v] = bwins ? ak : bk;
      ts_[v] = bwins ? as : bs;
    }
    win_k_ = wk[1];
    win_s_ = ws[1];
  }
  // pop the minimum (caller guarantees a live leaf remains)
  inline uint64_t pop() {
    const uint64_t out = win_k_;
    const uint32_t leaf = win_s_;
    const uint64_t* p = ++cur_[leaf];
    uint64_t nk;
    uint32_t ns;
    if (__builtin_expect(p < end_[leaf], 1)) {
      nk = *p;
      ns = leaf;
    } else {
      nk = ~0ull;
      ns = (uint32_t)K_ + leaf;
    }
    uint64_t* tk = tk_.data();
    uint32_t* ts = ts_.data();
    for (uint32_t v = ((uint32_t)K_ + leaf) >> 1; v >= 1; v >>= 1) {
      // swap (loser <-> candidate) when the stored loser beats the candidate; masks, no branches
      const uint64_t lk = tk[v];
      const uint32_t ls = ts[v];
      const uint64_t sw = (uint64_t)((lk < nk) | ((lk == nk) & (ls < ns)));
      const uint64_t mk = 0 - sw;
      const uint32_t ms = 0u - (uint32_t)sw;
      const uint64_t dk = (lk ^ nk) & mk;
      const uint32_t ds = (ls ^ ns) & ms;
      tk[v] = lk ^ dk;
      ts[v] = ls ^ ds;
      nk ^= dk;
      ns ^= ds;
    }
    win_k_ = nk;
    win_s_ = ns;
    return out;
  }

 private:
  int K_;
  std::vector<uint64_t> tk_;
  std::vector<uint32_t> ts_;
  std::vector<const uint64_t*> cur_, end_;
  uint64_t win_k_ = 0;
  uint32_t win_s_ = 0;
};

// Non-temporal 8-byte store (MOVNTI): the merge output is written once and not re-read, so it
// bypasses the cache and avoids the read-for-ownership of B (host DRAM bytes).
inline void st_nt(uint64_t* p, uint64_t v) {
  _mm_stream_si64((long long*)p, (long long)v);
}

}  // namespace

// Exact co-ranks of output position o (ties in run order).  Same definition as K4 (merge.cu).
// Runs are given as (start pointer, length) pairs, so they may lie anywhere in memory (the
// PIPEMERGE working memory holds merged pairs and batches at rotating places).
void host_corank_runs(const uint64_t* const* run, const uint64_t* len, int k, uint64_t o,
                      uint64_t* ranks) {
  std::vector<uint64_t> lo(k), hi(k);
  uint64_t total = 0;
  for (int j = 0; j < k; ++j) {
    lo[j] = 0;
    hi[j] = len[j];
    total += len[j];
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
        const uint64_t* r = run[j];
        mn = std::min(mn, r[lo[j]]);
        mx = std::max(mx, r[hi[j] - 1]);
      }
    L = std::max(L, mn);
    H = std::min(H, mx);
    if (L >= H) break;
    uint64_t mid = L + ((H - L) >> 1), s = 0;
    std::vector<uint64_t> u(k);
    for (int j = 0; j < k; ++j) {
      u[j] = ub(run[j], lo[j], hi[j], mid);
      s += u[j];
    }
    if (s > o) { H = mid; hi = u; }
    else { L = mid + 1; lo = u; }
  }
  const uint64_t v = L;
  uint64_t lt = 0;
  std::vector<uint64_t> eq(k);
  for (int j = 0; j < k; ++j) {
    const uint64_t* r = run[j];
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
static void merge_range(const uint64_t* const* run, const uint64_t* rlen, int k, const uint64_t* ra,
                        const uint64_t* rb, uint64_t* out, bool out_f64) {
  int live = 0, last = -1;
  for (int j = 0; j < k; ++j)
    if (rb[j] > ra[j]) { ++live; last = j; }
  if (live == 0) return;
  if (live == 1) {
    const uint64_t* s = run[last] + ra[last];
    const uint64_t len = rb[last] - ra[last];
    if (out_f64)
      for (uint64_t i = 0; i < len; ++i) st_nt(out + i, from_key(s[i]));
    else
      for (uint64_t i = 0; i < len; ++i) st_nt(out + i, s[i]);
    return;
  }
  if (live == 2) {
    int a = -1, b = -1;
    for (int j = 0; j < k; ++j)
      if (rb[j] > ra[j]) (a < 0 ? a : b) = j;
    const uint64_t *p = run[a] + ra[a], *pe = run[a] + rb[a];
    const uint64_t *q = run[b] + ra[b], *qe = run[b] + rb[b];
    uint64_t* o = out;
    while (p < pe && q < qe) {
      const uint64_t x = *p, y = *q;
      const bool takep = x <= y;
      const uint64_t v = takep ? x : y;
      p += takep;
      q += !takep;
      st_nt(o++, out_f64 ? from_key(v) : v);
    }
    while (p < pe) { st_nt(o++, out_f64 ? from_key(*p) : *p); ++p; }
    while (q < qe) { st_nt(o++, out_f64 ? from_key(*q) : *q); ++q; }
    return;
  }
  // k >= 3: the range is cut into NI sub-ranges by exact co-ranks and NI loser trees are
  // advanced in lock step, so NI independent replay chains are in flight (each pop depends on the
  // previous one of its own tree only).
  constexpr int NI = 4;
  uint64_t total = 0;
  for (int j = 0; j < k; ++j) total += rb[j] - ra[j];
  uint64_t oa = 0;
  for (int j = 0; j < k; ++j) oa += ra[j];  // absolute output position of this range
  std::vector<uint64_t> cr((NI + 1) * (size_t)k);
  std::memcpy(&cr[0], ra, k * 8);
  std::memcpy(&cr[(size_t)NI * k], rb, k * 8);
  for (int i = 1; i < NI; ++i) host_corank_runs(run, rlen, k, oa + total * i / NI, &cr[(size_t)i * k]);
  LoserTree* lt[NI];
  alignas(64) unsigned char mem[NI][sizeof(LoserTree)];
  uint64_t len[NI], pos[NI];
  for (int i = 0; i < NI; ++i) {
    lt[i] = new (mem[i]) LoserTree(k);
    len[i] = 0;
    for (int j = 0; j < k; ++j) {
      lt[i]->set_leaf(j, run[j] + cr[(size_t)i * k + j], run[j] + cr[(size_t)(i + 1) * k + j]);
      len[i] += cr[(size_t)(i + 1) * k + j] - cr[(size_t)i * k + j];
    }
    pos[i] = i == 0 ? 0 : pos[i - 1] + len[i - 1];
    lt[i]->build();
  }
  uint64_t m = len[0];
  for (int i = 1; i < NI; ++i) m = std::min(m, len[i]);
  if (out_f64) {
    for (uint64_t t = 0; t < m; ++t)
      for (int i = 0; i < NI; ++i) st_nt(out + pos[i] + t, from_key(lt[i]->pop()));
  } else {
    for (uint64_t t = 0; t < m; ++t)
      for (int i = 0; i < NI; ++i) st_nt(out + pos[i] + t, lt[i]->pop());
  }
  for (int i = 0; i < NI; ++i) {
    for (uint64_t t = m; t < len[i]; ++t) {
      const uint64_t v = lt[i]->pop();
      st_nt(out + pos[i] + t, out_f64 ? from_key(v) : v);
    }
    lt[i]->~LoserTree();
  }
}

// Merge positions [o_lo, o_hi) of the multiway merge of the k runs run[j][0 .. len[j]) into
// out[0 .. o_hi - o_lo).  The range is cut into ~4 pieces per thread by exact co-ranks.
void host_merge_runs_range(const uint64_t* const* run, const uint64_t* len, int k, uint64_t o_lo,
                           uint64_t o_hi, uint64_t* out, bool out_f64, int threads,
                           ThreadPool* pool) {
  if (threads <= 0) threads = host_threads();
  ThreadPool& tp = pool ? *pool : host_pool();
  uint64_t total = 0;
  for (int j = 0; j < k; ++j) total += len[j];
  if (o_hi > total) o_hi = total;
  if (o_lo >= o_hi) return;
  const uint64_t span = o_hi - o_lo;
  // ranges: ~4 per thread, each at least 64K keys
  int64_t R = std::max<int64_t>(1, std::min<int64_t>((int64_t)threads * 4, (int64_t)(span >> 16)));
  std::vector<uint64_t> ranks((R + 1) * (uint64_t)k);
  auto pos = [&](int64_t r) { return o_lo + (uint64_t)((__uint128_t)span * (uint64_t)r / (uint64_t)R); };
  tp.parallel_for(R + 1, threads, [&](int64_t r) {
    host_corank_runs(run, len, k, pos(r), &ranks[(uint64_t)r * k]);
  });
  tp.parallel_for(R, threads, [&](int64_t r) {
    merge_range(run, len, k, &ranks[(uint64_t)r * k], &ranks[(uint64_t)(r + 1) * k],
                out + (pos(r) - o_lo), out_f64);
    _mm_sfence();
  });
}

namespace {
struct RunView {  // (pointer, length) view of runs stored back to back: keys[off[j] .. off[j+1])
  std::vector<const uint64_t*> p;
  std::vector<uint64_t> len;
  RunView(const uint64_t* keys, const uint64_t* off, int k) : p(k), len(k) {
    for (int j = 0; j < k; ++j) {
      p[j] = keys + off[j];
      len[j] = off[j + 1] - off[j];
    }
  }
};
}  // namespace

void host_corank(const uint64_t* keys, const uint64_t* off, int k, uint64_t o, uint64_t* ranks) {
  RunView v(keys, off, k);
  host_corank_runs(v.p.data(), v.len.data(), k, o, ranks);
}

void host_merge_range(const uint64_t* keys, const uint64_t* off, int k, uint64_t o_lo,
                      uint64_t o_hi, uint64_t* out, bool out_f64, int threads) {
  RunView v(keys, off, k);
  host_merge_runs_range(v.p.data(), v.len.data(), k, o_lo, o_hi, out, out_f64, threads, nullptr);
}

void host_merge(const uint64_t* keys, const uint64_t* off, int k, uint64_t* out, bool out_f64,
                int threads) {
  host_merge_range(keys, off, k, 0, off[k] - off[0], out, out_f64, threads);
}

}  // namespace hsort
