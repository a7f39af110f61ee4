// pool.cpp — host worker pool and PARMEMCPY (§III-D2: "if host-to-host MCpy
// to/from pinned memory in Stage is a bottleneck when using std::memcpy, we can parallelize this
// step on the host").
#include <emmintrin.h>
#include "pool.h"

#include <algorithm>
#include <cstring>

namespace hsort {

ThreadPool::ThreadPool(int n_workers) {
  for (int i = 0; i < n_workers; ++i) workers_.emplace_back([this] { loop(); });
}

ThreadPool::~ThreadPool() {
  {
    std::lock_guard<std::mutex> g(m_);
    stop_ = true;
  }
  cv_.notify_all();
  for (auto& t : workers_) t.join();
}

void ThreadPool::drain(Job& j) {
  while (true) {
    int64_t i = j.next.fetch_add(1);
    if (i >= j.tasks) break;
    (*j.fn)(i);
    if (j.done.fetch_add(1) + 1 == j.tasks) {
      std::lock_guard<std::mutex> g(j.m);
      j.cv.notify_all();
    }
  }
}

void ThreadPool::loop() {
  while (true) {
    std::shared_ptr<Job> j;
    {
      std::unique_lock<std::mutex> lk(m_);
      cv_.wait(lk, [&] { return stop_ || !queue_.empty(); });
      if (stop_ && queue_.empty()) return;
      j = queue_.front();
      queue_.pop_front();
    }
    drain(*j);
  }
}

void ThreadPool::parallel_for(int64_t tasks, int width, const std::function<void(int64_t)>& fn) {
  if (tasks <= 0) return;
  if (width <= 1 || tasks == 1 || workers_.empty()) {
    for (int64_t i = 0; i < tasks; ++i) fn(i);
    return;
  }
  auto j = std::make_shared<Job>();
  j->tasks = tasks;
  j->fn = &fn;
  int helpers = (int)std::min<int64_t>(std::min<int64_t>(width - 1, tasks - 1), (int64_t)workers_.size());
  {
    std::lock_guard<std::mutex> g(m_);
    for (int h = 0; h < helpers; ++h) queue_.push_back(j);
  }
  if (helpers == 1) cv_.notify_one();
  else cv_.notify_all();
  drain(*j);
  std::unique_lock<std::mutex> lk(j->m);
  j->cv.wait(lk, [&] { return j->done.load() >= j->tasks; });
  // helpers that dequeue the job late find no task left; the shared_ptr keeps it alive
}

int host_threads() {
  unsigned h = std::thread::hardware_concurrency();
  return h ? (int)h : 4;
}

ThreadPool& host_pool() {
  static ThreadPool pool(host_threads() - 1 > 0 ? host_threads() - 1 : 1);
  return pool;
}

ThreadPool& merge_pool() {
  static ThreadPool pool(std::max(1, host_threads() - 1));
  return pool;
}

ThreadPool& pipe_pool() {
  static ThreadPool pool(std::max(1, host_threads() / 2 - 1));
  return pool;
}

bool g_memcpy_nt = true;  // option "memcpy_nt": streaming stores in PARMEMCPY

// memcpy with non-temporal 16-byte stores (SSE2): the destination is not read for ownership and
// does not displace the cache -- staging copies are write-once, read by DMA or by the caller later
static void memcpy_nt(void* dst, const void* src, uint64_t bytes) {
  char* d = (char*)dst;
  const char* s = (const char*)src;
  const uint64_t head = (16 - ((uintptr_t)d & 15)) & 15;
  if (bytes < head + 64) {
    std::memcpy(d, s, bytes);
    return;
  }
  std::memcpy(d, s, head);
  d += head;
  s += head;
  bytes -= head;
  const uint64_t body = bytes & ~63ull;
  for (uint64_t i = 0; i < body; i += 64) {
    const __m128i a = _mm_loadu_si128((const __m128i*)(s + i));
    const __m128i b = _mm_loadu_si128((const __m128i*)(s + i + 16));
    const __m128i c = _mm_loadu_si128((const __m128i*)(s + i + 32));
    const __m128i e = _mm_loadu_si128((const __m128i*)(s + i + 48));
    _mm_stream_si128((__m128i*)(d + i), a);
    _mm_stream_si128((__m128i*)(d + i + 16), b);
    _mm_stream_si128((__m128i*)(d + i + 32), c);
    _mm_stream_si128((__m128i*)(d + i + 48), e);
  }
  std::memcpy(d + body, s + body, bytes - body);
  _mm_sfence();
}

void par_memcpy(void* dst, const void* src, uint64_t bytes, int threads) {
  if (threads <= 0) threads = host_threads();
  constexpr uint64_t kMinChunk = 2ull << 20;
  if (threads == 1 || bytes < 2 * kMinChunk) {
    if (g_memcpy_nt && bytes >= kMinChunk) memcpy_nt(dst, src, bytes);
    else std::memcpy(dst, src, bytes);
    return;
  }
  int64_t tasks = (int64_t)std::min<uint64_t>((uint64_t)threads * 2, bytes / kMinChunk);
  uint64_t chunk = ((bytes + tasks - 1) / tasks + 63) & ~63ull;
  host_pool().parallel_for(tasks, threads, [&](int64_t t) {
    uint64_t lo = (uint64_t)t * chunk;
    if (lo >= bytes) return;
    uint64_t len = std::min<uint64_t>(chunk, bytes - lo);
    if (g_memcpy_nt) memcpy_nt((char*)dst + lo, (const char*)src + lo, len);
    else std::memcpy((char*)dst + lo, (const char*)src + lo, len);
  });
}

}  // namespace hsort
