// pool.cpp — host worker pool and PARMEMCPY (§III-D2: "if host-to-host MCpy
// to/from pinned memory in Stage is a bottleneck when using std::memcpy, we can parallelize this
// step on the host").
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

ThreadPool& pipe_pool() {
  static ThreadPool pool(std::max(1, host_threads() / 2 - 1));
  return pool;
}

void par_memcpy(void* dst, const void* src, uint64_t bytes, int threads) {
  if (threads <= 0) threads = host_threads();
  constexpr uint64_t kMinChunk = 2ull << 20;
  if (threads == 1 || bytes < 2 * kMinChunk) {
    std::memcpy(dst, src, bytes);
    return;
  }
  int64_t tasks = (int64_t)std::min<uint64_t>((uint64_t)threads * 2, bytes / kMinChunk);
  uint64_t chunk = ((bytes + tasks - 1) / tasks + 63) & ~63ull;
  host_pool().parallel_for(tasks, threads, [&](int64_t t) {
    uint64_t lo = (uint64_t)t * chunk;
    if (lo >= bytes) return;
    uint64_t len = std::min<uint64_t>(chunk, bytes - lo);
    std::memcpy((char*)dst + lo, (const char*)src + lo, len);
  });
}

}  // namespace hsort
