// pool.h — host worker pool for PARMEMCPY and the CPU multiway merge
// (P:237-249).  std::thread based (no OpenMP runtime inside a library loaded next to torch).
#pragma once
#include <atomic>
#include <condition_variable>
#include <cstdint>
#include <deque>
#include <functional>
#include <memory>
#include <mutex>
#include <thread>
#include <vector>

namespace hsort {

class ThreadPool {
 public:
  explicit ThreadPool(int n_workers);
  ~ThreadPool();
  ThreadPool(const ThreadPool&) = delete;
  ThreadPool& operator=(const ThreadPool&) = delete;

  // Run fn(i) for i in [0, tasks) using the calling thread plus up to width-1 pool workers;
  // returns when every task has finished.  Safe to call concurrently from several threads.
  void parallel_for(int64_t tasks, int width, const std::function<void(int64_t)>& fn);
  int size() const { return (int)workers_.size(); }

 private:
  struct Job {
    std::atomic<int64_t> next{0};
    std::atomic<int64_t> done{0};
    int64_t tasks = 0;
    const std::function<void(int64_t)>* fn = nullptr;
    std::mutex m;
    std::condition_variable cv;
  };
  static void drain(Job& j);
  void loop();
  std::vector<std::thread> workers_;
  std::deque<std::shared_ptr<Job>> queue_;
  std::mutex m_;
  std::condition_variable cv_;
  bool stop_ = false;
};

// Process-wide pool (created on first use, sized to the hardware threads).
ThreadPool& host_pool();
// Second pool for the PIPEMERGE pair merges that run during the sort phase, so they never queue
// ahead of the PARMEMCPY staging jobs on host_pool() (half the hardware threads).
ThreadPool& pipe_pool();
// Pool of the STREAM merge phase's CPU share, so its loser-tree tasks never queue ahead of the
// GPU share's staging copies on host_pool() (they ran FIFO on one pool in round 1).
ThreadPool& merge_pool();
int host_threads();

// PARMEMCPY: dst <- src (bytes) split over `threads` workers (0 = all host threads).
extern bool g_memcpy_nt;  // PARMEMCPY streaming stores (option "memcpy_nt", default on)
void par_memcpy(void* dst, const void* src, uint64_t bytes, int threads);

}  // namespace hsort
