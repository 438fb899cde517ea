// threadpool.cpp — persistent host worker pool behind parallel_for / parallel_dyn (internal.h).
#include <immintrin.h>

#include <atomic>
#include <condition_variable>
#include <mutex>

#include "internal.h"

namespace gcsm {

namespace {

// Workers spin on a generation counter for a short while after each job (a batch issues tens of parallel
// regions back to back: parking and waking 15 threads per region cost ~0.1 ms each) and park on a condition
// variable when the pool stays idle. run() calls from different host threads are serialised.
class Pool {
 public:
  Pool() {
    const int n = (int)std::max(1u, std::thread::hardware_concurrency());
    size_ = n;
    for (int i = 1; i < n; ++i) workers_.emplace_back([this, i] { loop(i); });
  }
  ~Pool() {
    {
      std::lock_guard<std::mutex> g(mu_);
      stop_.store(true);
      gen_.fetch_add(1);
    }
    cv_.notify_all();
    for (auto &t : workers_) t.join();
  }
  int size() const { return size_; }
  void run(int nthreads, const std::function<void(int)> &fn) {
    std::lock_guard<std::mutex> serial(run_mu_);
    if (nthreads > size_) nthreads = size_;
    job_ = &fn;
    job_threads_ = nthreads;
    // every worker acknowledges every generation (idle ids included), so no worker can still be reading this
    // job's parameters when the next run() overwrites them
    remaining_.store(size_ - 1);
    gen_.fetch_add(1);  // seq_cst: ordered before the parked_ check (see loop())
    if (parked_.load() > 0) {
      std::lock_guard<std::mutex> g(mu_);
      cv_.notify_all();
    }
    fn(0);
    while (remaining_.load(std::memory_order_acquire) != 0) _mm_pause();
    job_ = nullptr;
  }

 private:
  static constexpr int kSpin = 1 << 16;  // ~0.2-0.5 ms of pause loops before parking
  void loop(int id) {
    uint64_t seen = 0;
    for (;;) {
      uint64_t g;
      int spins = 0;
      while ((g = gen_.load(std::memory_order_acquire)) == seen) {
        if (++spins < kSpin) {
          _mm_pause();
          continue;
        }
        std::unique_lock<std::mutex> lk(mu_);
        parked_.fetch_add(1);  // seq_cst: either run() sees it and notifies, or we see the new generation
        cv_.wait(lk, [&] { return gen_.load() != seen; });
        parked_.fetch_sub(1);
        spins = 0;
      }
      seen = g;
      if (stop_.load()) return;
      if (id < job_threads_) (*job_)(id);
      remaining_.fetch_sub(1, std::memory_order_release);
    }
  }
  std::vector<std::thread> workers_;
  std::mutex mu_, run_mu_;
  std::condition_variable cv_;
  const std::function<void(int)> *job_ = nullptr;
  int job_threads_ = 0, size_ = 1;
  std::atomic<int> remaining_{0}, parked_{0};
  std::atomic<uint64_t> gen_{0};
  std::atomic<bool> stop_{false};
};

Pool &pool() {
  static Pool p;
  return p;
}

}  // namespace

void pool_run(int nthreads, const std::function<void(int)> &fn) {
  if (nthreads <= 1) {
    fn(0);
    return;
  }
  pool().run(nthreads, fn);
}

int pool_size() { return pool().size(); }

}  // namespace gcsm
