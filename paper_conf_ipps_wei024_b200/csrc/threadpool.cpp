// threadpool.cpp — persistent host worker pool behind parallel_for / parallel_dyn (internal.h).
#include <condition_variable>
#include <mutex>

#include "internal.h"

namespace gcsm {

namespace {

class Pool {
 public:
  Pool() {
    const int n = (int)std::max(1u, std::thread::hardware_concurrency());
    for (int i = 1; i < n; ++i) workers_.emplace_back([this, i] { loop(i); });
    size_ = n;
  }
  ~Pool() {
    {
      std::lock_guard<std::mutex> g(mu_);
      stop_ = true;
      ++gen_;
    }
    cv_.notify_all();
    for (auto &t : workers_) t.join();
  }
  int size() const { return size_; }
  void run(int nthreads, const std::function<void(int)> &fn) {
    std::lock_guard<std::mutex> serial(run_mu_);
    if (nthreads > size_) nthreads = size_;
    {
      std::lock_guard<std::mutex> g(mu_);
      job_ = &fn;
      job_threads_ = nthreads;
      remaining_ = nthreads - 1;
      ++gen_;
    }
    cv_.notify_all();
    fn(0);
    std::unique_lock<std::mutex> lk(mu_);
    done_cv_.wait(lk, [this] { return remaining_ == 0; });
    job_ = nullptr;
  }

 private:
  void loop(int id) {
    uint64_t seen = 0;
    for (;;) {
      const std::function<void(int)> *job = nullptr;
      {
        std::unique_lock<std::mutex> lk(mu_);
        cv_.wait(lk, [&] { return gen_ != seen; });
        seen = gen_;
        if (stop_) return;
        if (id >= job_threads_) continue;
        job = job_;
      }
      (*job)(id);
      {
        std::lock_guard<std::mutex> g(mu_);
        if (--remaining_ == 0) done_cv_.notify_one();
      }
    }
  }
  std::vector<std::thread> workers_;
  std::mutex mu_, run_mu_;
  std::condition_variable cv_, done_cv_;
  const std::function<void(int)> *job_ = nullptr;
  int job_threads_ = 0, remaining_ = 0, size_ = 1;
  uint64_t gen_ = 0;
  bool stop_ = false;
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
