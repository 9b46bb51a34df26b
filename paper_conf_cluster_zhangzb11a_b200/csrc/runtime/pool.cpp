#include "pool.h"

#include <algorithm>
#include <atomic>
#include <chrono>
#include <condition_variable>
#include <cstdlib>
#include <mutex>
#include <thread>
#include <vector>

namespace gpa {
namespace {

thread_local bool t_inside = false;   // inside a parallel region (pool workers always are)

class Pool {
 public:
  Pool() {
    unsigned hw = std::thread::hardware_concurrency();
    size_t n = hw ? hw : 1;
    if (const char* e = std::getenv("GPA_HOST_THREADS")) n = std::max(1, atoi(e));
    n = std::min<size_t>(n, 64);
    for (size_t i = 1; i < n; ++i) workers_.emplace_back([this] { loop(); });
    size_ = n;
  }
  ~Pool() {
    {
      std::lock_guard<std::mutex> lk(mu_);
      stop_ = true;
    }
    cv_.notify_all();
    for (auto& t : workers_) t.join();
  }
  size_t size() const { return size_; }

  void run(size_t n, const std::function<void(size_t)>& f) {
    if (n == 0) return;
    if (n == 1 || size_ == 1 || t_inside) {
      for (size_t i = 0; i < n; ++i) f(i);
      return;
    }
    std::lock_guard<std::mutex> region(region_mu_);
    {
      std::lock_guard<std::mutex> lk(mu_);
      fn_ = &f;
      n_ = n;
      next_.store(0);
      pending_ = workers_.size();
      ++gen_;
    }
    cv_.notify_all();
    t_inside = true;
    work();
    t_inside = false;
    std::unique_lock<std::mutex> lk(mu_);
    done_cv_.wait(lk, [this] { return pending_ == 0; });
    fn_ = nullptr;
  }

 private:
  void work() {
    for (;;) {
      size_t i = next_.fetch_add(1);
      if (i >= n_) break;
      (*fn_)(i);
    }
  }
  void loop() {
    t_inside = true;
    size_t seen = 0;
    for (;;) {
      {
        std::unique_lock<std::mutex> lk(mu_);
        cv_.wait(lk, [&] { return stop_ || gen_ != seen; });
        if (stop_) return;
        seen = gen_;
      }
      work();
      {
        std::lock_guard<std::mutex> lk(mu_);
        if (--pending_ == 0) done_cv_.notify_one();
      }
    }
  }
  std::vector<std::thread> workers_;
  size_t size_ = 1;
  std::mutex mu_, region_mu_;
  std::condition_variable cv_, done_cv_;
  const std::function<void(size_t)>* fn_ = nullptr;
  size_t n_ = 0, pending_ = 0, gen_ = 0;
  std::atomic<size_t> next_{0};
  bool stop_ = false;
};

Pool& pool() {
  static Pool p;
  return p;
}

}  // namespace

size_t pool_threads() { return pool().size(); }

bool trace_enabled() {
  static const bool on = [] {
    const char* e = std::getenv("GPA_TRACE");
    return e && *e && *e != '0';
  }();
  return on;
}

double wall_ms() {
  return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now().time_since_epoch()).count();
}
void parallel_for(size_t n, const std::function<void(size_t)>& f) { pool().run(n, f); }

}  // namespace gpa
