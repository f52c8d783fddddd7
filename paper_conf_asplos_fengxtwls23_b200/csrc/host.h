// Host-side helpers: a persistent thread pool and the per-stage AdamW
// update that runs "in DRAM" on the offloaded gradients (row a11;
// PAPER P:L462-463 "transferred to DRAM for parameter update"; optimizer
// choice = reading #16).
#pragma once

#include <condition_variable>
#include <cstdint>
#include <functional>
#include <mutex>
#include <thread>
#include <vector>

namespace mobius {

class ThreadPool {
 public:
  explicit ThreadPool(int n);
  ~ThreadPool();
  int size() const { return (int)workers_.size() + 1; }
  // run fn(i) for i in [0, n_tasks), caller participates; blocks until done
  void parallel_for(int n_tasks, const std::function<void(int)>& fn);

 private:
  void loop();
  std::vector<std::thread> workers_;
  std::mutex mu_;
  std::condition_variable cv_, done_cv_;
  const std::function<void(int)>* fn_ = nullptr;
  int n_tasks_ = 0, next_ = 0, pending_ = 0;
  uint64_t gen_ = 0;
  bool stop_ = false;
};

struct AdamWArgs {
  float lr, beta1, beta2, eps, wd;
  int64_t step;  // 1-based
};

// One AdamW step over n elements.  grad_kind: 0 = bf16 bits, 1 = fp32.
// weights_out_kind: 0 = bf16 bits (RNE of the new master), 1 = fp32.
void adamw_update(float* master, float* m, float* v, const void* grad, int grad_kind, void* weights_out,
                  int weights_kind, int64_t n, const AdamWArgs& a, ThreadPool& pool);

uint16_t f32_to_bf16_rne(float f);
float bf16_to_f32(uint16_t b);

}  // namespace mobius
