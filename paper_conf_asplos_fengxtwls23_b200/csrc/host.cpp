// Host thread pool + AdamW (K12 of SURVEY §2.2).  One fused pass per
// element: read grad (2 or 4 B), master/m/v (12 B), write master/m/v (12 B)
// and the new transfer-precision weight (2 or 4 B) = 28 B/param on the bf16
// path.  Auto-vectorised (AVX-512 / AVX2 clones).
#include "host.h"

#include <cmath>
#include <cstring>

namespace mobius {

ThreadPool::ThreadPool(int n) {
  for (int i = 0; i < n - 1; ++i) workers_.emplace_back([this] { loop(); });
}

ThreadPool::~ThreadPool() {
  {
    std::lock_guard<std::mutex> g(mu_);
    stop_ = true;
  }
  cv_.notify_all();
  for (auto& t : workers_) t.join();
}

void ThreadPool::loop() {
  uint64_t seen = 0;
  for (;;) {
    std::unique_lock<std::mutex> lk(mu_);
    cv_.wait(lk, [&] { return stop_ || (gen_ != seen && next_ < n_tasks_); });
    if (stop_) return;
    seen = gen_;
    while (next_ < n_tasks_) {
      int i = next_++;
      const std::function<void(int)>* fn = fn_;
      lk.unlock();
      (*fn)(i);
      lk.lock();
      if (--pending_ == 0) done_cv_.notify_all();
    }
  }
}

void ThreadPool::parallel_for(int n_tasks, const std::function<void(int)>& fn) {
  if (n_tasks <= 0) return;
  std::unique_lock<std::mutex> lk(mu_);
  fn_ = &fn;
  n_tasks_ = n_tasks;
  next_ = 0;
  pending_ = n_tasks;
  ++gen_;
  cv_.notify_all();
  while (next_ < n_tasks_) {
    int i = next_++;
    lk.unlock();
    fn(i);
    lk.lock();
    --pending_;
  }
  done_cv_.wait(lk, [&] { return pending_ == 0; });
  fn_ = nullptr;
  n_tasks_ = 0;
}

uint16_t f32_to_bf16_rne(float f) {
  uint32_t u;
  std::memcpy(&u, &f, 4);
  u += 0x7FFFu + ((u >> 16) & 1u);
  return (uint16_t)(u >> 16);
}
float bf16_to_f32(uint16_t b) {
  uint32_t u = (uint32_t)b << 16;
  float f;
  std::memcpy(&f, &u, 4);
  return f;
}

namespace {

template <int GK, int WK>
__attribute__((target_clones("avx512f", "avx2", "default"))) void adamw_chunk(
    float* __restrict__ w, float* __restrict__ m, float* __restrict__ v, const void* __restrict__ gp,
    void* __restrict__ wo, int64_t n, float lr, float b1, float b2, float eps, float wd, float bc1, float bc2) {
  const uint16_t* gb = (const uint16_t*)gp;
  const float* gf = (const float*)gp;
  uint16_t* wob = (uint16_t*)wo;
  float* wof = (float*)wo;
  const float omb1 = 1.f - b1, omb2 = 1.f - b2, lrwd = lr * wd;
  for (int64_t i = 0; i < n; ++i) {
    float g;
    if (GK == 0) {
      uint32_t u = (uint32_t)gb[i] << 16;
      std::memcpy(&g, &u, 4);
    } else {
      g = gf[i];
    }
    float x = w[i];
    x = x - lrwd * x;
    float mi = b1 * m[i] + omb1 * g;
    float vi = b2 * v[i] + omb2 * g * g;
    x = x - lr * (mi / bc1) / (std::sqrt(vi / bc2) + eps);
    m[i] = mi;
    v[i] = vi;
    w[i] = x;
    if (WK == 0) {
      uint32_t u;
      std::memcpy(&u, &x, 4);
      u += 0x7FFFu + ((u >> 16) & 1u);
      wob[i] = (uint16_t)(u >> 16);
    } else {
      wof[i] = x;
    }
  }
}

}  // namespace

void adamw_update(float* master, float* m, float* v, const void* grad, int grad_kind, void* weights_out,
                  int weights_kind, int64_t n, const AdamWArgs& a, ThreadPool& pool) {
  const float bc1 = (float)(1.0 - std::pow((double)a.beta1, (double)a.step));
  const float bc2 = (float)(1.0 - std::pow((double)a.beta2, (double)a.step));
  const int64_t chunk = 1 << 16;
  const int tasks = (int)((n + chunk - 1) / chunk);
  const int gs = grad_kind == 0 ? 2 : 4, ws = weights_kind == 0 ? 2 : 4;
  pool.parallel_for(tasks, [&](int t) {
    int64_t b = (int64_t)t * chunk, e = std::min<int64_t>(n, b + chunk);
    const void* g = (const char*)grad + b * gs;
    void* wo = (char*)weights_out + b * ws;
    if (grad_kind == 0 && weights_kind == 0)
      adamw_chunk<0, 0>(master + b, m + b, v + b, g, wo, e - b, a.lr, a.beta1, a.beta2, a.eps, a.wd, bc1, bc2);
    else if (grad_kind == 1 && weights_kind == 1)
      adamw_chunk<1, 1>(master + b, m + b, v + b, g, wo, e - b, a.lr, a.beta1, a.beta2, a.eps, a.wd, bc1, bc2);
    else if (grad_kind == 0)
      adamw_chunk<0, 1>(master + b, m + b, v + b, g, wo, e - b, a.lr, a.beta1, a.beta2, a.eps, a.wd, bc1, bc2);
    else
      adamw_chunk<1, 0>(master + b, m + b, v + b, g, wo, e - b, a.lr, a.beta1, a.beta2, a.eps, a.wd, bc1, bc2);
  });
}

}  // namespace mobius
