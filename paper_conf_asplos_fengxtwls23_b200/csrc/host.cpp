// Host thread pool + AdamW (K12 of SURVEY §2.2).  One fused pass per
// element: read grad (2 or 4 B), master/m/v (12 B), write master/m/v (12 B)
// and the new transfer-precision weight (2 or 4 B) = 28 B/param on the bf16
// path.  Auto-vectorised (AVX-512 / AVX2 clones).
#include "host.h"

#include <immintrin.h>

#include <cmath>
#include <cstdlib>
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

// bf16 grad -> bf16 weights (the bf16 path), explicit AVX-512: 16 params
// per iteration, the two bias-correction divisions folded into multiplies,
// and non-temporal stores for master/m/v/weights (no read-for-ownership:
// 28 B/param of DRAM traffic instead of ~42).  Same AdamW as adamw_chunk to
// fp32 rounding (FMA contraction and the folded reciprocals differ in the
// last bits; the oracle parity test allows 1e-6).
__attribute__((target("avx512f,avx512bw,avx512vl"))) void adamw_chunk_bf16_avx512(
    float* __restrict__ w, float* __restrict__ m, float* __restrict__ v, const uint16_t* __restrict__ g,
    uint16_t* __restrict__ wo, int64_t n, float lr, float b1, float b2, float eps, float wd, float bc1, float bc2) {
  const __m512 vb1 = _mm512_set1_ps(b1), vb2 = _mm512_set1_ps(b2);
  const __m512 vomb1 = _mm512_set1_ps(1.f - b1), vomb2 = _mm512_set1_ps(1.f - b2);
  const __m512 vlr = _mm512_set1_ps(lr), vlrwd = _mm512_set1_ps(lr * wd), veps = _mm512_set1_ps(eps);
  const __m512 vr1 = _mm512_set1_ps(1.f / bc1), vr2 = _mm512_set1_ps(1.f / bc2);
  const __m512i rnd = _mm512_set1_epi32(0x7FFF), one = _mm512_set1_epi32(1);
  const bool nt = ((reinterpret_cast<uintptr_t>(w) | reinterpret_cast<uintptr_t>(m) | reinterpret_cast<uintptr_t>(v)) &
                   63) == 0 &&
                  (reinterpret_cast<uintptr_t>(wo) & 31) == 0;
  int64_t i = 0;
  for (; i + 16 <= n; i += 16) {
    const __m256i gb = _mm256_loadu_si256(reinterpret_cast<const __m256i*>(g + i));
    const __m512 gv = _mm512_castsi512_ps(_mm512_slli_epi32(_mm512_cvtepu16_epi32(gb), 16));
    __m512 x = _mm512_loadu_ps(w + i);
    x = _mm512_fnmadd_ps(vlrwd, x, x);
    const __m512 mi = _mm512_fmadd_ps(vb1, _mm512_loadu_ps(m + i), _mm512_mul_ps(vomb1, gv));
    const __m512 vi = _mm512_fmadd_ps(vb2, _mm512_loadu_ps(v + i), _mm512_mul_ps(_mm512_mul_ps(vomb2, gv), gv));
    const __m512 den = _mm512_add_ps(_mm512_sqrt_ps(_mm512_mul_ps(vi, vr2)), veps);
    x = _mm512_sub_ps(x, _mm512_div_ps(_mm512_mul_ps(vlr, _mm512_mul_ps(mi, vr1)), den));
    // round-to-nearest-even to bf16
    const __m512i u = _mm512_castps_si512(x);
    const __m512i r = _mm512_add_epi32(u, _mm512_add_epi32(rnd, _mm512_and_si512(_mm512_srli_epi32(u, 16), one)));
    const __m256i wb = _mm512_cvtepi32_epi16(_mm512_srli_epi32(r, 16));
    if (nt) {
      _mm512_stream_ps(m + i, mi);
      _mm512_stream_ps(v + i, vi);
      _mm512_stream_ps(w + i, x);
      _mm256_stream_si256(reinterpret_cast<__m256i*>(wo + i), wb);
    } else {
      _mm512_storeu_ps(m + i, mi);
      _mm512_storeu_ps(v + i, vi);
      _mm512_storeu_ps(w + i, x);
      _mm256_storeu_si256(reinterpret_cast<__m256i*>(wo + i), wb);
    }
  }
  _mm_sfence();  // non-temporal stores visible before the chunk is reported done
  if (i < n)
    adamw_chunk<0, 0>(w + i, m + i, v + i, g + i, wo + i, n - i, lr, b1, b2, eps, wd, bc1, bc2);
}

bool have_avx512() {  // MOBIUS_ADAMW_SCALAR=1 forces the portable loop (A/B checks)
  static const int ok = __builtin_cpu_supports("avx512f") && __builtin_cpu_supports("avx512bw") &&
                        __builtin_cpu_supports("avx512vl") && !std::getenv("MOBIUS_ADAMW_SCALAR");
  return ok != 0;
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
    if (grad_kind == 0 && weights_kind == 0 && have_avx512())
      adamw_chunk_bf16_avx512(master + b, m + b, v + b, (const uint16_t*)g, (uint16_t*)wo, e - b, a.lr, a.beta1,
                              a.beta2, a.eps, a.wd, bc1, bc2);
    else if (grad_kind == 0 && weights_kind == 0)
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
