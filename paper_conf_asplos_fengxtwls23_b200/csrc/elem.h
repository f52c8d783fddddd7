// Fused HBM-bound kernels of the block / embedding / head (K5-K8, K10 of
// SURVEY §2.2).  T is the path type (__nv_bfloat16 or float); reductions
// and statistics are fp32.  All launchers are asynchronous on `s` and
// return a mobius_status.
#pragma once

#include <cstdint>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

namespace mobius {

// Workspace of the deterministic column reductions (colsum_accum, the
// LayerNorm parameter gradients): per-CTA partial sums and one arrival
// counter per column slab.  The counters must be zero before the first
// launch (the last CTA of a slab resets its counter), `part` holds
// colsum_ws_floats(rows, n, planes) floats.
struct RedWs {
  float* part = nullptr;
  unsigned* cnt = nullptr;   // RED_WS_COUNTERS entries
};
constexpr int RED_WS_COUNTERS = 1024;
int64_t colsum_ws_floats(int rows, int n, int planes);

// x0[r, :] = wte[tok(r)] + wpe[r % s],  r = b*s + i,  tok(r) = tok[b*(s+1) + i]
template <typename T>
int embed_fwd(const int32_t* tok, const T* wte, const T* wpe, T* x, int mbs, int s, int h, cudaStream_t st);
// dwte[tok(r)] += dx[r];  dwpe[i] += sum_b dx[b*s + i]   (fp32 accumulators).
// fp32 path deterministic (every dwte row owned by one CTA, which adds the
// rows of its tokens in position order, no atomics); bf16 path: vector
// reductions.  Token ids must be in [0, V) (mobius_step validates them).
template <typename T>
int embed_bwd(const int32_t* tok, const T* dx, float* dwte, float* dwpe, int mbs, int s, int h, int V,
              cudaStream_t st);

// y = g (x - mu) rstd + b over rows of length h; saves mu, rstd (fp32)
template <typename T>
int layernorm_fwd(const T* x, const T* g, const T* b, T* y, float* mu, float* rstd, int rows, int h, cudaStream_t st);
// dx = rstd (g dy - mean(g dy) - xhat mean(g dy xhat)) [+ dres];  dg += sum dy xhat; db += sum dy;
// and, if dres_sum is given, dres_sum += sum over rows of dres (the column
// sum of the residual gradient, e.g. the bias gradient of the layer whose
// output it is) - all sums in a fixed order: bitwise reproducible
template <typename T>
int layernorm_bwd(const T* dy, const T* x, const T* g, const float* mu, const float* rstd, const T* dres, T* dx,
                  float* dg, float* db, int rows, int h, const RedWs& ws, cudaStream_t st, float* dres_sum = nullptr);
// kernels one layernorm_bwd call launches
template <typename T>
int layernorm_bwd_launches(int h, bool dres, bool dres_sum);

// Causal row softmax of S (fp32, [B][s][s], row stride s) scaled by `scale`:
// P[i, j] = softmax_j<=i(scale S[i, :]) and 0 for i < j < roundup(i+1, 128).
template <typename T>
int softmax_causal_fwd(const float* S, T* P, int B, int s, float scale, cudaStream_t st);
// dS = scale * P (dP - sum_j P dP) on j <= i, 0 for i < j < roundup(i+1,128)
template <typename T>
int softmax_causal_bwd(const T* P, const float* dP, T* dS, int B, int s, float scale, cudaStream_t st);

// Row-wise cross entropy on logits [rows][V] (in place -> dlogits):
// loss_rows[r] = logsumexp(z_r) - z_r[t_r];  dz = (softmax(z) - onehot) * inv_ntok.
// t_r = tok[b*(s+1) + i + 1] for r = b*s + i.
template <typename T>
int cross_entropy_fwd_bwd(T* logits, const int32_t* tok, float* loss_rows, int rows, int V, int s, float inv_ntok,
                          cudaStream_t st);
// acc[0] += sum(loss_rows)  (double, single block: deterministic)
int loss_accumulate(const float* loss_rows, int rows, double* acc, cudaStream_t st);

// out[n] += sum_r X[r, n] (fp32 out), X row stride ld.  Per-CTA partials
// are summed in CTA order by the slab's last CTA: bitwise reproducible.
template <typename T>
int colsum_accum(const T* X, int64_t ld, int rows, int n, float* out, const RedWs& ws, cudaStream_t st);

// g = gelu_tanh(u) elementwise, the same arithmetic (tanh.approx, bf16
// rounding of the result) as the GEMM's EPI_BIAS_GELU epilogue, so a
// recomputed g is bit-identical to the one the forward wrote (bf16 only).
int gelu_fwd_bf16(const __nv_bfloat16* u, __nv_bfloat16* g, int64_t n, cudaStream_t st);

// dst = (T) src
template <typename T>
int cast_from_f32(const float* src, T* dst, int64_t n, cudaStream_t st);
// AdamW on device-resident fp32 master/m/v (the host update's formula,
// host.cpp adamw_chunk): g is the stage gradient in transfer precision T,
// w_out the new weights in T.  bc1 = 1 - b1^t, bc2 = 1 - b2^t.
template <typename T>
int adamw_device(float* w, float* m, float* v, const T* g, T* w_out, int64_t n, float lr, float b1, float b2,
                 float eps, float wd, float bc1, float bc2, cudaStream_t st);

// p[r][0..63] = (1, 0, ..., 0) for r < rows: the ones block the weight-
// gradient GEMM loads as the extra A row that yields the bias gradient
template <typename T>
int fill_ones_col(T* p, int rows, cudaStream_t st);

// dst = src (n token ids) and *bad_dev (device int) = number of ids outside [0, V)
int tokens_check_copy(const int32_t* src, int32_t* dst, int64_t n, int V, int* bad_dev, cudaStream_t st);

// device-side flag wait / set (inter-rank arrival flags, release/acquire at system scope)
int flag_wait(const volatile int* flag, int value, cudaStream_t st);
int flag_set(int* flag, int value, cudaStream_t st);
// *out = atomicAdd_system(counter, 1) (prefetch-chain tickets; counter may be peer memory)
int ticket_take(int* counter, int* out, cudaStream_t st);

}  // namespace mobius
