// Kernel-level test entry points (include/mobius_kernels.h).  Each launches
// on the legacy default stream and synchronises, so a Python test can hand
// in torch device pointers and compare with the CPU oracle.
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <cstdlib>
#include <vector>

#include "../../include/mobius_kernels.h"
#include "common.h"
#include "elem.h"
#include "gemm.h"
#include "flash.h"
#include "ops.h"

using namespace mobius;
typedef __nv_bfloat16 bf16;

namespace {
// grow-only device workspace reused across kernel-test calls (no cudaMalloc
// inside timed loops)
uint8_t* ws_get(int64_t bytes) {
  static uint8_t* buf = nullptr;
  static int64_t cap = 0;
  if (bytes > cap) {
    if (buf) cudaFree(buf);
    buf = nullptr;
    if (cudaMalloc(&buf, bytes) != cudaSuccess) {
      cap = 0;
      return nullptr;
    }
    cap = bytes;
  }
  return buf;
}
// reduction workspace of the kt column sums (counters zeroed once; the
// reduction kernels leave them zero)
RedWs red_ws_get(int64_t floats) {
  static RedWs w;
  static int64_t cap = -1;
  if (floats > cap) {
    if (w.part) cudaFree(w.part);
    if (!w.cnt && cudaMalloc(&w.cnt, RED_WS_COUNTERS * 4) == cudaSuccess) cudaMemset(w.cnt, 0, RED_WS_COUNTERS * 4);
    w.part = nullptr;
    cap = -1;
    if (cudaMalloc(&w.part, floats * 4 + 16) != cudaSuccess) return RedWs{};
    cap = floats;
  }
  return w;
}
int sync_rc(int rc) {
  if (rc) return rc;
  static int nosync = -1;  // MOBIUS_KT_NOSYNC=1: timing loops (launch-only, errors via cudaGetLastError)
  if (nosync < 0) {
    const char* v = getenv("MOBIUS_KT_NOSYNC");
    nosync = (v && v[0] == '1') ? 1 : 0;
  }
  cudaError_t e = nosync ? cudaGetLastError() : cudaDeviceSynchronize();
  if (e != cudaSuccess) MOBIUS_FAIL(MOBIUS_ECUDA, "kernel failed: %s", cudaGetErrorString(e));
  return MOBIUS_OK;
}
MatView V(const void* p, int64_t ld, int64_t b1 = 0, int64_t b2 = 0) {
  MatView v;
  v.ptr = p;
  v.ld = ld;
  v.bs1 = b1;
  v.bs2 = b2;
  return v;
}
}  // namespace

extern "C" int mobius_kt_gemm(int dtype, int M, int N, int K, int nb1, int nb2, const void* A, int64_t lda,
                              int64_t abs1, int64_t abs2, int a_mn, const void* B, int64_t ldb, int64_t bbs1,
                              int64_t bbs2, int b_mn, void* C, int64_t ldc, int64_t cbs1, int64_t cbs2, int c_f32,
                              int epi, float alpha, const void* bias, const void* R, int64_t ldr, void* AUX,
                              int64_t ldx, int causal, int accumulate) {
  GemmDesc d;
  d.M = M; d.N = N; d.K = K; d.nb1 = nb1; d.nb2 = nb2;
  d.A = V(A, lda, abs1, abs2); d.a_mn = a_mn != 0;
  d.B = V(B, ldb, bbs1, bbs2); d.b_mn = b_mn != 0;
  d.C = V(C, ldc, cbs1, cbs2); d.c_f32 = c_f32 != 0;
  d.epi = epi; d.alpha = alpha; d.bias = bias;
  d.R = V(R, ldr); d.AUX = V(AUX, ldx);
  d.causal = causal; d.accumulate = accumulate != 0;
  return sync_rc(dtype == MOBIUS_BF16 ? gemm_bf16(d, 0) : gemm_f32(d, 0));
}

extern "C" int mobius_kt_gemm_config(int two_cta, int stream_k) {
  if (two_cta < -1 || two_cta > 1 || stream_k < -1 || stream_k > 1)
    MOBIUS_FAIL(MOBIUS_EINVAL, "gemm_config: modes are -1, 0 or 1");
  gemm_set_config(two_cta, stream_k);
  return MOBIUS_OK;
}

extern "C" int mobius_kt_layernorm_fwd(int dtype, const void* x, const void* g, const void* b, void* y, float* mu,
                                       float* rstd, int rows, int h) {
  if (dtype == MOBIUS_BF16)
    return sync_rc(layernorm_fwd<bf16>((const bf16*)x, (const bf16*)g, (const bf16*)b, (bf16*)y, mu, rstd, rows, h, 0));
  return sync_rc(layernorm_fwd<float>((const float*)x, (const float*)g, (const float*)b, (float*)y, mu, rstd, rows, h, 0));
}

extern "C" int mobius_kt_layernorm_bwd(int dtype, const void* dy, const void* x, const void* g, const float* mu,
                                       const float* rstd, const void* dres, void* dx, float* dg, float* db, int rows,
                                       int h) {
  const RedWs ws = red_ws_get(colsum_ws_floats(rows, h, 2));
  if (dtype == MOBIUS_BF16)
    return sync_rc(layernorm_bwd<bf16>((const bf16*)dy, (const bf16*)x, (const bf16*)g, mu, rstd, (const bf16*)dres,
                                       (bf16*)dx, dg, db, rows, h, ws, 0));
  return sync_rc(layernorm_bwd<float>((const float*)dy, (const float*)x, (const float*)g, mu, rstd,
                                      (const float*)dres, (float*)dx, dg, db, rows, h, ws, 0));
}

extern "C" int mobius_kt_softmax_fwd(int dtype, const float* S, void* P, int B, int s, float scale) {
  if (dtype == MOBIUS_BF16) return sync_rc(softmax_causal_fwd<bf16>(S, (bf16*)P, B, s, scale, 0));
  return sync_rc(softmax_causal_fwd<float>(S, (float*)P, B, s, scale, 0));
}

extern "C" int mobius_kt_softmax_bwd(int dtype, const void* P, const float* dP, void* dS, int B, int s, float scale) {
  if (dtype == MOBIUS_BF16) return sync_rc(softmax_causal_bwd<bf16>((const bf16*)P, dP, (bf16*)dS, B, s, scale, 0));
  return sync_rc(softmax_causal_bwd<float>((const float*)P, dP, (float*)dS, B, s, scale, 0));
}

extern "C" int mobius_kt_cross_entropy(int dtype, void* logits, const int32_t* tok, float* loss_rows, int rows, int V,
                                       int s, float inv_ntok) {
  if (dtype == MOBIUS_BF16)
    return sync_rc(cross_entropy_fwd_bwd<bf16>((bf16*)logits, tok, loss_rows, rows, V, s, inv_ntok, 0));
  return sync_rc(cross_entropy_fwd_bwd<float>((float*)logits, tok, loss_rows, rows, V, s, inv_ntok, 0));
}

extern "C" int mobius_kt_embed_fwd(int dtype, const int32_t* tok, const void* wte, const void* wpe, void* x, int mbs,
                                   int s, int h) {
  if (dtype == MOBIUS_BF16)
    return sync_rc(embed_fwd<bf16>(tok, (const bf16*)wte, (const bf16*)wpe, (bf16*)x, mbs, s, h, 0));
  return sync_rc(embed_fwd<float>(tok, (const float*)wte, (const float*)wpe, (float*)x, mbs, s, h, 0));
}

extern "C" int mobius_kt_embed_bwd(int dtype, const int32_t* tok, const void* dx, float* dwte, float* dwpe, int mbs,
                                   int s, int h, int V) {
  if (dtype == MOBIUS_BF16) return sync_rc(embed_bwd<bf16>(tok, (const bf16*)dx, dwte, dwpe, mbs, s, h, V, 0));
  return sync_rc(embed_bwd<float>(tok, (const float*)dx, dwte, dwpe, mbs, s, h, V, 0));
}

extern "C" int mobius_kt_colsum(int dtype, const void* X, int64_t ld, int rows, int n, float* out) {
  const RedWs ws = red_ws_get(colsum_ws_floats(rows, n, 1));
  if (dtype == MOBIUS_BF16) return sync_rc(colsum_accum<bf16>((const bf16*)X, ld, rows, n, out, ws, 0));
  return sync_rc(colsum_accum<float>((const float*)X, ld, rows, n, out, ws, 0));
}

namespace {
template <typename T>
int kt_block(int hidden, int nh, int s, int mbs, const void* w, const void* x, void* y, const void* dy, void* dx,
             float* grads) {
  Shape sh{hidden, nh, s, mbs, 0};
  const int e = sizeof(T);
  const bool fl = use_flash<T>(sh);
  int64_t ab = block_acts_bytes(sh, e, fl), sb = scratch_bytes(sh, e, false, fl);
  uint8_t* buf = ws_get(ab + sb);
  if (!buf) MOBIUS_FAIL(MOBIUS_ENOMEM, "kt_block alloc");
  BlockActs<T> acts;
  Scratch<T> sc;
  carve_block_acts<T>(sh, buf, acts);
  carve_scratch<T>(sh, buf + ab, false, sc);
  if (int rz = scratch_zero<T>(sc, 0)) return rz;
  acts.x = (const T*)x;
  int rc = block_fwd<T>(sh, (const T*)w, acts, (T*)y, sc, 0);
  if (!rc && dy) rc = block_bwd<T>(sh, (const T*)w, acts, (const T*)dy, (T*)dx, grads, sc, 0);
  return sync_rc(rc);
}
}  // namespace

extern "C" int mobius_kt_block(int dtype, int hidden, int n_heads, int seq_len, int mbs, const void* w, const void* x,
                               void* y, const void* dy, void* dx, float* grads) {
  if (dtype == MOBIUS_BF16) return kt_block<bf16>(hidden, n_heads, seq_len, mbs, w, x, y, dy, dx, grads);
  return kt_block<float>(hidden, n_heads, seq_len, mbs, w, x, y, dy, dx, grads);
}

namespace {
template <typename T>
int kt_attn(int mbs, int s, int nh, int dh, const void* qkv, void* o, const void* dout, void* dqkv) {
  Shape sh{nh * dh, nh, s, mbs, 0};
  const int e = sizeof(T);
  const bool fl = use_flash<T>(sh);
  int64_t ab = block_acts_bytes(sh, e, fl), sb = scratch_bytes(sh, e, false, fl);
  uint8_t* buf = ws_get(ab + sb);
  if (!buf) MOBIUS_FAIL(MOBIUS_ENOMEM, "kt_attn alloc");
  BlockActs<T> acts;
  Scratch<T> sc;
  carve_block_acts<T>(sh, buf, acts);
  carve_scratch<T>(sh, buf + ab, false, sc);
  if (int rz = scratch_zero<T>(sc, 0)) return rz;
  int rc = attention_fwd<T>(sh, (const T*)qkv, (T*)o, acts.P, acts.lse, sc, 0);
  if (!rc && dout) rc = attention_bwd<T>(sh, (const T*)qkv, (const T*)o, acts.P, acts.lse, (const T*)dout, (T*)dqkv, sc, 0);
  return sync_rc(rc);
}
}  // namespace

extern "C" int mobius_kt_attention(int dtype, int mbs, int s, int n_heads, int head_dim, const void* qkv, void* o,
                                   const void* dout, void* dqkv) {
  if (dtype == MOBIUS_BF16) return kt_attn<bf16>(mbs, s, n_heads, head_dim, qkv, o, dout, dqkv);
  return kt_attn<float>(mbs, s, n_heads, head_dim, qkv, o, dout, dqkv);
}
