/*
 * mobius_kernels.h - kernel-level test entry points of libmobius (device
 * pointers, launched on the legacy default stream and synchronised before
 * returning).  They exist so the GPU parity tests can check every hot-path
 * kernel against the CPU oracle's op-level functions; the training step
 * itself uses the same kernels internally (mobius.h).
 *
 * dtype: MOBIUS_BF16 (bf16 tensors, tcgen05 GEMM) or MOBIUS_F32 (fp32
 * tensors, SIMT GEMM).  All return a mobius_status (mobius.h); errors set
 * mobius_last_error().
 */
#ifndef MOBIUS_KERNELS_H
#define MOBIUS_KERNELS_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif
#if defined(__GNUC__)
#pragma GCC visibility push(default)
#endif

/* C[m,n] = epi(alpha * sum_k A[m,k] B[n,k]) over batches (b1 < nb1, b2 < nb2).
 * A: a_mn=0 -> element (m,k) at A + b1*abs1 + b2*abs2 + m*lda + k;
 *    a_mn=1 -> at ... + k*lda + m.  B likewise with (n,k).
 * C: (m,n) at C + b1*cbs1 + b2*cbs2 + m*ldc + n; fp32 if c_f32 (bf16 path) .
 * epi: 0 store, 1 +bias[n], 2 u=+bias -> AUX=u, C=gelu(u), 3 +bias+R[m,n],
 *      4 *gelu'(R[m,n]), 5 fp32 accumulate (C += if accumulate).
 * causal: 0 none, 1 skip tiles above the diagonal, 2 k < m-tile end,
 *         3 k >= m-tile start (PAPER's GPT blocks are causal). */
int mobius_kt_gemm(int dtype, int M, int N, int K, int nb1, int nb2, const void* A, int64_t lda, int64_t abs1,
                   int64_t abs2, int a_mn, const void* B, int64_t ldb, int64_t bbs1, int64_t bbs2, int b_mn, void* C,
                   int64_t ldc, int64_t cbs1, int64_t cbs2, int c_f32, int epi, float alpha, const void* bias,
                   const void* R, int64_t ldr, void* AUX, int64_t ldx, int causal, int accumulate);

/* Process-wide bf16 GEMM kernel selection (perf A/B and tests; not part of
 * the step contract): two_cta selects the cta_group::2 256x256 kernel for
 * plain GEMMs, stream_k its Stream-K tail (the last partial wave's tiles are
 * split along K over all SM pairs and reduced deterministically in segment
 * order).  Each is -1 (environment default MOBIUS_GEMM_2CTA /
 * MOBIUS_GEMM_SK, on unless set to 0), 0 or 1; anything else is
 * MOBIUS_EINVAL.  Takes effect for GEMMs launched after the call. */
int mobius_kt_gemm_config(int two_cta, int stream_k);

int mobius_kt_layernorm_fwd(int dtype, const void* x, const void* g, const void* b, void* y, float* mu, float* rstd,
                            int rows, int h);
int mobius_kt_layernorm_bwd(int dtype, const void* dy, const void* x, const void* g, const float* mu,
                            const float* rstd, const void* dres, void* dx, float* dg, float* db, int rows, int h);
int mobius_kt_softmax_fwd(int dtype, const float* S, void* P, int B, int s, float scale);
int mobius_kt_softmax_bwd(int dtype, const void* P, const float* dP, void* dS, int B, int s, float scale);
int mobius_kt_cross_entropy(int dtype, void* logits, const int32_t* tok, float* loss_rows, int rows, int V, int s,
                            float inv_ntok);
int mobius_kt_embed_fwd(int dtype, const int32_t* tok, const void* wte, const void* wpe, void* x, int mbs, int s,
                        int h);
int mobius_kt_embed_bwd(int dtype, const int32_t* tok, const void* dx, float* dwte, float* dwpe, int mbs, int s,
                        int h, int V);
int mobius_kt_colsum(int dtype, const void* X, int64_t ld, int rows, int n, float* out);
/* Causal attention core of a block (the path the block uses: fused tcgen05
 * flash kernels on the bf16 path when head_dim in {64,128} and s % 128 == 0,
 * else GEMM + softmax).  qkv [mbs*s, 3h] -> o [mbs*s, h]; if dout != NULL,
 * dqkv [mbs*s, 3h] = d(sum o*dout)/d qkv. */
int mobius_kt_attention(int dtype, int mbs, int s, int n_heads, int head_dim, const void* qkv, void* o,
                        const void* dout, void* dqkv);
/* One transformer block forward + backward through the runtime's block ops
 * (weights in oracle layout, path dtype, on device).  x [T,h] -> y [T,h];
 * dy [T,h] -> dx [T,h], grads (fp32, oracle layout of one block) +=. */
int mobius_kt_block(int dtype, int hidden, int n_heads, int seq_len, int mbs, const void* w, const void* x, void* y,
                    const void* dy, void* dx, float* grads);

#if defined(__GNUC__)
#pragma GCC visibility pop
#endif
#ifdef __cplusplus
}
#endif
#endif
