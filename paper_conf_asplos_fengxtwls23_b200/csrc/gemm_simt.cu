// fp32 SIMT GEMM for the debug path (K11 of SURVEY §2.2): same GemmDesc
// semantics and fused epilogues as the tcgen05 kernel, plain fp32 FMA (no
// TF32), 64x64 tiles, 4x4 outputs per thread, batched over blockIdx.z.
#include <cuda_runtime.h>

#include "common.h"
#include "gemm.h"

namespace mobius {
namespace {

constexpr int TM = 64, TN = 64, TK = 16;

struct SParams {
  int M, N, K, nb2;
  const float *A, *B;
  int64_t lda, abs1, abs2, ldb, bbs1, bbs2;
  int a_mn, b_mn;
  int ones_row;  // A row M-1 is all ones (bias gradient next to dW)
  float* C;
  int64_t ldc, cbs1, cbs2;
  int epi, causal, accumulate;
  float alpha;
  const float* bias;
  const float* R;
  int64_t ldr, rbs1, rbs2;
  float* AUX;
  int64_t ldx, xbs1, xbs2;
};

__device__ __forceinline__ float gelu_f(float u) {
  const float c = 0.7978845608028654f, a = 0.044715f;
  return 0.5f * u * (1.f + tanhf(c * (u + a * u * u * u)));
}
__device__ __forceinline__ float gelu_grad_f(float u) {
  const float c = 0.7978845608028654f, a = 0.044715f;
  float t = tanhf(c * (u + a * u * u * u));
  return 0.5f * (1.f + t) + 0.5f * u * (1.f - t * t) * c * (1.f + 3.f * a * u * u);
}

__global__ void __launch_bounds__(256) gemm_simt_kernel(const SParams p) {
  __shared__ float As[TK][TM + 4];
  __shared__ float Bs[TK][TN + 4];
  const int bz = blockIdx.z;
  const int b1 = bz / p.nb2, b2 = bz % p.nb2;
  const int m0 = blockIdx.y * TM, n0 = blockIdx.x * TN;
  if (p.causal == CAUSAL_SKIP_UPPER && n0 > m0 + TM - 1) return;
  int k_begin = 0, k_end = p.K;
  if (p.causal == CAUSAL_K_LT_MEND) k_end = min(p.K, m0 + TM);
  if (p.causal == CAUSAL_K_GE_M0) k_begin = m0;
  const float* A = p.A + b1 * p.abs1 + b2 * p.abs2;
  const float* B = p.B + b1 * p.bbs1 + b2 * p.bbs2;
  const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;
  float acc[4][4] = {};
  for (int k0 = k_begin; k0 < k_end; k0 += TK) {
    for (int i = threadIdx.x; i < TK * TM; i += 256) {
      int kk, mm;
      if (p.a_mn) { kk = i / TM; mm = i % TM; } else { mm = i / TK; kk = i % TK; }
      int gm = m0 + mm, gk = k0 + kk;
      float v = 0.f;
      if (gm < p.M && gk < k_end)
        v = (p.ones_row && gm == p.M - 1) ? 1.f : p.a_mn ? A[(int64_t)gk * p.lda + gm] : A[(int64_t)gm * p.lda + gk];
      As[kk][mm] = v;
    }
    for (int i = threadIdx.x; i < TK * TN; i += 256) {
      int kk, nn;
      if (p.b_mn) { kk = i / TN; nn = i % TN; } else { nn = i / TK; kk = i % TK; }
      int gn = n0 + nn, gk = k0 + kk;
      float v = 0.f;
      if (gn < p.N && gk < k_end) v = p.b_mn ? B[(int64_t)gk * p.ldb + gn] : B[(int64_t)gn * p.ldb + gk];
      Bs[kk][nn] = v;
    }
    __syncthreads();
#pragma unroll
    for (int kk = 0; kk < TK; ++kk) {
      float a[4], b[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) a[i] = As[kk][ty * 4 + i];
#pragma unroll
      for (int j = 0; j < 4; ++j) b[j] = Bs[kk][tx * 4 + j];
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
    }
    __syncthreads();
  }
  for (int i = 0; i < 4; ++i) {
    int m = m0 + ty * 4 + i;
    if (m >= p.M) continue;
    for (int j = 0; j < 4; ++j) {
      int n = n0 + tx * 4 + j;
      if (n >= p.N) continue;
      float v = acc[i][j] * p.alpha;
      if (p.epi == EPI_BIAS || p.epi == EPI_BIAS_GELU || p.epi == EPI_BIAS_RESID) v += p.bias[n];
      if (p.epi == EPI_BIAS_GELU) {
        p.AUX[b1 * p.xbs1 + b2 * p.xbs2 + (int64_t)m * p.ldx + n] = v;
        v = gelu_f(v);
      }
      if (p.epi == EPI_BIAS_RESID) v += p.R[b1 * p.rbs1 + b2 * p.rbs2 + (int64_t)m * p.ldr + n];
      if (p.epi == EPI_GELU_BWD) v *= gelu_grad_f(p.R[b1 * p.rbs1 + b2 * p.rbs2 + (int64_t)m * p.ldr + n]);
      float* c = p.C + b1 * p.cbs1 + b2 * p.cbs2 + (int64_t)m * p.ldc + n;
      if (p.epi == EPI_ACCUM && p.accumulate) v += *c;
      *c = v;
    }
  }
}

}  // namespace

int gemm_f32(const GemmDesc& d, cudaStream_t s) {
  MOBIUS_CHECK_ARG(d.M > 0 && d.N > 0 && d.K > 0, "gemm_f32: empty shape");
  SParams p;
  p.M = d.M; p.N = d.N; p.K = d.K; p.nb2 = d.nb2;
  p.A = (const float*)d.A.ptr; p.lda = d.A.ld; p.abs1 = d.A.bs1; p.abs2 = d.A.bs2; p.a_mn = d.a_mn;
  p.B = (const float*)d.B.ptr; p.ldb = d.B.ld; p.bbs1 = d.B.bs1; p.bbs2 = d.B.bs2; p.b_mn = d.b_mn;
  p.ones_row = d.ones_row ? 1 : 0;
  p.C = (float*)d.C.ptr; p.ldc = d.C.ld; p.cbs1 = d.C.bs1; p.cbs2 = d.C.bs2;
  p.epi = d.epi; p.causal = d.causal; p.accumulate = d.accumulate; p.alpha = d.alpha;
  p.bias = (const float*)d.bias;
  p.R = (const float*)d.R.ptr; p.ldr = d.R.ld; p.rbs1 = d.R.bs1; p.rbs2 = d.R.bs2;
  p.AUX = (float*)d.AUX.ptr; p.ldx = d.AUX.ld; p.xbs1 = d.AUX.bs1; p.xbs2 = d.AUX.bs2;
  dim3 grid((d.N + TN - 1) / TN, (d.M + TM - 1) / TM, d.nb1 * d.nb2);
  gemm_simt_kernel<<<grid, 256, 0, s>>>(p);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) MOBIUS_FAIL(MOBIUS_ECUDA, "gemm_f32 launch: %s", cudaGetErrorString(e));
  return MOBIUS_OK;
}

}  // namespace mobius
