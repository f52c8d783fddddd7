// Internal GEMM interface used by the block/head ops (K1, K2, K3, K4, K9 of
// SURVEY §2.2).  C[m, n] = epilogue( alpha * sum_k A[m, k] * B[n, k] ).
#pragma once

#include <cstdint>
#include <cuda_runtime.h>

namespace mobius {

// A (possibly batched) strided matrix: element (r, c) of batch (b1, b2) is
// at ptr + b1*bs1 + b2*bs2 + r*ld + c   (units: elements).
struct MatView {
  const void* ptr = nullptr;
  int64_t ld = 0;
  int64_t bs1 = 0, bs2 = 0;
};

enum Epi : int {
  EPI_STORE = 0,       // C = alpha*acc
  EPI_BIAS = 1,        // C = alpha*acc + bias[n]
  EPI_BIAS_GELU = 2,   // u = alpha*acc + bias[n]; AUX = u; C = gelu_tanh(u)
  EPI_BIAS_RESID = 3,  // C = alpha*acc + bias[n] + R[m, n]
  EPI_GELU_BWD = 4,    // C = alpha*acc * gelu_tanh'(R[m, n])
  EPI_ACCUM = 5,       // C(f32) = (accumulate ? C : 0) + alpha*acc
};

enum Causal : int {
  CAUSAL_NONE = 0,
  CAUSAL_SKIP_UPPER = 1,  // skip output tiles entirely above the diagonal (n0 > m0+BM-1)
  CAUSAL_K_LT_MEND = 2,   // k range [0, m0+BM)   (P V, dS K)
  CAUSAL_K_GE_M0 = 3,     // k range [m0, K)      (P^T dO, dS^T Q)
};

struct GemmDesc {
  int M = 0, N = 0, K = 0;
  int nb1 = 1, nb2 = 1;       // batch dims (b1 outer, b2 inner)
  // A logical [M, K]: a_mn=false -> row-major [M][K] (K contiguous);
  //                   a_mn=true  -> stored [K][M] (M contiguous), ld = row stride over k.
  MatView A;
  bool a_mn = false;
  // B logical [N, K] (C = A B^T): b_mn=false -> [N][K]; b_mn=true -> stored [K][N].
  MatView B;
  bool b_mn = false;
  MatView C;
  bool c_f32 = false;         // C element type: fp32 (else the path type)
  int epi = EPI_STORE;
  float alpha = 1.f;
  const void* bias = nullptr; // [N], path type
  MatView R;                  // residual (EPI_BIAS_RESID) or gelu input u (EPI_GELU_BWD)
  MatView AUX;                // EPI_BIAS_GELU: pre-activation output (path type)
  int causal = CAUSAL_NONE;
  bool accumulate = false;    // EPI_ACCUM
  // Bias gradient in the weight-gradient GEMM (a_mn, EPI_ACCUM): logical row
  // M-1 of A is all ones (A holds only rows 0..M-2), so row M-1 of C gets
  // sum_k B[n, k] - the column sums of dY - next to dW (the packed block
  // layout stores each bias right after its weight).  bf16: `ones` is a
  // [>= K][64] buffer whose column 0 is 1 (row M-1 is loaded from it; M-1 a
  // multiple of 64); fp32 debug path: the kernel synthesises the row.
  bool ones_row = false;
  const void* ones = nullptr;
};

// true when gemm_bf16 / gemm_f32 run d with ones_row (else the caller sums
// the bias gradient itself)
bool gemm_ones_row_supported(const GemmDesc& d, bool f32);

// tcgen05/TMEM/TMA kernel (bf16 operands, fp32 accumulate).  Returns a
// mobius_status.
int gemm_bf16(const GemmDesc& d, cudaStream_t s);
// fp32 SIMT debug kernel (no TF32).  Same semantics, fp32 operands.
int gemm_f32(const GemmDesc& d, cudaStream_t s);

int num_sms();

// Stream-K workspaces are kept per (device, stream); the owner of a stream
// frees its entry before destroying the stream.
void gemm_release_stream(cudaStream_t s);
size_t gemm_workspace_entries();

// Kernel selection knobs (tests / perf A-B): -1 = environment default
// (MOBIUS_GEMM_2CTA, MOBIUS_GEMM_SK), 0 = off, 1 = on.
void gemm_set_config(int two_cta, int stream_k);

}  // namespace mobius
