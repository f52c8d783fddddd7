// Layer-level operations of the GPT stage compute (rows a4, a6, a7 of
// SURVEY §8(a)).  Weights are the packed oracle-layout tensors of one
// profile layer in the path type T; gradients are fp32 accumulators of the
// same layout.  Everything is launched on one stream.
#pragma once

#include <cstdint>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include "../../include/mobius.h"
#include "elem.h"

namespace mobius {

struct Shape {
  int h, nh, s, mbs, V;
  int head_rows = 0;  // LM head row chunk (multiple of s; 0 = all T rows at once)
  bool no_keep = false;  // no kept activations: the scratch has no compact-keep recompute targets
  int T() const { return mbs * s; }
  int dh() const { return h / nh; }
  int head_chunk() const { return head_rows > 0 && head_rows < T() ? head_rows : T(); }
};

// element offsets of the block tensors inside one packed block (oracle order)
struct BlockLayout {
  int64_t ln1_g, ln1_b, w_qkv, b_qkv, w_o, b_o, ln2_g, ln2_b, w_1, b_1, w_2, b_2, total;
  explicit BlockLayout(int64_t h);
};
struct EmbedLayout {
  int64_t wte, wpe, total;
  EmbedLayout(int64_t h, int64_t V, int64_t s);
};
struct HeadLayout {
  int64_t lnf_g, lnf_b, w_head, total;
  HeadLayout(int64_t h, int64_t V);
};

// Saved activations of one block for one microbatch (all device pointers).
template <typename T>
struct BlockActs {
  const T* x;      // input [T, h]
  T* a;            // LN1(x)
  float *mu1, *rs1;
  T* qkv;          // [T, 3h]
  T* P;            // [mbs*nh, s, s] causal softmax probabilities (materialised path only)
  float* lse;      // [mbs*nh*s] log2-domain row logsumexp (flash path only)
  T* o;            // attention output [T, h]
  T* x1;           // x + o Wo + bo
  T* a2;           // LN2(x1)
  float *mu2, *rs2;
  T* u;            // a2 W1 + b1  [T, 4h]
  T* g;            // gelu(u)     [T, 4h]
};

template <typename T>
struct Scratch {
  float* S;        // [mbs*nh, s, s] fp32 scores / dP (materialised path only)
  T* dS;           // [mbs*nh, s, s] (materialised path only)
  float* dq;       // [T, h] fp32 dQ accumulator (flash path only)
  float* dsum;     // [mbs*nh*s] rowsum(dO*O) (flash path only)
  T* big1;         // [T, 4h]
  T* t1;           // [T, h]
  T* t2;           // [T, h]
  T* t3;           // [T, h]
  T* qkv_g;        // [T, 3h]
  T* logits;       // [T, V]
  float* loss_rows;  // [T]
  float *mu, *rs;  // [T] (head LN)
  T *ra, *ra2, *rg;  // recompute targets of a compact BlockActs: [T, h], [T, h], [T, 4h]
  RedWs red;       // deterministic column-reduction workspace (counters zeroed by scratch_zero)
  T* ones = nullptr;   // bf16 path: [T][64], column 0 = 1 (ones row of the fused bias gradients; scratch_zero fills it)
  int ones_rows = 0;
};
// zero the reduction counters of a freshly carved Scratch (once per arena)
template <typename T>
int scratch_zero(const Scratch<T>& sc, cudaStream_t st);

// true when the fused tcgen05 attention is used (bf16, dh in {64,128}, s % 128 == 0)
template <typename T>
bool use_flash(const Shape& sh);
// attention core: qkv -> o (fwd) and dO -> dqkv (bwd)
template <typename T>
int attention_fwd(const Shape& sh, const T* qkv, T* o, T* P, float* lse, Scratch<T>& sc, cudaStream_t st);
template <typename T>
int attention_bwd(const Shape& sh, const T* qkv, const T* o, const T* P, const float* lse, const T* dO, T* dqkv,
                  Scratch<T>& sc, cudaStream_t st);

// bytes of one BlockActs set / of the Scratch (for arena planning)
// compact: the kept-activation layout (bf16 flash path) without the LN
// outputs a, a2 and g = gelu(u); block_bwd recomputes those three (two LN
// forwards and an elementwise GeLU, bit-identical to the forward's values)
// into scratch.  The stored set is x, qkv, o, x1, u, lse and the LN stats.
int64_t block_acts_bytes(const Shape& sh, int elem, bool flash, bool compact = false);
int64_t scratch_bytes(const Shape& sh, int elem, bool with_head, bool flash);
template <typename T>
void carve_block_acts(const Shape& sh, uint8_t* base, BlockActs<T>& a, bool compact = false);
template <typename T>
void carve_scratch(const Shape& sh, uint8_t* base, bool with_head, Scratch<T>& s);

// y = block(x); fills acts (acts.x must be set)
template <typename T>
int block_fwd(const Shape& sh, const T* w, BlockActs<T>& acts, T* y, Scratch<T>& sc, cudaStream_t st);
// dx = d block / dx (dy); grads (fp32, block layout) +=
template <typename T>
int block_bwd(const Shape& sh, const T* w, const BlockActs<T>& acts, const T* dy, T* dx, float* grads,
              Scratch<T>& sc, cudaStream_t st);
// x0 = wte[tok] + wpe; tok = microbatch tokens [mbs][s+1]
template <typename T>
int embed_layer_fwd(const Shape& sh, const T* w, const int32_t* tok, T* x, cudaStream_t st);
template <typename T>
int embed_layer_bwd(const Shape& sh, const T* w, const int32_t* tok, const T* dx, float* grads, cudaStream_t st);
// LN_f + LM head + CE fwd+bwd: loss accumulated into loss_acc (sum of token
// losses, double); dx = d/dx of (sum loss) * inv_ntok; grads +=
template <typename T>
int head_layer_fwd_bwd(const Shape& sh, const T* w, const T* x, const int32_t* tok, float inv_ntok, T* dx,
                       float* grads, double* loss_acc, Scratch<T>& sc, cudaStream_t st);

// GEMM dispatch on the path type
template <typename T>
int gemm(const struct GemmDesc& d, cudaStream_t st);

// per-kernel-class timing hooks (set by the runtime when MOBIUS_FLAG_TIMING)
struct KernelTimer {
  virtual ~KernelTimer() {}
  virtual void begin(int cls, cudaStream_t st) = 0;
  virtual void end(int cls, cudaStream_t st, int64_t flops) = 0;
};
enum { KCLS_GEMM = 0, KCLS_ATTN = 1, KCLS_ELEM = 2 };
void set_kernel_timer(KernelTimer* t);
KernelTimer* kernel_timer();
extern thread_local int64_t g_kernel_launches;

}  // namespace mobius
