// GPT layer forward/backward composed from the tcgen05 GEMM (bf16 path) or
// the SIMT GEMM (fp32 debug path) and the fused HBM-bound kernels.
// Equations: SURVEY §8(c) O-2 (reading #1 of the paper's "GPT-like"
// blocks).
#include <algorithm>
#include <cmath>

#include "common.h"
#include "elem.h"
#include "flash.h"
#include "gemm.h"
#include "ops.h"

namespace mobius {

thread_local int64_t g_kernel_launches = 0;
static KernelTimer* g_timer = nullptr;
void set_kernel_timer(KernelTimer* t) { g_timer = t; }
KernelTimer* kernel_timer() { return g_timer; }

BlockLayout::BlockLayout(int64_t h) {
  int64_t p = 0;
  ln1_g = p; p += h;
  ln1_b = p; p += h;
  w_qkv = p; p += h * 3 * h;
  b_qkv = p; p += 3 * h;
  w_o = p; p += h * h;
  b_o = p; p += h;
  ln2_g = p; p += h;
  ln2_b = p; p += h;
  w_1 = p; p += h * 4 * h;
  b_1 = p; p += 4 * h;
  w_2 = p; p += 4 * h * h;
  b_2 = p; p += h;
  total = p;
}
EmbedLayout::EmbedLayout(int64_t h, int64_t V, int64_t s) {
  wte = 0;
  wpe = V * h;
  total = V * h + s * h;
}
HeadLayout::HeadLayout(int64_t h, int64_t V) {
  lnf_g = 0;
  lnf_b = h;
  w_head = 2 * h;
  total = 2 * h + h * V;
}

template <>
int gemm<__nv_bfloat16>(const GemmDesc& d, cudaStream_t st) {
  return gemm_bf16(d, st);
}
template <>
int gemm<float>(const GemmDesc& d, cudaStream_t st) {
  return gemm_f32(d, st);
}

namespace {

inline int64_t align256(int64_t x) { return (x + 255) & ~int64_t(255); }

struct Carver {
  uint8_t* base;
  int64_t off = 0;
  template <typename P>
  P* take(int64_t bytes) {
    P* p = base ? reinterpret_cast<P*>(base + off) : nullptr;
    off += align256(bytes);
    return p;
  }
};

MatView mv(const void* p, int64_t ld, int64_t bs1 = 0, int64_t bs2 = 0) {
  MatView v;
  v.ptr = p;
  v.ld = ld;
  v.bs1 = bs1;
  v.bs2 = bs2;
  return v;
}

template <typename T>
int run_gemm(GemmDesc& d, cudaStream_t st, int cls) {
  KernelTimer* t = g_timer;
  // algorithmic GEMM work: a ones row (the fused bias gradient) is not counted
  int64_t flops = 2LL * (d.ones_row ? d.M - 1 : d.M) * d.N * d.K * d.nb1 * d.nb2;
  if (d.causal != CAUSAL_NONE) flops /= 2;  // algorithmic work of a causal product
  if (t) t->begin(cls, st);
  int rc = gemm<T>(d, st);
  if (t) t->end(cls, st, flops);
  ++g_kernel_launches;
  return rc;
}

#define RC(x)              \
  do {                     \
    int _rc = (x);         \
    if (_rc) return _rc;   \
  } while (0)

struct ElemScope {
  cudaStream_t st;
  int n;
  bool open = true;
  ElemScope(cudaStream_t s, int n_) : st(s), n(n_) {
    if (g_timer) g_timer->begin(KCLS_ELEM, st);
  }
  void timed_end() {  // close the timing bracket early (work that follows belongs to another class)
    if (!open) return;
    open = false;
    if (g_timer) g_timer->end(KCLS_ELEM, st, 0);
    g_kernel_launches += n;
  }
  ~ElemScope() { timed_end(); }
};

}  // namespace

// The weight-gradient GEMM d (C += A^T B, A = X^T MN-major) also produces
// the bias gradient sum_rows B as the row after the weight's last row (where
// the packed layout keeps the bias) when the GEMM kernel supports a ones row
// there; returns whether it does (else the caller runs a column sum).
template <typename T>
bool with_bias_row(GemmDesc& d, const Scratch<T>& sc) {
  static const bool off = getenv("MOBIUS_NO_BIAS_ROW") != nullptr;  // A/B: separate column sums
  if (off) return false;
  GemmDesc t = d;
  t.M = d.M + 1;
  t.ones_row = true;
  t.ones = sc.ones;
  const bool f32 = sizeof(T) == 4;
  if ((!f32 && !sc.ones) || !gemm_ones_row_supported(t, f32)) return false;
  d = t;
  return true;
}

template <>
bool use_flash<float>(const Shape&) {
  return false;
}
template <>
bool use_flash<__nv_bfloat16>(const Shape& sh) {
  return flash_supported(sh.dh(), sh.s) != 0;
}

int64_t block_acts_bytes(const Shape& sh, int e, bool flash, bool compact) {
  Carver c{nullptr};
  const int64_t T = sh.T(), h = sh.h, B = (int64_t)sh.mbs * sh.nh, s = sh.s;
  const int64_t full = compact ? 0 : 1;
  c.take<char>(full * T * h * e);      // a
  c.take<char>(T * 4);          // mu1
  c.take<char>(T * 4);          // rs1
  c.take<char>(T * 3 * h * e);  // qkv
  c.take<char>(flash ? 0 : B * s * s * e);  // P
  c.take<char>(flash ? B * s * 4 : 0);      // lse
  c.take<char>(T * h * e);      // o
  c.take<char>(T * h * e);      // x1
  c.take<char>(full * T * h * e);      // a2
  c.take<char>(T * 4);
  c.take<char>(T * 4);
  c.take<char>(T * 4 * h * e);  // u
  c.take<char>(full * T * 4 * h * e);  // g
  return c.off;
}

template <typename T>
void carve_block_acts(const Shape& sh, uint8_t* base, BlockActs<T>& a, bool compact) {
  Carver c{base};
  const int64_t Tn = sh.T(), h = sh.h, B = (int64_t)sh.mbs * sh.nh, s = sh.s, e = sizeof(T);
  const int64_t full = compact ? 0 : 1;
  a.a = compact ? nullptr : c.take<T>(Tn * h * e);
  a.mu1 = c.take<float>(Tn * 4);
  a.rs1 = c.take<float>(Tn * 4);
  const bool fl = use_flash<T>(sh);
  a.qkv = c.take<T>(Tn * 3 * h * e);
  a.P = c.take<T>(fl ? 0 : B * s * s * e);
  a.lse = c.take<float>(fl ? B * s * 4 : 0);
  a.o = c.take<T>(Tn * h * e);
  a.x1 = c.take<T>(Tn * h * e);
  a.a2 = compact ? nullptr : c.take<T>(Tn * h * e);
  a.mu2 = c.take<float>(Tn * 4);
  a.rs2 = c.take<float>(Tn * 4);
  a.u = c.take<T>(Tn * 4 * h * e);
  a.g = compact ? nullptr : c.take<T>(Tn * 4 * h * e);
  (void)full;
}

// partial sums of the widest column reduction of a block / head backward
static int64_t red_ws_floats(const Shape& sh) {
  const int T = sh.T(), h = sh.h;
  return std::max({colsum_ws_floats(T, 4 * h, 1), colsum_ws_floats(T, 3 * h, 1), colsum_ws_floats(T, h, 2)});
}

int64_t scratch_bytes(const Shape& sh, int e, bool with_head, bool flash) {
  const int64_t T = sh.T(), h = sh.h, B = (int64_t)sh.mbs * sh.nh, s = sh.s;
  Carver c{nullptr};
  c.take<char>(flash ? 0 : B * s * s * 4);
  c.take<char>(flash ? 0 : B * s * s * e);
  c.take<char>(flash ? T * h * 4 : 0);
  c.take<char>(flash ? B * s * 4 : 0);
  c.take<char>(T * 4 * h * e);
  c.take<char>(T * h * e);
  c.take<char>(T * h * e);
  c.take<char>(T * h * e);
  c.take<char>(T * 3 * h * e);
  c.take<char>(with_head ? (int64_t)sh.head_chunk() * sh.V * e : 0);
  c.take<char>(T * 4);
  c.take<char>(T * 4);
  c.take<char>(T * 4);
  const int64_t kt = sh.no_keep ? 0 : 1;
  c.take<char>(kt * T * h * e);      // ra
  c.take<char>(kt * T * h * e);      // ra2
  c.take<char>(kt * T * 4 * h * e);  // rg
  c.take<char>(red_ws_floats(sh) * 4);
  c.take<char>(RED_WS_COUNTERS * 4);
  c.take<char>(e == 2 ? T * 64 * 2 : 0);  // ones column block of the fused bias gradients
  return c.off;
}

template <typename T>
void carve_scratch(const Shape& sh, uint8_t* base, bool with_head, Scratch<T>& sc) {
  const int64_t Tn = sh.T(), h = sh.h, B = (int64_t)sh.mbs * sh.nh, s = sh.s, e = sizeof(T);
  Carver c{base};
  const bool fl = use_flash<T>(sh);
  sc.S = c.take<float>(fl ? 0 : B * s * s * 4);
  sc.dS = c.take<T>(fl ? 0 : B * s * s * e);
  sc.dq = c.take<float>(fl ? Tn * h * 4 : 0);
  sc.dsum = c.take<float>(fl ? B * s * 4 : 0);
  sc.big1 = c.take<T>(Tn * 4 * h * e);
  sc.t1 = c.take<T>(Tn * h * e);
  sc.t2 = c.take<T>(Tn * h * e);
  sc.t3 = c.take<T>(Tn * h * e);
  sc.qkv_g = c.take<T>(Tn * 3 * h * e);
  sc.logits = c.take<T>(with_head ? (int64_t)sh.head_chunk() * sh.V * e : 0);
  sc.loss_rows = c.take<float>(Tn * 4);
  sc.mu = c.take<float>(Tn * 4);
  sc.rs = c.take<float>(Tn * 4);
  const int64_t kt = sh.no_keep ? 0 : 1;
  sc.ra = kt ? c.take<T>(Tn * h * e) : nullptr;
  sc.ra2 = kt ? c.take<T>(Tn * h * e) : nullptr;
  sc.rg = kt ? c.take<T>(Tn * 4 * h * e) : nullptr;
  sc.red.part = c.take<float>(red_ws_floats(sh) * 4);
  sc.red.cnt = c.take<unsigned>(RED_WS_COUNTERS * 4);
  sc.ones = sizeof(T) == 2 ? c.take<T>(Tn * 64 * 2) : nullptr;
  sc.ones_rows = Tn;
}

template <typename T>
int scratch_zero(const Scratch<T>& sc, cudaStream_t st) {
  if (cudaMemsetAsync(sc.red.cnt, 0, RED_WS_COUNTERS * 4, st) != cudaSuccess)
    MOBIUS_FAIL(MOBIUS_ECUDA, "scratch_zero");
  if (sc.ones) return fill_ones_col(sc.ones, sc.ones_rows, st);
  return MOBIUS_OK;
}

// ------------------------------------------------------------ attention
template <typename T>
int attention_fwd(const Shape& sh, const T* qkv, T* o, T* P, float* lse, Scratch<T>& sc, cudaStream_t st) {
  const int h = sh.h, nh = sh.nh, s = sh.s, dh = sh.dh(), mbs = sh.mbs;
  const int64_t Sbs2 = (int64_t)s * s, Sbs1 = nh * Sbs2;
  if (use_flash<T>(sh)) {
    KernelTimer* t = g_timer;
    if (t) t->begin(KCLS_ATTN, st);
    int rc = flash_attn_fwd(reinterpret_cast<const __nv_bfloat16*>(qkv), reinterpret_cast<__nv_bfloat16*>(o), lse,
                            mbs, s, nh, dh, st);
    if (t) t->end(KCLS_ATTN, st, 2LL * mbs * nh * s * s * dh);
    ++g_kernel_launches;
    return rc;
  }
  {  // S = q k^T (fp32), causal tiles only
    GemmDesc d;
    d.M = s; d.N = s; d.K = dh; d.nb1 = mbs; d.nb2 = nh;
    d.A = mv(qkv, 3 * h, (int64_t)s * 3 * h, dh);
    d.B = mv(qkv + h, 3 * h, (int64_t)s * 3 * h, dh);
    d.C = mv(sc.S, s, Sbs1, Sbs2); d.c_f32 = true;
    d.causal = CAUSAL_SKIP_UPPER;
    RC(run_gemm<T>(d, st, KCLS_ATTN));
  }
  {
    ElemScope es(st, 1);
    RC(softmax_causal_fwd<T>(sc.S, P, mbs * nh, s, 1.0f / sqrtf((float)dh), st));
  }
  {  // o = P v
    GemmDesc d;
    d.M = s; d.N = dh; d.K = s; d.nb1 = mbs; d.nb2 = nh;
    d.A = mv(P, s, Sbs1, Sbs2);
    d.B = mv(qkv + 2 * h, 3 * h, (int64_t)s * 3 * h, dh); d.b_mn = true;
    d.C = mv(o, h, (int64_t)s * h, dh);
    d.causal = CAUSAL_K_LT_MEND;
    RC(run_gemm<T>(d, st, KCLS_ATTN));
  }
  return MOBIUS_OK;
}

template <typename T>
int attention_bwd(const Shape& sh, const T* qkv, const T* o, const T* P, const float* lse, const T* dO, T* dqkv,
                  Scratch<T>& sc, cudaStream_t st) {
  const int h = sh.h, nh = sh.nh, s = sh.s, dh = sh.dh(), mbs = sh.mbs;
  const int64_t Sbs2 = (int64_t)s * s, Sbs1 = nh * Sbs2;
  const float scale = 1.0f / sqrtf((float)dh);
  if (use_flash<T>(sh)) {
    KernelTimer* t = g_timer;
    if (t) t->begin(KCLS_ATTN, st);
    int rc = flash_attn_bwd(reinterpret_cast<const __nv_bfloat16*>(qkv), reinterpret_cast<const __nv_bfloat16*>(o),
                            reinterpret_cast<const __nv_bfloat16*>(dO), lse, sc.dsum, sc.dq,
                            reinterpret_cast<__nv_bfloat16*>(dqkv), mbs, s, nh, dh, st);
    if (t) t->end(KCLS_ATTN, st, 4LL * mbs * nh * s * s * dh);
    g_kernel_launches += 3;
    return rc;
  }
  {  // dP = do v^T (fp32)
    GemmDesc d;
    d.M = s; d.N = s; d.K = dh; d.nb1 = mbs; d.nb2 = nh;
    d.A = mv(dO, h, (int64_t)s * h, dh);
    d.B = mv(qkv + 2 * h, 3 * h, (int64_t)s * 3 * h, dh);
    d.C = mv(sc.S, s, Sbs1, Sbs2); d.c_f32 = true;
    d.causal = CAUSAL_SKIP_UPPER;
    RC(run_gemm<T>(d, st, KCLS_ATTN));
  }
  {
    ElemScope es(st, 1);
    RC(softmax_causal_bwd<T>(P, sc.S, sc.dS, mbs * nh, s, scale, st));
  }
  {  // dV = P^T do
    GemmDesc d;
    d.M = s; d.N = dh; d.K = s; d.nb1 = mbs; d.nb2 = nh;
    d.A = mv(P, s, Sbs1, Sbs2); d.a_mn = true;
    d.B = mv(dO, h, (int64_t)s * h, dh); d.b_mn = true;
    d.C = mv(dqkv + 2 * h, 3 * h, (int64_t)s * 3 * h, dh);
    d.causal = CAUSAL_K_GE_M0;
    RC(run_gemm<T>(d, st, KCLS_ATTN));
  }
  {  // dQ = dS K
    GemmDesc d;
    d.M = s; d.N = dh; d.K = s; d.nb1 = mbs; d.nb2 = nh;
    d.A = mv(sc.dS, s, Sbs1, Sbs2);
    d.B = mv(qkv + h, 3 * h, (int64_t)s * 3 * h, dh); d.b_mn = true;
    d.C = mv(dqkv, 3 * h, (int64_t)s * 3 * h, dh);
    d.causal = CAUSAL_K_LT_MEND;
    RC(run_gemm<T>(d, st, KCLS_ATTN));
  }
  {  // dK = dS^T Q
    GemmDesc d;
    d.M = s; d.N = dh; d.K = s; d.nb1 = mbs; d.nb2 = nh;
    d.A = mv(sc.dS, s, Sbs1, Sbs2); d.a_mn = true;
    d.B = mv(qkv, 3 * h, (int64_t)s * 3 * h, dh); d.b_mn = true;
    d.C = mv(dqkv + h, 3 * h, (int64_t)s * 3 * h, dh);
    d.causal = CAUSAL_K_GE_M0;
    RC(run_gemm<T>(d, st, KCLS_ATTN));
  }
  return MOBIUS_OK;
}

// ------------------------------------------------------------------ block
template <typename T>
int block_fwd(const Shape& sh, const T* w, BlockActs<T>& A_in, T* y, Scratch<T>& sc, cudaStream_t st) {
  const BlockLayout L(sh.h);
  BlockActs<T> A = A_in;
  if (!A.a) {  // compact kept activations: a, a2, g go to scratch (recomputed in backward)
    A.a = sc.ra;
    A.a2 = sc.ra2;
    A.g = sc.rg;
  }
  const int Tn = sh.T(), h = sh.h, nh = sh.nh, s = sh.s, dh = sh.dh(), mbs = sh.mbs;
  const int64_t Sbs2 = (int64_t)s * s, Sbs1 = nh * Sbs2;
  {
    ElemScope es(st, 1);
    RC(layernorm_fwd<T>(A.x, w + L.ln1_g, w + L.ln1_b, A.a, A.mu1, A.rs1, Tn, h, st));
  }
  {  // qkv = a Wqkv + bqkv
    GemmDesc d;
    d.M = Tn; d.N = 3 * h; d.K = h;
    d.A = mv(A.a, h);
    d.B = mv(w + L.w_qkv, 3 * h); d.b_mn = true;
    d.C = mv(A.qkv, 3 * h);
    d.epi = EPI_BIAS; d.bias = w + L.b_qkv;
    RC(run_gemm<T>(d, st, KCLS_GEMM));
  }
  RC(attention_fwd<T>(sh, A.qkv, A.o, A.P, A.lse, sc, st));
  {  // x1 = x + o Wo + bo
    GemmDesc d;
    d.M = Tn; d.N = h; d.K = h;
    d.A = mv(A.o, h);
    d.B = mv(w + L.w_o, h); d.b_mn = true;
    d.C = mv(A.x1, h);
    d.epi = EPI_BIAS_RESID; d.bias = w + L.b_o; d.R = mv(A.x, h);
    RC(run_gemm<T>(d, st, KCLS_GEMM));
  }
  {
    ElemScope es(st, 1);
    RC(layernorm_fwd<T>(A.x1, w + L.ln2_g, w + L.ln2_b, A.a2, A.mu2, A.rs2, Tn, h, st));
  }
  {  // u = a2 W1 + b1 ; g = gelu(u)
    GemmDesc d;
    d.M = Tn; d.N = 4 * h; d.K = h;
    d.A = mv(A.a2, h);
    d.B = mv(w + L.w_1, 4 * h); d.b_mn = true;
    d.C = mv(A.g, 4 * h);
    d.epi = EPI_BIAS_GELU; d.bias = w + L.b_1; d.AUX = mv(A.u, 4 * h);
    RC(run_gemm<T>(d, st, KCLS_GEMM));
  }
  {  // y = x1 + g W2 + b2
    GemmDesc d;
    d.M = Tn; d.N = h; d.K = 4 * h;
    d.A = mv(A.g, 4 * h);
    d.B = mv(w + L.w_2, h); d.b_mn = true;
    d.C = mv(y, h);
    d.epi = EPI_BIAS_RESID; d.bias = w + L.b_2; d.R = mv(A.x1, h);
    RC(run_gemm<T>(d, st, KCLS_GEMM));
  }
  return MOBIUS_OK;
}

template <typename T>
int block_bwd(const Shape& sh, const T* w, const BlockActs<T>& A_in, const T* dy, T* dx, float* G, Scratch<T>& sc,
              cudaStream_t st) {
  const BlockLayout L(sh.h);
  const int Tn = sh.T(), h = sh.h, nh = sh.nh, s = sh.s, dh = sh.dh(), mbs = sh.mbs;
  const int64_t Sbs2 = (int64_t)s * s, Sbs1 = nh * Sbs2;
  const float scale = 1.0f / sqrtf((float)dh);
  BlockActs<T> A = A_in;
  const bool compact = !A.a;
  if (compact) {  // compact kept activations: recompute a, a2 (LN forwards); g = gelu(u) comes from the du GEMM
    if constexpr (sizeof(T) != 2) {
      MOBIUS_FAIL(MOBIUS_EINVAL, "block_bwd: compact activations are bf16-only");
    } else {
      ElemScope es(st, 2);
      A.a = sc.ra;
      A.a2 = sc.ra2;
      A.g = sc.rg;
      RC(layernorm_fwd<T>(A.x, w + L.ln1_g, w + L.ln1_b, A.a, A.mu1, A.rs1, Tn, h, st));
      RC(layernorm_fwd<T>(A.x1, w + L.ln2_g, w + L.ln2_b, A.a2, A.mu2, A.rs2, Tn, h, st));
    }
  }
  T* du = sc.big1;
  {  // du = (dy W2^T) * gelu'(u); compact: also g = gelu(u) (AUX), bit-identical to the forward's
    GemmDesc d;
    d.M = Tn; d.N = 4 * h; d.K = h;
    d.A = mv(dy, h);
    d.B = mv(w + L.w_2, h);
    d.C = mv(du, 4 * h);
    d.epi = EPI_GELU_BWD; d.R = mv(A.u, 4 * h);
    if (compact) d.AUX = mv(A.g, 4 * h);
    RC(run_gemm<T>(d, st, KCLS_GEMM));
  }
  {  // dW2 += g^T dy
    GemmDesc d;
    d.M = 4 * h; d.N = h; d.K = Tn;
    d.A = mv(A.g, 4 * h); d.a_mn = true;
    d.B = mv(dy, h); d.b_mn = true;
    d.C = mv(G + L.w_2, h); d.c_f32 = true;
    d.epi = EPI_ACCUM; d.accumulate = true;
    RC(run_gemm<T>(d, st, KCLS_GEMM));
  }
  {  // dW1 += a2^T du, and db1 += sum du as its ones row (b_1 follows w_1 in the layout)
    GemmDesc d;
    d.M = h; d.N = 4 * h; d.K = Tn;
    d.A = mv(A.a2, h); d.a_mn = true;
    d.B = mv(du, 4 * h); d.b_mn = true;
    d.C = mv(G + L.w_1, 4 * h); d.c_f32 = true;
    d.epi = EPI_ACCUM; d.accumulate = true;
    const bool fused = with_bias_row<T>(d, sc);
    if (!fused) {
      ElemScope es(st, 1);
      RC(colsum_accum<T>(du, 4 * h, Tn, 4 * h, G + L.b_1, sc.red, st));
      es.timed_end();
    }
    RC(run_gemm<T>(d, st, KCLS_GEMM));
  }
  {  // da2 = du W1^T
    GemmDesc d;
    d.M = Tn; d.N = h; d.K = 4 * h;
    d.A = mv(du, 4 * h);
    d.B = mv(w + L.w_1, 4 * h);
    d.C = mv(sc.t1, h);
    RC(run_gemm<T>(d, st, KCLS_GEMM));
  }
  T* dx1 = sc.t2;
  {
    ElemScope es(st, layernorm_bwd_launches<T>(h, true, true));
    // db2 += sum dy rides along: dy is this LN's residual gradient
    RC(layernorm_bwd<T>(sc.t1, A.x1, w + L.ln2_g, A.mu2, A.rs2, dy, dx1, G + L.ln2_g, G + L.ln2_b, Tn, h, sc.red, st,
                        G + L.b_2));
  }
  {  // dWo += o^T dx1, db_o += sum dx1 as its ones row
    GemmDesc d;
    d.M = h; d.N = h; d.K = Tn;
    d.A = mv(A.o, h); d.a_mn = true;
    d.B = mv(dx1, h); d.b_mn = true;
    d.C = mv(G + L.w_o, h); d.c_f32 = true;
    d.epi = EPI_ACCUM; d.accumulate = true;
    const bool fused = with_bias_row<T>(d, sc);
    RC(run_gemm<T>(d, st, KCLS_GEMM));
    if (!fused) {
      ElemScope es(st, 1);
      RC(colsum_accum<T>(dx1, h, Tn, h, G + L.b_o, sc.red, st));
    }
  }
  T* dO = sc.t3;
  {  // do = dx1 Wo^T
    GemmDesc d;
    d.M = Tn; d.N = h; d.K = h;
    d.A = mv(dx1, h);
    d.B = mv(w + L.w_o, h);
    d.C = mv(dO, h);
    RC(run_gemm<T>(d, st, KCLS_GEMM));
  }
  T* dqkv = sc.qkv_g;
  RC(attention_bwd<T>(sh, A.qkv, A.o, A.P, A.lse, dO, dqkv, sc, st));
  {  // dWqkv += a^T dqkv, db_qkv += sum dqkv as its ones row
    GemmDesc d;
    d.M = h; d.N = 3 * h; d.K = Tn;
    d.A = mv(A.a, h); d.a_mn = true;
    d.B = mv(dqkv, 3 * h); d.b_mn = true;
    d.C = mv(G + L.w_qkv, 3 * h); d.c_f32 = true;
    d.epi = EPI_ACCUM; d.accumulate = true;
    const bool fused = with_bias_row<T>(d, sc);
    RC(run_gemm<T>(d, st, KCLS_GEMM));
    if (!fused) {
      ElemScope es(st, 1);
      RC(colsum_accum<T>(dqkv, 3 * h, Tn, 3 * h, G + L.b_qkv, sc.red, st));
    }
  }
  {  // da = dqkv Wqkv^T
    GemmDesc d;
    d.M = Tn; d.N = h; d.K = 3 * h;
    d.A = mv(dqkv, 3 * h);
    d.B = mv(w + L.w_qkv, 3 * h);
    d.C = mv(sc.t1, h);
    RC(run_gemm<T>(d, st, KCLS_GEMM));
  }
  {
    ElemScope es(st, 2);
    RC(layernorm_bwd<T>(sc.t1, A.x, w + L.ln1_g, A.mu1, A.rs1, dx1, dx, G + L.ln1_g, G + L.ln1_b, Tn, h, sc.red, st));
  }
  return MOBIUS_OK;
}

template <typename T>
int embed_layer_fwd(const Shape& sh, const T* w, const int32_t* tok, T* x, cudaStream_t st) {
  const EmbedLayout L(sh.h, sh.V, sh.s);
  ElemScope es(st, 1);
  return embed_fwd<T>(tok, w + L.wte, w + L.wpe, x, sh.mbs, sh.s, sh.h, st);
}

template <typename T>
int embed_layer_bwd(const Shape& sh, const T* w, const int32_t* tok, const T* dx, float* G, cudaStream_t st) {
  const EmbedLayout L(sh.h, sh.V, sh.s);
  ElemScope es(st, 2);
  return embed_bwd<T>(tok, dx, G + L.wte, G + L.wpe, sh.mbs, sh.s, sh.h, sh.V, st);
}

template <typename T>
int head_layer_fwd_bwd(const Shape& sh, const T* w, const T* x, const int32_t* tok, float inv_ntok, T* dx, float* G,
                       double* loss_acc, Scratch<T>& sc, cudaStream_t st) {
  const HeadLayout L(sh.h, sh.V);
  const int Tn = sh.T(), h = sh.h, V = sh.V;
  {
    ElemScope es(st, 1);
    RC(layernorm_fwd<T>(x, w + L.lnf_g, w + L.lnf_b, sc.t1, sc.mu, sc.rs, Tn, h, st));
  }
  // row chunks of hc rows (whole sequences): logits [hc, V] live in scratch,
  // CE in place, dW accumulated chunk by chunk (fp32), da chunk into t2
  const int hc = sh.head_chunk();
  for (int r0 = 0; r0 < Tn; r0 += hc) {
    const int rows = std::min(hc, Tn - r0);
    const T* a = sc.t1 + (int64_t)r0 * h;
    const int32_t* tk = tok + (int64_t)(r0 / sh.s) * (sh.s + 1);
    {  // logits = a Whead
      GemmDesc d;
      d.M = rows; d.N = V; d.K = h;
      d.A = mv(a, h);
      d.B = mv(w + L.w_head, V); d.b_mn = true;
      d.C = mv(sc.logits, V);
      RC(run_gemm<T>(d, st, KCLS_GEMM));
    }
    {
      ElemScope es(st, 2);
      RC(cross_entropy_fwd_bwd<T>(sc.logits, tk, sc.loss_rows, rows, V, sh.s, inv_ntok, st));
      RC(loss_accumulate(sc.loss_rows, rows, loss_acc, st));
    }
    {  // dWhead += a^T dlogits
      GemmDesc d;
      d.M = h; d.N = V; d.K = rows;
      d.A = mv(a, h); d.a_mn = true;
      d.B = mv(sc.logits, V); d.b_mn = true;
      d.C = mv(G + L.w_head, V); d.c_f32 = true;
      d.epi = EPI_ACCUM; d.accumulate = true;
      RC(run_gemm<T>(d, st, KCLS_GEMM));
    }
    {  // da = dlogits Whead^T
      GemmDesc d;
      d.M = rows; d.N = h; d.K = V;
      d.A = mv(sc.logits, V);
      d.B = mv(w + L.w_head, V);
      d.C = mv(sc.t2 + (int64_t)r0 * h, h);
      RC(run_gemm<T>(d, st, KCLS_GEMM));
    }
  }
  {
    ElemScope es(st, 2);
    RC(layernorm_bwd<T>(sc.t2, x, w + L.lnf_g, sc.mu, sc.rs, (const T*)nullptr, dx, G + L.lnf_g, G + L.lnf_b, Tn,
                        h, sc.red, st));
  }
  return MOBIUS_OK;
}

#define INST(T)                                                                                                   \
  template void carve_block_acts<T>(const Shape&, uint8_t*, BlockActs<T>&, bool);                                      \
  template void carve_scratch<T>(const Shape&, uint8_t*, bool, Scratch<T>&);                                     \
  template int scratch_zero<T>(const Scratch<T>&, cudaStream_t);                                                  \
  template int block_fwd<T>(const Shape&, const T*, BlockActs<T>&, T*, Scratch<T>&, cudaStream_t);               \
  template int block_bwd<T>(const Shape&, const T*, const BlockActs<T>&, const T*, T*, float*, Scratch<T>&,      \
                            cudaStream_t);                                                                       \
  template int embed_layer_fwd<T>(const Shape&, const T*, const int32_t*, T*, cudaStream_t);                      \
  template int embed_layer_bwd<T>(const Shape&, const T*, const int32_t*, const T*, float*, cudaStream_t);        \
  template int head_layer_fwd_bwd<T>(const Shape&, const T*, const T*, const int32_t*, float, T*, float*, double*, \
                                     Scratch<T>&, cudaStream_t);                                                  \
  template int attention_fwd<T>(const Shape&, const T*, T*, T*, float*, Scratch<T>&, cudaStream_t);                \
  template int attention_bwd<T>(const Shape&, const T*, const T*, const T*, const float*, const T*, T*, Scratch<T>&, \
                                cudaStream_t);
INST(float)
INST(__nv_bfloat16)

}  // namespace mobius
