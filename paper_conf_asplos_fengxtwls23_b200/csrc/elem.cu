// HBM-bound fused kernels (LayerNorm, causal softmax, cross-entropy,
// embedding, column sums, casts) for sm_100a.  128-bit vectorised,
// coalesced, fp32 math; one CTA (or warp) per row.
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <algorithm>

#include <cooperative_groups.h>

#include "common.h"
#include "elem.h"

namespace mobius {
namespace {

template <typename T>
struct Vec;
template <>
struct Vec<float> {
  static constexpr int N = 4;
  __device__ static void load(const float* p, float* f) {
    float4 v = *reinterpret_cast<const float4*>(p);
    f[0] = v.x; f[1] = v.y; f[2] = v.z; f[3] = v.w;
  }
  __device__ static void store(float* p, const float* f) {
    *reinterpret_cast<float4*>(p) = make_float4(f[0], f[1], f[2], f[3]);
  }
};
template <>
struct Vec<__nv_bfloat16> {
  static constexpr int N = 8;
  __device__ static void load(const __nv_bfloat16* p, float* f) {
    uint4 v = *reinterpret_cast<const uint4*>(p);
    const __nv_bfloat162* h = reinterpret_cast<const __nv_bfloat162*>(&v);
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      float2 t = __bfloat1622float2(h[i]);
      f[2 * i] = t.x;
      f[2 * i + 1] = t.y;
    }
  }
  __device__ static void store(__nv_bfloat16* p, const float* f) {
    uint4 v;
    __nv_bfloat162* h = reinterpret_cast<__nv_bfloat162*>(&v);
#pragma unroll
    for (int i = 0; i < 4; ++i) h[i] = __floats2bfloat162_rn(f[2 * i], f[2 * i + 1]);
    *reinterpret_cast<uint4*>(p) = v;
  }
};

// 4 elements: one 16-byte (float) or 8-byte (bf16) access
template <typename T>
struct Vec4;
template <>
struct Vec4<float> {
  __device__ static void load(const float* p, float* f) {
    const float4 v = *reinterpret_cast<const float4*>(p);
    f[0] = v.x; f[1] = v.y; f[2] = v.z; f[3] = v.w;
  }
  __device__ static void store(float* p, const float* f) {
    *reinterpret_cast<float4*>(p) = make_float4(f[0], f[1], f[2], f[3]);
  }
};
template <>
struct Vec4<__nv_bfloat16> {
  __device__ static void load(const __nv_bfloat16* p, float* f) {
    const uint2 v = *reinterpret_cast<const uint2*>(p);
    const float2 a = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(&v.x));
    const float2 b = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(&v.y));
    f[0] = a.x; f[1] = a.y; f[2] = b.x; f[3] = b.y;
  }
  __device__ static void store(__nv_bfloat16* p, const float* f) {
    const __nv_bfloat162 a = __floats2bfloat162_rn(f[0], f[1]), b = __floats2bfloat162_rn(f[2], f[3]);
    uint2 v;
    v.x = *reinterpret_cast<const uint32_t*>(&a);
    v.y = *reinterpret_cast<const uint32_t*>(&b);
    *reinterpret_cast<uint2*>(p) = v;
  }
};

__device__ __forceinline__ float to_f(float x) { return x; }
__device__ __forceinline__ float to_f(__nv_bfloat16 x) { return __bfloat162float(x); }
template <typename T>
__device__ __forceinline__ T from_f(float x);
template <>
__device__ __forceinline__ float from_f<float>(float x) { return x; }
template <>
__device__ __forceinline__ __nv_bfloat16 from_f<__nv_bfloat16>(float x) { return __float2bfloat16_rn(x); }

__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}
__device__ __forceinline__ float warp_max(float v) {
#pragma unroll
  for (int o = 16; o; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}
// block-wide sum for blockDim.x == NT (multiple of 32, <= 1024)
template <int NT>
__device__ __forceinline__ float block_sum(float v, float* red) {
  v = warp_sum(v);
  const int w = threadIdx.x / 32, l = threadIdx.x % 32;
  __syncthreads();
  if (l == 0) red[w] = v;
  __syncthreads();
  float t = (threadIdx.x < NT / 32) ? red[threadIdx.x] : 0.f;
  if (w == 0) t = warp_sum(t);
  if (threadIdx.x == 0) red[32] = t;
  __syncthreads();
  return red[32];
}
template <int NT>
__device__ __forceinline__ float block_max(float v, float* red) {
  v = warp_max(v);
  const int w = threadIdx.x / 32, l = threadIdx.x % 32;
  __syncthreads();
  if (l == 0) red[w] = v;
  __syncthreads();
  float t = (threadIdx.x < NT / 32) ? red[threadIdx.x] : -INFINITY;
  if (w == 0) t = warp_max(t);
  if (threadIdx.x == 0) red[32] = t;
  __syncthreads();
  return red[32];
}

// ------------------------------------------------------------ embedding
template <typename T>
__global__ void embed_fwd_k(const int32_t* tok, const T* wte, const T* wpe, T* x, int s, int h) {
  constexpr int V = Vec<T>::N;
  const int r = blockIdx.x;
  const int b = r / s, i = r % s;
  const int t = tok[(int64_t)b * (s + 1) + i];
  const T* we = wte + (int64_t)t * h;
  const T* wp = wpe + (int64_t)i * h;
  T* o = x + (int64_t)r * h;
  for (int c = threadIdx.x * V; c < h; c += blockDim.x * V) {
    float a[V], p[V];
    Vec<T>::load(we + c, a);
    Vec<T>::load(wp + c, p);
#pragma unroll
    for (int k = 0; k < V; ++k) a[k] += p[k];
    Vec<T>::store(o + c, a);
  }
}

// dWte scatter, bf16 path: vector reductions (red.global.add.v4.f32) of
// each dx row into its token's fp32 row - one pass over dx, L2 resolves
// repeated tokens (the bf16 path is not bitwise reproducible anyway: the
// flash backward reduces dQ with TMA reduce-adds).
template <typename T>
__global__ void embed_bwd_wte_red_k(const int32_t* tok, const T* dx, float* dwte, int s, int h) {
  constexpr int V = Vec<T>::N;
  const int r = blockIdx.x;
  const int b = r / s, i = r % s;
  const int t = tok[(int64_t)b * (s + 1) + i];
  const T* g = dx + (int64_t)r * h;
  float* o = dwte + (int64_t)t * h;
  for (int c = threadIdx.x * V; c < h; c += blockDim.x * V) {
    float a[V];
    Vec<T>::load(g + c, a);
#pragma unroll
    for (int k = 0; k < V; k += 4)
      asm volatile("red.relaxed.gpu.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(o + c + k), "f"(a[k]),
                   "f"(a[k + 1]), "f"(a[k + 2]), "f"(a[k + 3])
                   : "memory");
  }
}

// dWte scatter, fp32 debug path: no float atomics, bitwise reproducible
// (the synchronous-update equivalence of P:L596-602 is checked bit for bit
// on this path).  CTA b owns the vocabulary rows [b*ids, (b+1)*ids).  It
// scans the microbatch's token ids in position order, EB_CHUNK at a time
// (each warp compacts a contiguous run of positions with ballots, so the
// per-warp lists concatenated in warp order are in position order), then
// every thread adds the dx rows of the matches into its own columns of the
// owned rows, in list order; a run of equal ids is summed in registers
// first.  Same-address read-modify-writes of one thread are program
// ordered, so the sums are in position order.
constexpr int EB_THREADS = 256;
constexpr int EB_CHUNK = 4096;                      // positions per scan round
constexpr int EB_PER_WARP = EB_CHUNK / (EB_THREADS / 32);
template <typename T>
__global__ void __launch_bounds__(EB_THREADS) embed_bwd_wte_det_k(const int32_t* __restrict__ tok,
                                                                  const T* __restrict__ dx, float* __restrict__ dwte,
                                                                  int mbs, int s, int h, int ids) {
  constexpr int V = Vec<T>::N;
  __shared__ int2 list[EB_CHUNK];                   // (row r, token id)
  __shared__ int wcount[EB_THREADS / 32];
  const int v0 = blockIdx.x * ids, v1 = v0 + ids;
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int T_ = mbs * s;
  for (int base = 0; base < T_; base += EB_CHUNK) {
    int n = 0;
    const int p0 = base + warp * EB_PER_WARP;
#pragma unroll 4
    for (int i = 0; i < EB_PER_WARP; i += 32) {
      const int r = p0 + i + lane;
      int t = -1;
      if (r < T_) t = __ldg(tok + (int64_t)(r / s) * (s + 1) + (r % s));
      const bool hit = t >= v0 && t < v1;
      const unsigned b = __ballot_sync(0xffffffffu, hit);
      if (hit) list[warp * EB_PER_WARP + n + __popc(b & ((1u << lane) - 1))] = make_int2(r, t);
      n += __popc(b);
    }
    if (lane == 0) wcount[warp] = n;
    __syncthreads();
    for (int c = threadIdx.x * V; c < h; c += EB_THREADS * V) {
      float acc[V];
      int prev = -1;
      for (int w = 0; w < EB_THREADS / 32; ++w) {
        const int nw = wcount[w];
        for (int k = 0; k < nw; ++k) {
          const int2 e = list[w * EB_PER_WARP + k];
          if (e.y != prev) {
            if (prev >= 0) {
              float* o = dwte + (int64_t)prev * h + c;
#pragma unroll
              for (int q = 0; q < V; ++q) o[q] += acc[q];
            }
#pragma unroll
            for (int q = 0; q < V; ++q) acc[q] = 0.f;
            prev = e.y;
          }
          float a[V];
          Vec<T>::load(dx + (int64_t)e.x * h + c, a);
#pragma unroll
          for (int q = 0; q < V; ++q) acc[q] += a[q];
        }
      }
      if (prev >= 0) {
        float* o = dwte + (int64_t)prev * h + c;
#pragma unroll
        for (int q = 0; q < V; ++q) o[q] += acc[q];
      }
    }
    __syncthreads();
  }
}

template <typename T>
__global__ void embed_bwd_wpe_k(const T* dx, float* dwpe, int mbs, int s, int h) {
  const int i = blockIdx.x;
  for (int c = threadIdx.x; c < h; c += blockDim.x) {
    float acc = 0.f;
    for (int b = 0; b < mbs; ++b) acc += to_f(dx[((int64_t)b * s + i) * h + c]);
    dwpe[(int64_t)i * h + c] += acc;
  }
}

// ------------------------------------------------------------ LayerNorm
// warp per row, the row held in registers (NV 16-byte vectors per lane)
template <typename T, int NV>
__global__ void __launch_bounds__(256) ln_fwd_warp_k(const T* __restrict__ x, const T* __restrict__ g,
                                                     const T* __restrict__ b, T* __restrict__ y, float* mu_out,
                                                     float* rstd_out, int rows, int h) {
  constexpr int V = Vec<T>::N;
  const int lane = threadIdx.x % 32;
  const int r = blockIdx.x * (blockDim.x / 32) + threadIdx.x / 32;
  if (r >= rows) return;
  const T* xr = x + (int64_t)r * h;
  float v[NV][V];
  float sum = 0.f;
#pragma unroll
  for (int k = 0; k < NV; ++k) {
    const int c = (lane + 32 * k) * V;
    if (c < h) {
      Vec<T>::load(xr + c, v[k]);
#pragma unroll
      for (int e = 0; e < V; ++e) sum += v[k][e];
    }
  }
  const float m = warp_sum(sum) / h;
  float q = 0.f;
#pragma unroll
  for (int k = 0; k < NV; ++k) {
    const int c = (lane + 32 * k) * V;
    if (c < h) {
#pragma unroll
      for (int e = 0; e < V; ++e) {
        const float d = v[k][e] - m;
        q += d * d;
      }
    }
  }
  const float rs = rsqrtf(warp_sum(q) / h + 1e-5f);
  if (lane == 0) {
    mu_out[r] = m;
    rstd_out[r] = rs;
  }
  T* yr = y + (int64_t)r * h;
#pragma unroll
  for (int k = 0; k < NV; ++k) {
    const int c = (lane + 32 * k) * V;
    if (c < h) {
      float gg[V], bb[V], o[V];
      Vec<T>::load(g + c, gg);
      Vec<T>::load(b + c, bb);
#pragma unroll
      for (int e = 0; e < V; ++e) o[e] = (v[k][e] - m) * rs * gg[e] + bb[e];
      Vec<T>::store(yr + c, o);
    }
  }
}

// bf16 LayerNorm, warp per row, the row held PACKED (8 bf16 per uint4
// register quad) so a warp needs 4*NV registers for it: ~2x the resident
// warps of the float-cached version, all row loads issued up front.  Same
// arithmetic and summation order as ln_fwd_warp_k / ln_bwd_dx_k, so the
// results are bit-identical to them.
__device__ __forceinline__ void unpack8(const uint4& u, float* f) {
  const __nv_bfloat162* h2 = reinterpret_cast<const __nv_bfloat162*>(&u);
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const float2 t = __bfloat1622float2(h2[i]);
    f[2 * i] = t.x;
    f[2 * i + 1] = t.y;
  }
}
__device__ __forceinline__ uint4 pack8(const float* f) {
  uint4 v;
  __nv_bfloat162* h2 = reinterpret_cast<__nv_bfloat162*>(&v);
#pragma unroll
  for (int i = 0; i < 4; ++i) h2[i] = __floats2bfloat162_rn(f[2 * i], f[2 * i + 1]);
  return v;
}

template <int NV>
__global__ void __launch_bounds__(256, 3) ln_fwd_bf16_k(const __nv_bfloat16* __restrict__ x,
                                                     const __nv_bfloat16* __restrict__ g,
                                                     const __nv_bfloat16* __restrict__ b, __nv_bfloat16* __restrict__ y,
                                                     float* mu_out, float* rstd_out, int rows, int h) {
  const int lane = threadIdx.x % 32;
  const int r = blockIdx.x * (blockDim.x / 32) + threadIdx.x / 32;
  if (r >= rows) return;
  const int nvec = h / 8;
  const uint4* xr = reinterpret_cast<const uint4*>(x + (int64_t)r * h);
  uint4 xv[NV];
#pragma unroll
  for (int k = 0; k < NV; ++k)
    if (lane + 32 * k < nvec) xv[k] = xr[lane + 32 * k];
  // packed f32x2 arithmetic (FADD2 / FFMA2 / FMUL2): the kernel is
  // instruction-issue bound (25.5 us warm vs 27 us cold at 16384 x 1600)
  float2 s2 = make_float2(0.f, 0.f);
#pragma unroll
  for (int k = 0; k < NV; ++k)
    if (lane + 32 * k < nvec) {
      const __nv_bfloat162* h2 = reinterpret_cast<const __nv_bfloat162*>(&xv[k]);
#pragma unroll
      for (int i = 0; i < 4; ++i) s2 = __fadd2_rn(s2, __bfloat1622float2(h2[i]));
    }
  const float m = warp_sum(s2.x + s2.y) / h;
  const float2 nm2 = make_float2(-m, -m);
  float2 q2 = make_float2(0.f, 0.f);
#pragma unroll
  for (int k = 0; k < NV; ++k)
    if (lane + 32 * k < nvec) {
      const __nv_bfloat162* h2 = reinterpret_cast<const __nv_bfloat162*>(&xv[k]);
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const float2 d = __fadd2_rn(__bfloat1622float2(h2[i]), nm2);
        q2 = __ffma2_rn(d, d, q2);
      }
    }
  const float rs = rsqrtf(warp_sum(q2.x + q2.y) / h + 1e-5f);
  if (lane == 0) {
    mu_out[r] = m;
    rstd_out[r] = rs;
  }
  const float2 rs2 = make_float2(rs, rs);
  uint4* yr = reinterpret_cast<uint4*>(y + (int64_t)r * h);
#pragma unroll
  for (int k = 0; k < NV; ++k)
    if (lane + 32 * k < nvec) {
      const uint4 gu = __ldg(reinterpret_cast<const uint4*>(g) + lane + 32 * k);
      const uint4 bu = __ldg(reinterpret_cast<const uint4*>(b) + lane + 32 * k);
      const __nv_bfloat162* x2 = reinterpret_cast<const __nv_bfloat162*>(&xv[k]);
      const __nv_bfloat162* g2 = reinterpret_cast<const __nv_bfloat162*>(&gu);
      const __nv_bfloat162* b2 = reinterpret_cast<const __nv_bfloat162*>(&bu);
      uint4 ov;
      __nv_bfloat162* o2 = reinterpret_cast<__nv_bfloat162*>(&ov);
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const float2 t = __fmul2_rn(__fadd2_rn(__bfloat1622float2(x2[i]), nm2), rs2);
        const float2 o = __ffma2_rn(t, __bfloat1622float2(g2[i]), __bfloat1622float2(b2[i]));
        o2[i] = __floats2bfloat162_rn(o.x, o.y);
      }
      yr[lane + 32 * k] = ov;
    }
}

template <typename T, int LN_NT, int LN_MAXV>
__global__ void __launch_bounds__(LN_NT) ln_fwd_k(const T* x, const T* g, const T* b, T* y, float* mu_out,
                                                   float* rstd_out, int h) {
  constexpr int V = Vec<T>::N;
  __shared__ float red[33];
  const int r = blockIdx.x;
  const T* xr = x + (int64_t)r * h;
  float v[LN_MAXV][V];
  float s = 0.f;
#pragma unroll
  for (int k = 0; k < LN_MAXV; ++k) {
    int c = (threadIdx.x + k * LN_NT) * V;
    if (c < h) {
      Vec<T>::load(xr + c, v[k]);
#pragma unroll
      for (int e = 0; e < V; ++e) s += v[k][e];
    }
  }
  const float mu = block_sum<LN_NT>(s, red) / h;
  float q = 0.f;
#pragma unroll
  for (int k = 0; k < LN_MAXV; ++k) {
    int c = (threadIdx.x + k * LN_NT) * V;
    if (c < h) {
#pragma unroll
      for (int e = 0; e < V; ++e) {
        float d = v[k][e] - mu;
        q += d * d;
      }
    }
  }
  const float var = block_sum<LN_NT>(q, red) / h;
  const float rs = rsqrtf(var + 1e-5f);
  if (threadIdx.x == 0) {
    mu_out[r] = mu;
    rstd_out[r] = rs;
  }
  T* yr = y + (int64_t)r * h;
#pragma unroll
  for (int k = 0; k < LN_MAXV; ++k) {
    int c = (threadIdx.x + k * LN_NT) * V;
    if (c < h) {
      float gg[V], bb[V], o[V];
      Vec<T>::load(g + c, gg);
      Vec<T>::load(b + c, bb);
#pragma unroll
      for (int e = 0; e < V; ++e) o[e] = (v[k][e] - mu) * rs * gg[e] + bb[e];
      Vec<T>::store(yr + c, o);
    }
  }
}

// ------------------------------------------------------ causal softmax
// one warp per row; row i of batch b: valid columns [0, i]
template <typename T>
__global__ void softmax_fwd_k(const float* S, T* P, int B, int s, float scale) {
  const int warps = blockDim.x / 32;
  const int64_t row = (int64_t)blockIdx.x * warps + threadIdx.x / 32;
  const int lane = threadIdx.x % 32;
  if (row >= (int64_t)B * s) return;
  const int i = (int)(row % s);
  const float* sr = S + row * s;
  T* pr = P + row * s;
  const int valid = i + 1;
  const int wend = min(s, ((i + 128) / 128) * 128);
  const float sl2 = scale * 1.4426950408889634f;
  float m = -INFINITY, l = 0.f;
  for (int j = lane; j < valid; j += 32) {
    float v = sr[j] * sl2;
    float nm = fmaxf(m, v);
    l = l * exp2f(m - nm) + exp2f(v - nm);
    m = nm;
  }
  float gm = warp_max(m);
  l = (m == -INFINITY) ? 0.f : l * exp2f(m - gm);
  l = warp_sum(l);
  const float inv = 1.f / l;
  for (int j = lane; j < wend; j += 32) {
    float p = 0.f;
    if (j < valid) p = exp2f(sr[j] * sl2 - gm) * inv;
    pr[j] = from_f<T>(p);
  }
}

template <typename T>
__global__ void softmax_bwd_k(const T* P, const float* dP, T* dS, int B, int s, float scale) {
  const int warps = blockDim.x / 32;
  const int64_t row = (int64_t)blockIdx.x * warps + threadIdx.x / 32;
  const int lane = threadIdx.x % 32;
  if (row >= (int64_t)B * s) return;
  const int i = (int)(row % s);
  const T* pr = P + row * s;
  const float* dr = dP + row * s;
  T* out = dS + row * s;
  const int valid = i + 1;
  const int wend = min(s, ((i + 128) / 128) * 128);
  float c = 0.f;
  for (int j = lane; j < valid; j += 32) c += to_f(pr[j]) * dr[j];
  c = warp_sum(c);
  for (int j = lane; j < wend; j += 32) {
    float v = 0.f;
    if (j < valid) v = scale * to_f(pr[j]) * (dr[j] - c);
    out[j] = from_f<T>(v);
  }
}

// ------------------------------------------------------- cross entropy
constexpr int CE_NT = 512;
template <typename T>
__global__ void __launch_bounds__(CE_NT) ce_k(T* z, const int32_t* tok, float* loss_rows, int V, int s,
                                              float inv_ntok) {
  constexpr int VW = Vec<T>::N;
  __shared__ float red[33];
  const int r = blockIdx.x;
  const int b = r / s, i = r % s;
  const int t = tok[(int64_t)b * (s + 1) + i + 1];
  T* zr = z + (int64_t)r * V;
  // online max / sum, rescaled once per vector (VW + 1 exponentials per VW
  // logits instead of 2 VW: the pass is MUFU-bound, not HBM-bound)
  float m = -INFINITY, l = 0.f;
  for (int c = threadIdx.x * VW; c < V; c += CE_NT * VW) {
    float f[VW];
    Vec<T>::load(zr + c, f);
    float vm = f[0];
#pragma unroll
    for (int e = 1; e < VW; ++e) vm = fmaxf(vm, f[e]);
    const float nm = fmaxf(m, vm);
    float sv = 0.f;
#pragma unroll
    for (int e = 0; e < VW; ++e) sv += __expf(f[e] - nm);
    l = l * __expf(m - nm) + sv;
    m = nm;
  }
  const float gm = block_max<CE_NT>(m, red);
  l = (m == -INFINITY) ? 0.f : l * __expf(m - gm);
  const float gl = block_sum<CE_NT>(l, red);
  const float zt = to_f(zr[t]);
  __syncthreads();  // everyone read zr[t] before it is overwritten
  const float inv = 1.f / gl;
  for (int c = threadIdx.x * VW; c < V; c += CE_NT * VW) {
    float f[VW];
    Vec<T>::load(zr + c, f);
#pragma unroll
    for (int e = 0; e < VW; ++e) {
      float p = __expf(f[e] - gm) * inv;
      if (c + e == t) p -= 1.f;
      f[e] = p * inv_ntok;
    }
    Vec<T>::store(zr + c, f);
  }
  if (threadIdx.x == 0) loss_rows[r] = logf(gl) + gm - zt;
}

__global__ void loss_acc_k(const float* loss_rows, int rows, double* acc) {
  __shared__ double red[32];
  double v = 0.0;
  for (int r = threadIdx.x; r < rows; r += blockDim.x) v += (double)loss_rows[r];
#pragma unroll
  for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  if (threadIdx.x % 32 == 0) red[threadIdx.x / 32] = v;
  __syncthreads();
  if (threadIdx.x == 0) {
    double t = 0.0;
    for (int w = 0; w < (int)blockDim.x / 32; ++w) t += red[w];
    acc[0] += t;
  }
}

// ----------------------------------------------------------- col sums
// ---------------------------------------------- LayerNorm backward (v2)
// dx only: one warp per row, two passes over the row (statistics, then dx),
// 16-byte vectors, no atomics.  dg/db come from ln_param_grad_k.
template <typename T>
__global__ void __launch_bounds__(256) ln_bwd_dx_k(const T* __restrict__ dy, const T* __restrict__ x,
                                                   const T* __restrict__ g, const float* __restrict__ mu,
                                                   const float* __restrict__ rstd, const T* __restrict__ dres,
                                                   T* __restrict__ dx, int rows, int h) {
  constexpr int V = Vec<T>::N;
  const int warps = blockDim.x / 32, lane = threadIdx.x % 32;
  for (int r = blockIdx.x * warps + threadIdx.x / 32; r < rows; r += gridDim.x * warps) {
    const float m = mu[r], rs = rstd[r];
    const T* xr = x + (int64_t)r * h;
    const T* dr = dy + (int64_t)r * h;
    float s1 = 0.f, s2 = 0.f;
#pragma unroll 4
    for (int c = lane * V; c < h; c += 32 * V) {
      float xv[V], dv[V], gv[V];
      Vec<T>::load(xr + c, xv);
      Vec<T>::load(dr + c, dv);
      Vec<T>::load(g + c, gv);
#pragma unroll
      for (int e = 0; e < V; ++e) {
        const float dh = dv[e] * gv[e];
        s1 += dh;
        s2 += dh * (xv[e] - m) * rs;
      }
    }
    s1 = warp_sum(s1) / h;
    s2 = warp_sum(s2) / h;
    T* o = dx + (int64_t)r * h;
    const T* rr = dres ? dres + (int64_t)r * h : nullptr;
#pragma unroll 4
    for (int c = lane * V; c < h; c += 32 * V) {
      float xv[V], dv[V], gv[V], ov[V];
      Vec<T>::load(xr + c, xv);
      Vec<T>::load(dr + c, dv);
      Vec<T>::load(g + c, gv);
      if (rr) Vec<T>::load(rr + c, ov);
#pragma unroll
      for (int e = 0; e < V; ++e) {
        const float val = rs * (dv[e] * gv[e] - s1 - (xv[e] - m) * rs * s2);
        ov[e] = rr ? ov[e] + val : val;
      }
      Vec<T>::store(o + c, ov);
    }
  }
}

// ------------------------------------- LayerNorm backward, fused (bf16)
// One pass over dy / x (/ dres): a persistent CTA per SM walks blocks of R
// rows; each block's dy, x (and dres) rows arrive in shared memory by bulk
// copies through a ring of LNF_NBUF buffers (the next LNF_NBUF - 1 blocks'
// rows are in flight while one is computed), then
//   phase A (warp per row): s1 = mean(dy g), s2 = mean(dy g xhat)
//   phase B (thread per 8-column vector, all R rows): dx = rstd (dy g - s1 -
//           xhat s2) (+ dres), and the thread's dgamma / dbeta partials
//           (sum of dy xhat, dy) over every row the CTA handles
// Each CTA writes its partial rows to part[cta] (fixed row order inside the
// CTA); ln_param_reduce_k adds the G partial rows in CTA order into dg / db:
// deterministic, dy and x read from DRAM once (the two-kernel version read
// them twice: 158 us at 32768 x 1600).
constexpr int LNF_THREADS = 256;
constexpr int LNF_MAXV = 4;  // column vectors per thread (h <= 256 * 8 * 4 = 8192)
constexpr int LNF_MAX_GRID = 512;
#ifndef MOBIUS_LNF_NBUF
#define MOBIUS_LNF_NBUF 2
#endif
constexpr int LNF_NBUF = MOBIUS_LNF_NBUF;  // row-block buffers in flight (ring)

__device__ __forceinline__ void lnf_bulk_g2s(uint32_t dst, const void* src, uint32_t bytes, uint32_t bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
               "l"(reinterpret_cast<uint64_t>(src)), "r"(bytes), "r"(bar)
               : "memory");
}
__device__ __forceinline__ uint32_t lnf_smem(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

#ifndef MOBIUS_LNF_CTAS
#define MOBIUS_LNF_CTAS 2  // CTAs per SM (shared-memory budget split between them)
#endif
template <int MAXV>  // column vectors per thread: ceil(h / 8 / LNF_THREADS)
__global__ void __launch_bounds__(LNF_THREADS, MOBIUS_LNF_CTAS)
    ln_bwd_fused_k(const __nv_bfloat16* __restrict__ dy, const __nv_bfloat16* __restrict__ x,
                   const __nv_bfloat16* __restrict__ g, const float* __restrict__ mu, const float* __restrict__ rstd,
                   const __nv_bfloat16* __restrict__ dres, __nv_bfloat16* __restrict__ dx, float* __restrict__ part,
                   int rows, int h, int R, int planes) {
  extern __shared__ __align__(128) uint8_t lnf_smem_raw[];
  // [LNF_NBUF buffers][dy | x (| dres)][R rows][h] bf16 (a block's rows are
  // contiguous in each tensor: one bulk copy per tensor), then R floats each
  // of mu, rstd, s1, s2, then LNF_NBUF mbarriers
  const int NT = dres ? 3 : 2;  // tensors per row
  __nv_bfloat16* buf = reinterpret_cast<__nv_bfloat16*>(lnf_smem_raw);
  float* st = reinterpret_cast<float*>(buf + (size_t)LNF_NBUF * R * NT * h);  // [4][R]
  uint64_t* bar = reinterpret_cast<uint64_t*>(st + 4 * R + 2);
  bar = reinterpret_cast<uint64_t*>((reinterpret_cast<uintptr_t>(bar) + 7) & ~uintptr_t(7));
  const int tid = threadIdx.x, warp = tid / 32, lane = tid % 32;
  const int nvec = h / 8;
  const int nblk = (rows + R - 1) / R;
  if (tid == 0) {
    for (int i = 0; i < LNF_NBUF; ++i)
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(lnf_smem(&bar[i])) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  auto issue = [&](int blk, int b) {  // one thread: rows of block blk -> buffer b
    const int r0 = blk * R, nr = min(R, rows - r0);
    const uint32_t bytes = (uint32_t)nr * NT * h * 2;
    const uint32_t bb = lnf_smem(&bar[b]);
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bb), "r"(bytes) : "memory");
    __nv_bfloat16* base = buf + (size_t)b * R * NT * h;
    const uint32_t tb = (uint32_t)nr * h * 2;
    lnf_bulk_g2s(lnf_smem(base), dy + (int64_t)r0 * h, tb, bb);
    lnf_bulk_g2s(lnf_smem(base + (size_t)R * h), x + (int64_t)r0 * h, tb, bb);
    if (dres) lnf_bulk_g2s(lnf_smem(base + (size_t)2 * R * h), dres + (int64_t)r0 * h, tb, bb);
  };
  // this thread's column vectors and their gamma
  float gv[MAXV][8], adg[MAXV][8], adb[MAXV][8], adr[MAXV][8];  // adr: column sums of dres (planes == 3)
#pragma unroll
  for (int k = 0; k < MAXV; ++k) {
    const int v = tid + k * LNF_THREADS;
#pragma unroll
    for (int e = 0; e < 8; ++e) adg[k][e] = adb[k][e] = adr[k][e] = 0.f;
    if (v < nvec) Vec<__nv_bfloat16>::load(g + v * 8, gv[k]);
  }
  const float inv_h = 1.f / (float)h;
  int it = 0;
  if (tid == 0)
    for (int k = 0; k < LNF_NBUF - 1; ++k)
      if ((int)blockIdx.x + k * (int)gridDim.x < nblk) issue(blockIdx.x + k * gridDim.x, k);
  for (int blk = blockIdx.x; blk < nblk; blk += gridDim.x, ++it) {
    const int b = it % LNF_NBUF;
    const int r0 = blk * R, nr = min(R, rows - r0);
    // buffer (it - 1) % LNF_NBUF was released by the __syncthreads that ended the previous block
    const int ahead = blk + (LNF_NBUF - 1) * (int)gridDim.x;
    if (tid == 0 && ahead < nblk) issue(ahead, (it + LNF_NBUF - 1) % LNF_NBUF);
    {
      const uint32_t bb = lnf_smem(&bar[b]), ph = (uint32_t)(it / LNF_NBUF) & 1u;
      asm volatile(
          "{\n\t.reg .pred P1;\n\tLNF_WAIT:\n\t"
          "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1, 10000000;\n\t"
          "@P1 bra LNF_DONE;\n\tbra LNF_WAIT;\n\tLNF_DONE:\n\t}\n" ::"r"(bb),
          "r"(ph)
          : "memory");
    }
    const __nv_bfloat16* bs = buf + (size_t)b * R * NT * h;
    float* sm = st;  // mu | rstd | s1 | s2 of this block
    // phase A: row statistics, warp per row
    for (int r = warp; r < nr; r += LNF_THREADS / 32) {
      const float m = mu[r0 + r], rs = rstd[r0 + r];
      const __nv_bfloat16* dr = bs + (size_t)r * h;
      float s1 = 0.f, s2 = 0.f;
      for (int v = lane; v < nvec; v += 32) {
        float dv[8], xv[8], gg[8];
        Vec<__nv_bfloat16>::load(dr + v * 8, dv);
        Vec<__nv_bfloat16>::load(dr + (size_t)R * h + v * 8, xv);
        Vec<__nv_bfloat16>::load(g + v * 8, gg);
#pragma unroll
        for (int e = 0; e < 8; ++e) {
          const float dh = dv[e] * gg[e];
          s1 += dh;
          s2 += dh * (xv[e] - m) * rs;
        }
      }
      s1 = warp_sum(s1);
      s2 = warp_sum(s2);
      if (lane == 0) {
        sm[r] = m;
        sm[R + r] = rs;
        sm[2 * R + r] = s1 * inv_h;
        sm[3 * R + r] = s2 * inv_h;
      }
    }
    __syncthreads();
    // phase B: dx and the parameter-gradient partials, thread per column vector
#pragma unroll
    for (int k = 0; k < MAXV; ++k) {
      const int v = tid + k * LNF_THREADS;
      if (v >= nvec) continue;
      for (int r = 0; r < nr; ++r) {
        const float m = sm[r], rs = sm[R + r], s1 = sm[2 * R + r], s2 = sm[3 * R + r];
        const __nv_bfloat16* dr = bs + (size_t)r * h;
        float dv[8], xv[8], ov[8];
        Vec<__nv_bfloat16>::load(dr + v * 8, dv);
        Vec<__nv_bfloat16>::load(dr + (size_t)R * h + v * 8, xv);
        const int64_t off = (int64_t)(r0 + r) * h + v * 8;
        if (dres) {
          Vec<__nv_bfloat16>::load(dr + (size_t)2 * R * h + v * 8, ov);
#pragma unroll
          for (int e = 0; e < 8; ++e) adr[k][e] += ov[e];
        }
#pragma unroll
        for (int e = 0; e < 8; ++e) {
          const float xh = (xv[e] - m) * rs;
          const float val = rs * (dv[e] * gv[k][e] - s1 - (xv[e] - m) * rs * s2);
          ov[e] = dres ? ov[e] + val : val;
          adg[k][e] += dv[e] * xh;
          adb[k][e] += dv[e];
        }
        Vec<__nv_bfloat16>::store(dx + off, ov);
      }
    }
    __syncthreads();  // buffer b and the row statistics are free again
  }
  // partial rows: part[cta][0][c] = dgamma, part[cta][1][c] = dbeta (, part[cta][2][c] = sum dres)
  float* pr = part + (size_t)blockIdx.x * planes * h;
#pragma unroll
  for (int k = 0; k < MAXV; ++k) {
    const int v = tid + k * LNF_THREADS;
    if (v >= nvec) continue;
#pragma unroll
    for (int e = 0; e < 8; e += 4) {
      *reinterpret_cast<float4*>(pr + v * 8 + e) = make_float4(adg[k][e], adg[k][e + 1], adg[k][e + 2], adg[k][e + 3]);
      *reinterpret_cast<float4*>(pr + h + v * 8 + e) =
          make_float4(adb[k][e], adb[k][e + 1], adb[k][e + 2], adb[k][e + 3]);
      if (planes == 3)
        *reinterpret_cast<float4*>(pr + 2 * h + v * 8 + e) =
            make_float4(adr[k][e], adr[k][e + 1], adr[k][e + 2], adr[k][e + 3]);
    }
  }
}

// dg[c] += sum_{cta} part[cta][0][c], db[c] += sum_{cta} part[cta][1][c]:
// a CTA per 32 columns (lane = column, coalesced), warp w sums partials
// w, w + 32, ... in order, warp 0 adds the 32 warp sums in order - a fixed
// summation order (deterministic).  (A thread per column summing all G
// partials serially took 21 us at h 1600, G 296.)
constexpr int LNR_WARPS = 32;
__global__ void __launch_bounds__(32 * LNR_WARPS) ln_param_reduce_k(const float* __restrict__ part, int G, int h,
                                                                    int planes, float* dg, float* db, float* dr) {
  __shared__ float red[LNR_WARPS][32];
  const int lane = threadIdx.x % 32, w = threadIdx.x / 32;
  const int i = blockIdx.x * 32 + lane;
  float s = 0.f;
  if (i < planes * h) {
#pragma unroll 4
    for (int c = w; c < G; c += LNR_WARPS) s += part[(size_t)c * planes * h + i];
  }
  red[w][lane] = s;
  __syncthreads();
  if (w == 0 && i < planes * h) {
    float t = 0.f;
#pragma unroll
    for (int k = 0; k < LNR_WARPS; ++k) t += red[k][lane];
    if (i < h)
      dg[i] += t;
    else if (i < 2 * h)
      db[i - h] += t;
    else
      dr[i - 2 * h] += t;
  }
}

// Column reductions over `rows` rows, 16-byte vectors per thread, partial
// sums in registers, CTA-level smem reduction.  mode 0: out0[c] += sum_r
// X[r,c].  mode 1 (LayerNorm parameters): out0[c] += sum_r X[r,c] *
// (Y[r,c] - mu[r]) * rstd[r] (dgamma), out1[c] += sum_r X[r,c] (dbeta).
// Deterministic, no float atomics: the CS_CL CTAs of a cluster (stacked
// along the rows) add their column totals through distributed shared memory
// in rank order; each cluster leader writes one partial row; the last
// leader of a column slab to arrive (arrival counter, reset by it) adds the
// gridDim.y / CS_CL partials to out in order.
constexpr int CS_THREADS = 256;
constexpr int CS_COLV = 32;  // column vectors (of 8/4 elements) per CTA
constexpr int CS_CL = 8;     // CTAs per cluster (rows direction)
template <typename T, int MODE>
__global__ void __cluster_dims__(1, CS_CL, 1) __launch_bounds__(CS_THREADS)
    colsum2_k(const T* __restrict__ X, int64_t ld, const T* __restrict__ Y, const float* __restrict__ mu,
              const float* __restrict__ rstd, int rows, int n, float* out0, float* out1, int rows_per_cta,
              float* part, unsigned* cnt) {
  constexpr int V = Vec<T>::N;
  constexpr int W = CS_COLV * V;  // columns per CTA
  __shared__ float red0[CS_THREADS / CS_COLV][W];
  __shared__ float red1[MODE == 1 ? CS_THREADS / CS_COLV : 1][MODE == 1 ? W : 1];
  __shared__ float tot[MODE == 1 ? 2 : 1][W];
  __shared__ bool last;
  const int cv = threadIdx.x % CS_COLV;  // column vector within the CTA's slab
  const int rg = threadIdx.x / CS_COLV;  // row group (CS_THREADS / CS_COLV groups)
  const int c = (blockIdx.x * CS_COLV + cv) * V;
  const int r0 = blockIdx.y * rows_per_cta, r1 = min(rows, r0 + rows_per_cta);
  float a0[V], a1[V];
#pragma unroll
  for (int e = 0; e < V; ++e) a0[e] = a1[e] = 0.f;
  if (c < n) {
#pragma unroll 4
    for (int r = r0 + rg; r < r1; r += CS_THREADS / CS_COLV) {
      float xv[V];
      Vec<T>::load(X + (int64_t)r * ld + c, xv);
      if (MODE == 0) {
#pragma unroll
        for (int e = 0; e < V; ++e) a0[e] += xv[e];
      } else {
        float yv[V];
        Vec<T>::load(Y + (int64_t)r * ld + c, yv);
        const float m = mu[r], rs = rstd[r];
#pragma unroll
        for (int e = 0; e < V; ++e) {
          a0[e] += xv[e] * (yv[e] - m) * rs;
          a1[e] += xv[e];
        }
      }
    }
  }
#pragma unroll
  for (int e = 0; e < V; ++e) {
    red0[rg][cv * V + e] = a0[e];
    if (MODE == 1) red1[rg][cv * V + e] = a1[e];
  }
  __syncthreads();
  for (int i = threadIdx.x; i < W; i += CS_THREADS) {
    float t0 = 0.f, t1 = 0.f;
#pragma unroll
    for (int g2 = 0; g2 < CS_THREADS / CS_COLV; ++g2) {
      t0 += red0[g2][i];
      if (MODE == 1) t1 += red1[g2][i];
    }
    tot[0][i] = t0;
    if (MODE == 1) tot[MODE][i] = t1;
  }
  // cluster: the leader adds the CS_CL CTA totals in rank order (DSMEM)
  namespace cg = cooperative_groups;
  cg::cluster_group cluster = cg::this_cluster();
  cluster.sync();
  const bool leader = cluster.block_rank() == 0;
  const int64_t nparts = gridDim.y / CS_CL;
  const int64_t prow = blockIdx.y / CS_CL;
  if (leader) {
    for (int i = threadIdx.x; i < W; i += CS_THREADS) {
      const int col = blockIdx.x * W + i;
      float t0 = 0.f, t1 = 0.f;
#pragma unroll
      for (int r = 0; r < CS_CL; ++r) {
        const float* rt = cluster.map_shared_rank(&tot[0][0], r);
        t0 += rt[i];
        if (MODE == 1) t1 += rt[W + i];
      }
      if (col < n) {
        part[prow * n + col] = t0;
        if (MODE == 1) part[(nparts + prow) * n + col] = t1;
      }
    }
  }
  cluster.sync();  // remote reads done before any CTA of the cluster exits
  if (!leader) return;
  __threadfence();
  __syncthreads();
  if (threadIdx.x == 0) last = atomicInc(cnt + blockIdx.x, (unsigned)nparts - 1) == (unsigned)nparts - 1;  // wraps to 0
  __syncthreads();
  if (!last) return;
  __threadfence();
  for (int i = threadIdx.x; i < W; i += CS_THREADS) {
    const int col = blockIdx.x * W + i;
    if (col >= n) continue;
    float t0 = 0.f, t1 = 0.f;
    for (int64_t g2 = 0; g2 < nparts; ++g2) {
      t0 += __ldcg(part + g2 * n + col);
      if (MODE == 1) t1 += __ldcg(part + (nparts + g2) * n + col);
    }
    out0[col] += t0;
    if (MODE == 1) out1[col] += t1;
  }
}

// generic fallback (unaligned / odd widths): one thread per column sums all
// rows in order (deterministic; never on the hot path)
template <typename T>
__global__ void colsum_k(const T* X, int64_t ld, int rows, int n, float* out) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= n) return;
  float acc = 0.f;
  for (int r = 0; r < rows; ++r) acc += to_f(X[(int64_t)r * ld + c]);
  out[c] += acc;
}

template <typename T>
__global__ void cast_k(const float* src, T* dst, int64_t n) {
  int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) * 4;
  int64_t stride = (int64_t)gridDim.x * blockDim.x * 4;
  for (; i < n; i += stride) {
    if (i + 4 <= n) {
      float4 v = *reinterpret_cast<const float4*>(src + i);
      dst[i] = from_f<T>(v.x);
      dst[i + 1] = from_f<T>(v.y);
      dst[i + 2] = from_f<T>(v.z);
      dst[i + 3] = from_f<T>(v.w);
    } else {
      for (int64_t k = i; k < n; ++k) dst[k] = from_f<T>(src[k]);
    }
  }
}

template <typename T>
__global__ void fill_ones_col_k(T* p, int64_t n) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    p[i] = from_f<T>((i & 63) == 0 ? 1.f : 0.f);
}

__global__ void tokens_check_k(const int32_t* __restrict__ src, int32_t* __restrict__ dst, int64_t n, int V,
                               int* bad) {
  int cnt = 0;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t t = src[i];
    cnt += (uint32_t)t >= (uint32_t)V;
    dst[i] = t;
  }
  cnt = __reduce_add_sync(0xffffffffu, cnt);
  if (cnt && threadIdx.x % 32 == 0) atomicAdd(bad, cnt);  // integer count: order-independent
}

__global__ void flag_wait_k(const volatile int* flag, int value) {
  int v;
  do {
    asm volatile("ld.acquire.sys.global.s32 %0, [%1];" : "=r"(v) : "l"(flag) : "memory");
    if (v >= value) break;
    __nanosleep(200);
  } while (true);
}
__global__ void flag_set_k(int* flag, int value) {
  asm volatile("st.release.sys.global.s32 [%0], %1;" ::"l"(flag), "r"(value) : "memory");
}

int check_launch(const char* what) {
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) MOBIUS_FAIL(MOBIUS_ECUDA, "%s: %s", what, cudaGetErrorString(e));
  return MOBIUS_OK;
}

// rows per CTA so the column reduction launches >= ~4 waves of 148 SMs
int colsum_rows_per_cta(int col_ctas, int rows) {
  int rpc = 256;
  while (rpc > 32 && (int64_t)col_ctas * ((rows + rpc - 1) / rpc) < 4 * 148) rpc /= 2;
  return rpc;
}
// grid of colsum2_k for n columns of vector width vw (gy a multiple of the
// cluster size; trailing CTAs of a short last cluster have no rows)
void colsum_grid(int rows, int n, int vw, int* gx, int* gy, int* rpc) {
  *gx = (n / vw + CS_COLV - 1) / CS_COLV;
  *rpc = colsum_rows_per_cta(*gx, rows);
  *gy = ((rows + *rpc - 1) / *rpc + CS_CL - 1) / CS_CL * CS_CL;
}

template <typename T>
bool aligned16(const T* p) {
  return (reinterpret_cast<uintptr_t>(p) & 15) == 0;
}

}  // namespace

template <typename T>
int embed_fwd(const int32_t* tok, const T* wte, const T* wpe, T* x, int mbs, int s, int h, cudaStream_t st) {
  MOBIUS_CHECK_ARG(h % Vec<T>::N == 0, "embed: h %% vec");
  embed_fwd_k<T><<<mbs * s, 128, 0, st>>>(tok, wte, wpe, x, s, h);
  return check_launch("embed_fwd");
}
template <typename T>
int embed_bwd(const int32_t* tok, const T* dx, float* dwte, float* dwpe, int mbs, int s, int h, int V,
              cudaStream_t st) {
  MOBIUS_CHECK_ARG(h % 8 == 0 && (reinterpret_cast<uintptr_t>(dwte) & 15) == 0 && V > 0,
                   "embed_bwd: h %% 8 and a 16-byte aligned dWte are required");
  if constexpr (sizeof(T) == 2) {
    embed_bwd_wte_red_k<T><<<mbs * s, 128, 0, st>>>(tok, dx, dwte, s, h);
  } else {
    // ~4 CTAs per SM, each owning ceil(V / grid) vocabulary rows
    const int grid = std::min(V, 148 * 4);
    const int ids = (V + grid - 1) / grid;
    embed_bwd_wte_det_k<T><<<(V + ids - 1) / ids, EB_THREADS, 0, st>>>(tok, dx, dwte, mbs, s, h, ids);
  }
  int rc = check_launch("embed_bwd_wte");
  if (rc) return rc;
  embed_bwd_wpe_k<T><<<s, 256, 0, st>>>(dx, dwpe, mbs, s, h);
  return check_launch("embed_bwd_wpe");
}

// (threads, vectors per thread) from the number of 16-byte vectors per row
#define LN_DISPATCH(KERNEL, GRID, ...)                                         \
  do {                                                                         \
    const int nv = h / Vec<T>::N;                                              \
    if (nv <= 128) KERNEL<T, 128, 1><<<GRID, 128, 0, st>>>(__VA_ARGS__);      \
    else if (nv <= 256) KERNEL<T, 128, 2><<<GRID, 128, 0, st>>>(__VA_ARGS__); \
    else if (nv <= 512) KERNEL<T, 128, 4><<<GRID, 128, 0, st>>>(__VA_ARGS__); \
    else if (nv <= 1024) KERNEL<T, 256, 4><<<GRID, 256, 0, st>>>(__VA_ARGS__);\
    else if (nv <= 2048) KERNEL<T, 256, 8><<<GRID, 256, 0, st>>>(__VA_ARGS__);\
    else MOBIUS_FAIL(MOBIUS_EINVAL, "layernorm: h=%d too large", h);          \
  } while (0)

// MOBIUS_LN_FLOATROW=1 selects the float-cached row LN forward (A/B timing)
static bool ln_packed() {
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("MOBIUS_LN_FLOATROW");
    v = (e && e[0] == '1') ? 0 : 1;
  }
  return v == 1;
}

template <typename T>
int layernorm_fwd(const T* x, const T* g, const T* b, T* y, float* mu, float* rstd, int rows, int h, cudaStream_t st) {
  MOBIUS_CHECK_ARG(h % Vec<T>::N == 0, "layernorm: unsupported h=%d", h);
  const int nv = (h / Vec<T>::N + 31) / 32;  // vectors per lane
  const unsigned blocks = (unsigned)((rows + 7) / 8);
  if constexpr (sizeof(T) == 2) {
    if (ln_packed() && nv <= 8 && aligned16(x) && aligned16(y) && aligned16(g) && aligned16(b)) {
#define LNF(NV) ln_fwd_bf16_k<NV><<<blocks, 256, 0, st>>>(x, g, b, y, mu, rstd, rows, h)
      if (nv <= 4) LNF(4);
      else if (nv == 5) LNF(5);
      else if (nv == 6) LNF(6);
      else if (nv == 7) LNF(7);
      else LNF(8);
#undef LNF
      return check_launch("layernorm_fwd");
    }
  }
  if (nv <= 4)
    ln_fwd_warp_k<T, 4><<<blocks, 256, 0, st>>>(x, g, b, y, mu, rstd, rows, h);
  else if (nv <= 8)
    ln_fwd_warp_k<T, 8><<<blocks, 256, 0, st>>>(x, g, b, y, mu, rstd, rows, h);
  else
    LN_DISPATCH(ln_fwd_k, rows, x, g, b, y, mu, rstd, h);
  return check_launch("layernorm_fwd");
}
// rows per block of the fused bf16 LN backward (LNF_NBUF buffers of R rows
// of nt tensors in <= 200 KB of shared memory), 0 when it does not apply
// (at least 4 rows: with fewer, phase A leaves most warps idle and the
// per-block barriers dominate - h 5120 with 1-2 rows per block was slower
// than the two-kernel path)
static int lnf_rows(int h, int nt) {
  if (h % 8 || h > 256 * 8 * LNF_MAXV) return 0;
  const int r = std::min((200 * 1024 / MOBIUS_LNF_CTAS) / (LNF_NBUF * nt * h * 2), 16);
  return r >= 4 ? r : 0;
}
static int lnf_smem_bytes(int h, int R, int nt) { return LNF_NBUF * R * nt * h * 2 + 4 * R * 4 + 8 * LNF_NBUF + 64; }
static int lnf_grid() {
  static int g = 0;
  if (!g) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&g, cudaDevAttrMultiProcessorCount, dev);
    g = std::min(g * MOBIUS_LNF_CTAS, LNF_MAX_GRID);
  }
  return g;
}

template <int MV>
static int lnf_launch(int G, int smem, cudaStream_t st, const __nv_bfloat16* dy, const __nv_bfloat16* x,
                      const __nv_bfloat16* g, const float* mu, const float* rstd, const __nv_bfloat16* dres,
                      __nv_bfloat16* dx, float* part, int rows, int h, int R, int planes) {
  static int smem_set = 0;  // per instantiation
  if (smem > smem_set) {
    if (cudaFuncSetAttribute(ln_bwd_fused_k<MV>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) != cudaSuccess)
      MOBIUS_FAIL(MOBIUS_ECUDA, "layernorm_bwd: smem attribute");
    smem_set = smem;
  }
  ln_bwd_fused_k<MV><<<G, LNF_THREADS, smem, st>>>(dy, x, g, mu, rstd, dres, dx, part, rows, h, R, planes);
  return MOBIUS_OK;
}

static bool lnf_enabled() {
  static int fused = -1;
  if (fused < 0) {
    const char* e = getenv("MOBIUS_LN_BWD_FUSED");
    fused = e ? atoi(e) : 1;
  }
  return fused != 0;
}

template <typename T>
int layernorm_bwd_launches(int h, bool dres, bool dres_sum) {
  if (sizeof(T) == 2 && lnf_enabled() && lnf_rows(h, dres ? 3 : 2)) return 2;
  return dres_sum ? 3 : 2;
}

template <typename T>
int layernorm_bwd(const T* dy, const T* x, const T* g, const float* mu, const float* rstd, const T* dres, T* dx,
                  float* dg, float* db, int rows, int h, const RedWs& ws, cudaStream_t st, float* dres_sum) {
  MOBIUS_CHECK_ARG(h % Vec<T>::N == 0, "layernorm: unsupported h=%d", h);
  MOBIUS_CHECK_ARG(!dres_sum || dres, "layernorm_bwd: dres_sum needs dres");
  if constexpr (sizeof(T) == 2) {
    const int nt = dres ? 3 : 2;
    const int R = lnf_rows(h, nt);
    if (lnf_enabled() && R && aligned16(dy) && aligned16(x) && aligned16(dx) && (!dres || aligned16(dres))) {
      MOBIUS_CHECK_ARG(ws.part, "layernorm_bwd: reduction workspace");
      const int G = std::min(lnf_grid(), (rows + R - 1) / R);
      const int smem = lnf_smem_bytes(h, R, nt);
      const int mv = (h / 8 + LNF_THREADS - 1) / LNF_THREADS;
      const int planes = dres_sum ? 3 : 2;
      const auto* a = (const __nv_bfloat16*)dy;
      int rc = mv == 1   ? lnf_launch<1>(G, smem, st, a, (const __nv_bfloat16*)x, (const __nv_bfloat16*)g, mu, rstd,
                                         (const __nv_bfloat16*)dres, (__nv_bfloat16*)dx, ws.part, rows, h, R, planes)
               : mv == 2 ? lnf_launch<2>(G, smem, st, a, (const __nv_bfloat16*)x, (const __nv_bfloat16*)g, mu, rstd,
                                         (const __nv_bfloat16*)dres, (__nv_bfloat16*)dx, ws.part, rows, h, R, planes)
                         : lnf_launch<4>(G, smem, st, a, (const __nv_bfloat16*)x, (const __nv_bfloat16*)g, mu, rstd,
                                         (const __nv_bfloat16*)dres, (__nv_bfloat16*)dx, ws.part, rows, h, R, planes);
      if (rc) return rc;
      rc = check_launch("layernorm_bwd_fused");
      if (rc) return rc;
      ln_param_reduce_k<<<(planes * h + 31) / 32, 32 * LNR_WARPS, 0, st>>>(ws.part, G, h, planes, dg, db, dres_sum);
      return check_launch("layernorm_param_reduce");
    }
  }
  // dx, then gamma / beta grads by a column-reduction pass.  Caching the
  // row's x and dy in registers for the second pass (one read each instead
  // of a re-read that hits L1/L2 anyway) was measured slower at 32768 x
  // 1600: 179 us (warp per row, 128 registers) and 166 us (two warps per
  // row, 80 registers) against 158 us for this kernel + the column pass -
  // fewer resident warps cost more than the L2 re-reads save.  Fusing the
  // param grads into the dx pass was measured slower at 8192 x 1600 (42 us
  // unfused; 114 us with red.shared.add per element - 8-way bank conflicts
  // on the 8-column lane vectors; 64 us with per-warp private smem slices)
  {
    int blocks = (rows + 7) / 8;
    if (blocks > 148 * 16) blocks = 148 * 16;
    ln_bwd_dx_k<T><<<blocks, 256, 0, st>>>(dy, x, g, mu, rstd, dres, dx, rows, h);
  }
  int rc = check_launch("layernorm_bwd_dx");
  if (rc) return rc;
  {
    int gx, gy, rpc;
    colsum_grid(rows, h, Vec<T>::N, &gx, &gy, &rpc);
    MOBIUS_CHECK_ARG(ws.part && ws.cnt && gx <= RED_WS_COUNTERS, "layernorm_bwd: reduction workspace");
    colsum2_k<T, 1><<<dim3(gx, gy), CS_THREADS, 0, st>>>(dy, h, x, mu, rstd, rows, h, dg, db, rpc, ws.part, ws.cnt);
  }
  int rc2 = check_launch("layernorm_param_grad");
  if (rc2 || !dres_sum) return rc2;
  return colsum_accum<T>(dres, h, rows, h, dres_sum, ws, st);
}

template <typename T>
int softmax_causal_fwd(const float* S, T* P, int B, int s, float scale, cudaStream_t st) {
  int64_t rows = (int64_t)B * s;
  softmax_fwd_k<T><<<(unsigned)((rows + 7) / 8), 256, 0, st>>>(S, P, B, s, scale);
  return check_launch("softmax_fwd");
}
template <typename T>
int softmax_causal_bwd(const T* P, const float* dP, T* dS, int B, int s, float scale, cudaStream_t st) {
  int64_t rows = (int64_t)B * s;
  softmax_bwd_k<T><<<(unsigned)((rows + 7) / 8), 256, 0, st>>>(P, dP, dS, B, s, scale);
  return check_launch("softmax_bwd");
}

template <typename T>
int cross_entropy_fwd_bwd(T* logits, const int32_t* tok, float* loss_rows, int rows, int V, int s, float inv_ntok,
                          cudaStream_t st) {
  MOBIUS_CHECK_ARG(V % Vec<T>::N == 0, "cross_entropy: V %% vec");
  ce_k<T><<<rows, CE_NT, 0, st>>>(logits, tok, loss_rows, V, s, inv_ntok);
  return check_launch("cross_entropy");
}

int loss_accumulate(const float* loss_rows, int rows, double* acc, cudaStream_t st) {
  loss_acc_k<<<1, 1024, 0, st>>>(loss_rows, rows, acc);
  return check_launch("loss_accumulate");
}

int64_t colsum_ws_floats(int rows, int n, int planes) {
  // the bf16 grid (8-wide vectors) has fewer column CTAs, hence more row CTAs;
  // the fused LN backward (planes 2) needs one partial row pair per CTA
  int64_t best = planes == 2 ? (int64_t)LNF_MAX_GRID * n * 3 : 0;  // (+ the dres column sums)
  for (int vw : {4, 8}) {
    int gx, gy, rpc;
    colsum_grid(rows, n, vw, &gx, &gy, &rpc);
    best = std::max<int64_t>(best, (int64_t)(gy / CS_CL) * n * planes);
  }
  return best;
}

template <typename T>
int colsum_accum(const T* X, int64_t ld, int rows, int n, float* out, const RedWs& ws, cudaStream_t st) {
  if (n % Vec<T>::N == 0 && ld % Vec<T>::N == 0 && aligned16(X)) {
    int gx, gy, rpc;
    colsum_grid(rows, n, Vec<T>::N, &gx, &gy, &rpc);
    MOBIUS_CHECK_ARG(ws.part && ws.cnt && gx <= RED_WS_COUNTERS, "colsum: reduction workspace");
    colsum2_k<T, 0><<<dim3(gx, gy), CS_THREADS, 0, st>>>(X, ld, (const T*)nullptr, nullptr, nullptr, rows, n, out,
                                                         nullptr, rpc, ws.part, ws.cnt);
    return check_launch("colsum");
  }
  colsum_k<T><<<(n + 255) / 256, 256, 0, st>>>(X, ld, rows, n, out);
  return check_launch("colsum");
}

// AdamW, one thread per 4 parameters (float4 master/m/v, 4 gradients);
// arithmetic in the order of host.cpp adamw_chunk (x -= lr*wd*x; m, v
// moments; x -= lr * (m/bc1) / (sqrt(v/bc2) + eps)), no FMA contraction so
// the result matches the scalar host update bit for bit.
__device__ __forceinline__ float adamw_one(float& w, float& m, float& v, float g, float lr, float b1, float b2,
                                           float eps, float lrwd, float bc1, float bc2) {
  float x = __fsub_rn(w, __fmul_rn(lrwd, w));
  const float mi = __fadd_rn(__fmul_rn(b1, m), __fmul_rn(__fsub_rn(1.f, b1), g));
  const float vi = __fadd_rn(__fmul_rn(b2, v), __fmul_rn(__fmul_rn(__fsub_rn(1.f, b2), g), g));
  x = __fsub_rn(x, __fdiv_rn(__fmul_rn(lr, __fdiv_rn(mi, bc1)), __fadd_rn(__fsqrt_rn(__fdiv_rn(vi, bc2)), eps)));
  m = mi;
  v = vi;
  w = x;
  return x;
}

template <typename T>
__global__ void adamw_k(float4* __restrict__ w, float4* __restrict__ m, float4* __restrict__ v, const T* __restrict__ g,
                        T* __restrict__ wo, int64_t n, float lr, float b1, float b2, float eps, float lrwd, float bc1,
                        float bc2) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i * 4 < n; i += (int64_t)gridDim.x * blockDim.x) {
    if (i * 4 + 4 <= n) {
      float4 a = w[i], b = m[i], c = v[i];
      float gg[4], o[4];
      Vec4<T>::load(g + i * 4, gg);
      o[0] = adamw_one(a.x, b.x, c.x, gg[0], lr, b1, b2, eps, lrwd, bc1, bc2);
      o[1] = adamw_one(a.y, b.y, c.y, gg[1], lr, b1, b2, eps, lrwd, bc1, bc2);
      o[2] = adamw_one(a.z, b.z, c.z, gg[2], lr, b1, b2, eps, lrwd, bc1, bc2);
      o[3] = adamw_one(a.w, b.w, c.w, gg[3], lr, b1, b2, eps, lrwd, bc1, bc2);
      w[i] = a;
      m[i] = b;
      v[i] = c;
      Vec4<T>::store(wo + i * 4, o);
    } else {
      float* wf = reinterpret_cast<float*>(w);
      float* mf = reinterpret_cast<float*>(m);
      float* vf = reinterpret_cast<float*>(v);
      for (int64_t k = i * 4; k < n; ++k)
        wo[k] = from_f<T>(adamw_one(wf[k], mf[k], vf[k], to_f(g[k]), lr, b1, b2, eps, lrwd, bc1, bc2));
    }
  }
}

template <typename T>
int adamw_device(float* w, float* m, float* v, const T* g, T* w_out, int64_t n, float lr, float b1, float b2,
                 float eps, float wd, float bc1, float bc2, cudaStream_t st) {
  if (n <= 0) return MOBIUS_OK;
  MOBIUS_CHECK_ARG(((uintptr_t)w | (uintptr_t)m | (uintptr_t)v) % 16 == 0 && (uintptr_t)g % 8 == 0 &&
                       (uintptr_t)w_out % 8 == 0,
                   "adamw_device: misaligned buffers");
  const int64_t n4 = (n + 3) / 4;
  const int64_t blocks = std::min<int64_t>((n4 + 255) / 256, 148 * 16);
  adamw_k<T><<<(unsigned)blocks, 256, 0, st>>>(reinterpret_cast<float4*>(w), reinterpret_cast<float4*>(m),
                                               reinterpret_cast<float4*>(v), g, w_out, n, lr, b1, b2, eps, lr * wd,
                                               bc1, bc2);
  return check_launch("adamw_device");
}

template <typename T>
int cast_from_f32(const float* src, T* dst, int64_t n, cudaStream_t st) {
  if (n <= 0) return MOBIUS_OK;
  int64_t blocks = (n / 4 + 255) / 256;
  if (blocks > 148 * 16) blocks = 148 * 16;
  if (blocks < 1) blocks = 1;
  cast_k<T><<<(unsigned)blocks, 256, 0, st>>>(src, dst, n);
  return check_launch("cast");
}

namespace {
__device__ __forceinline__ float gelu_tanh_approx(float u) {  // == gemm_common.cuh gelu_f (same ops)
  const float c = 0.7978845608028654f, ca = 0.7978845608028654f * 0.044715f;
  float t;
  asm("tanh.approx.f32 %0, %1;" : "=f"(t) : "f"(u * fmaf(ca, u * u, c)));
  const float hu = 0.5f * u;
  return fmaf(hu, t, hu);
}
__global__ void gelu_fwd_k(const uint4* __restrict__ u, uint4* __restrict__ g, int64_t n8) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n8; i += (int64_t)gridDim.x * blockDim.x) {
    uint4 x = u[i];
    __nv_bfloat162* h = reinterpret_cast<__nv_bfloat162*>(&x);
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const float2 f = __bfloat1622float2(h[j]);
      h[j] = __floats2bfloat162_rn(gelu_tanh_approx(f.x), gelu_tanh_approx(f.y));
    }
    g[i] = x;
  }
}
}  // namespace

int gelu_fwd_bf16(const __nv_bfloat16* u, __nv_bfloat16* g, int64_t n, cudaStream_t st) {
  if (n <= 0) return MOBIUS_OK;
  if (n % 8 || (reinterpret_cast<uintptr_t>(u) | reinterpret_cast<uintptr_t>(g)) & 15)
    MOBIUS_FAIL(MOBIUS_EINVAL, "gelu_fwd: n %% 8 and 16-byte alignment required");
  const int64_t n8 = n / 8;
  int64_t blocks = (n8 + 255) / 256;
  if (blocks > 148 * 8) blocks = 148 * 8;
  gelu_fwd_k<<<(unsigned)blocks, 256, 0, st>>>(reinterpret_cast<const uint4*>(u), reinterpret_cast<uint4*>(g), n8);
  return check_launch("gelu_fwd");
}

template <typename T>
int fill_ones_col(T* p, int rows, cudaStream_t st) {
  const int64_t n = (int64_t)rows * 64;
  fill_ones_col_k<T><<<(unsigned)std::min<int64_t>(148 * 8, (n + 255) / 256), 256, 0, st>>>(p, n);
  return check_launch("fill_ones_col");
}

int tokens_check_copy(const int32_t* src, int32_t* dst, int64_t n, int V, int* bad_dev, cudaStream_t st) {
  if (cudaMemsetAsync(bad_dev, 0, sizeof(int), st) != cudaSuccess) MOBIUS_FAIL(MOBIUS_ECUDA, "tokens_check: memset");
  const int grid = (int)std::min<int64_t>(148 * 2, (n + 255) / 256);
  tokens_check_k<<<std::max(grid, 1), 256, 0, st>>>(src, dst, n, V, bad_dev);
  return check_launch("tokens_check");
}

int flag_wait(const volatile int* flag, int value, cudaStream_t st) {
  flag_wait_k<<<1, 1, 0, st>>>(flag, value);
  return check_launch("flag_wait");
}
__global__ void ticket_take_k(int* counter, int* out) { *out = atomicAdd_system(counter, 1); }
int ticket_take(int* counter, int* out, cudaStream_t st) {
  ticket_take_k<<<1, 1, 0, st>>>(counter, out);
  return check_launch("ticket_take");
}
int flag_set(int* flag, int value, cudaStream_t st) {
  flag_set_k<<<1, 1, 0, st>>>(flag, value);
  return check_launch("flag_set");
}

#define INST(T)                                                                                                  \
  template int embed_fwd<T>(const int32_t*, const T*, const T*, T*, int, int, int, cudaStream_t);               \
  template int embed_bwd<T>(const int32_t*, const T*, float*, float*, int, int, int, int, cudaStream_t);        \
  template int layernorm_fwd<T>(const T*, const T*, const T*, T*, float*, float*, int, int, cudaStream_t);      \
  template int layernorm_bwd<T>(const T*, const T*, const T*, const float*, const float*, const T*, T*, float*, \
                                float*, int, int, const RedWs&, cudaStream_t, float*);                          \
  template int layernorm_bwd_launches<T>(int, bool, bool);                                                      \
  template int softmax_causal_fwd<T>(const float*, T*, int, int, float, cudaStream_t);                          \
  template int softmax_causal_bwd<T>(const T*, const float*, T*, int, int, float, cudaStream_t);                \
  template int cross_entropy_fwd_bwd<T>(T*, const int32_t*, float*, int, int, int, float, cudaStream_t);        \
  template int colsum_accum<T>(const T*, int64_t, int, int, float*, const RedWs&, cudaStream_t);               \
  template int cast_from_f32<T>(const float*, T*, int64_t, cudaStream_t);                                       \
  template int fill_ones_col<T>(T*, int, cudaStream_t);                                                          \
  template int adamw_device<T>(float*, float*, float*, const T*, T*, int64_t, float, float, float, float, float,   \
                               float, float, cudaStream_t);
INST(float)
INST(__nv_bfloat16)

}  // namespace mobius
