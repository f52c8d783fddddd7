// HBM-bound fused kernels (LayerNorm, causal softmax, cross-entropy,
// embedding, column sums, casts) for sm_100a.  128-bit vectorised,
// coalesced, fp32 math; one CTA (or warp) per row.
#include <cuda_bf16.h>
#include <cuda_runtime.h>

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

template <typename T>
__global__ void embed_bwd_wte_k(const int32_t* tok, const T* dx, float* dwte, int s, int h) {
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
    for (int k = 0; k < V; ++k) atomicAdd(o + c + k, a[k]);
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

constexpr int LNB_ROWS = 16;  // rows per CTA in backward (amortises dg/db atomics)

template <typename T, int LN_NT, int LN_MAXV>
__global__ void __launch_bounds__(LN_NT) ln_bwd_k(const T* dy, const T* x, const T* g, const float* mu,
                                                   const float* rstd, const T* dres, T* dx, float* dg, float* db,
                                                   int rows, int h) {
  constexpr int V = Vec<T>::N;
  __shared__ float red[33];
  float gacc[LN_MAXV][V], bacc[LN_MAXV][V], gv[LN_MAXV][V];
#pragma unroll
  for (int k = 0; k < LN_MAXV; ++k) {
    int c = (threadIdx.x + k * LN_NT) * V;
#pragma unroll
    for (int e = 0; e < V; ++e) gacc[k][e] = bacc[k][e] = 0.f;
    if (c < h) Vec<T>::load(g + c, gv[k]);
  }
  const int r0 = blockIdx.x * LNB_ROWS;
  for (int r = r0; r < min(rows, r0 + LNB_ROWS); ++r) {
    const float m = mu[r], rs = rstd[r];
    float xh[LN_MAXV][V], dyv[LN_MAXV][V];
    float s1 = 0.f, s2 = 0.f;
#pragma unroll
    for (int k = 0; k < LN_MAXV; ++k) {
      int c = (threadIdx.x + k * LN_NT) * V;
      if (c < h) {
        Vec<T>::load(x + (int64_t)r * h + c, xh[k]);
        Vec<T>::load(dy + (int64_t)r * h + c, dyv[k]);
#pragma unroll
        for (int e = 0; e < V; ++e) {
          xh[k][e] = (xh[k][e] - m) * rs;
          float dh = dyv[k][e] * gv[k][e];
          s1 += dh;
          s2 += dh * xh[k][e];
          gacc[k][e] += dyv[k][e] * xh[k][e];
          bacc[k][e] += dyv[k][e];
        }
      }
    }
    const float c1 = block_sum<LN_NT>(s1, red) / h;
    const float c2 = block_sum<LN_NT>(s2, red) / h;
#pragma unroll
    for (int k = 0; k < LN_MAXV; ++k) {
      int c = (threadIdx.x + k * LN_NT) * V;
      if (c < h) {
        float o[V], rr[V];
        if (dres) Vec<T>::load(dres + (int64_t)r * h + c, rr);
#pragma unroll
        for (int e = 0; e < V; ++e) {
          o[e] = rs * (dyv[k][e] * gv[k][e] - c1 - xh[k][e] * c2);
          if (dres) o[e] += rr[e];
        }
        Vec<T>::store(dx + (int64_t)r * h + c, o);
      }
    }
  }
#pragma unroll
  for (int k = 0; k < LN_MAXV; ++k) {
    int c = (threadIdx.x + k * LN_NT) * V;
    if (c < h) {
#pragma unroll
      for (int e = 0; e < V; ++e) {
        atomicAdd(dg + c + e, gacc[k][e]);
        atomicAdd(db + c + e, bacc[k][e]);
      }
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
  float m = -INFINITY, l = 0.f;
  for (int c = threadIdx.x * VW; c < V; c += CE_NT * VW) {
    float f[VW];
    Vec<T>::load(zr + c, f);
#pragma unroll
    for (int e = 0; e < VW; ++e) {
      float nm = fmaxf(m, f[e]);
      l = l * __expf(m - nm) + __expf(f[e] - nm);
      m = nm;
    }
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
template <typename T>
__global__ void colsum_k(const T* X, int64_t ld, int rows, int n, float* out, int rows_per_block) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= n) return;
  const int r0 = blockIdx.y * rows_per_block;
  const int r1 = min(rows, r0 + rows_per_block);
  float acc = 0.f;
  for (int r = r0; r < r1; ++r) acc += to_f(X[(int64_t)r * ld + c]);
  atomicAdd(out + c, acc);
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
int embed_bwd(const int32_t* tok, const T* dx, float* dwte, float* dwpe, int mbs, int s, int h, cudaStream_t st) {
  embed_bwd_wte_k<T><<<mbs * s, 128, 0, st>>>(tok, dx, dwte, s, h);
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

template <typename T>
int layernorm_fwd(const T* x, const T* g, const T* b, T* y, float* mu, float* rstd, int rows, int h, cudaStream_t st) {
  MOBIUS_CHECK_ARG(h % Vec<T>::N == 0, "layernorm: unsupported h=%d", h);
  LN_DISPATCH(ln_fwd_k, rows, x, g, b, y, mu, rstd, h);
  return check_launch("layernorm_fwd");
}
template <typename T>
int layernorm_bwd(const T* dy, const T* x, const T* g, const float* mu, const float* rstd, const T* dres, T* dx,
                  float* dg, float* db, int rows, int h, cudaStream_t st) {
  MOBIUS_CHECK_ARG(h % Vec<T>::N == 0, "layernorm: unsupported h=%d", h);
  LN_DISPATCH(ln_bwd_k, (rows + LNB_ROWS - 1) / LNB_ROWS, dy, x, g, mu, rstd, dres, dx, dg, db, rows, h);
  return check_launch("layernorm_bwd");
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

template <typename T>
int colsum_accum(const T* X, int64_t ld, int rows, int n, float* out, cudaStream_t st) {
  const int rpb = 128;
  dim3 grid((n + 255) / 256, (rows + rpb - 1) / rpb);
  colsum_k<T><<<grid, 256, 0, st>>>(X, ld, rows, n, out, rpb);
  return check_launch("colsum");
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

int flag_wait(const volatile int* flag, int value, cudaStream_t st) {
  flag_wait_k<<<1, 1, 0, st>>>(flag, value);
  return check_launch("flag_wait");
}
int flag_set(int* flag, int value, cudaStream_t st) {
  flag_set_k<<<1, 1, 0, st>>>(flag, value);
  return check_launch("flag_set");
}

#define INST(T)                                                                                                  \
  template int embed_fwd<T>(const int32_t*, const T*, const T*, T*, int, int, int, cudaStream_t);               \
  template int embed_bwd<T>(const int32_t*, const T*, float*, float*, int, int, int, cudaStream_t);             \
  template int layernorm_fwd<T>(const T*, const T*, const T*, T*, float*, float*, int, int, cudaStream_t);      \
  template int layernorm_bwd<T>(const T*, const T*, const T*, const float*, const float*, const T*, T*, float*, \
                                float*, int, int, cudaStream_t);                                                \
  template int softmax_causal_fwd<T>(const float*, T*, int, int, float, cudaStream_t);                          \
  template int softmax_causal_bwd<T>(const T*, const float*, T*, int, int, float, cudaStream_t);                \
  template int cross_entropy_fwd_bwd<T>(T*, const int32_t*, float*, int, int, int, float, cudaStream_t);        \
  template int colsum_accum<T>(const T*, int64_t, int, int, float*, cudaStream_t);                              \
  template int cast_from_f32<T>(const float*, T*, int64_t, cudaStream_t);
INST(float)
INST(__nv_bfloat16)

}  // namespace mobius
