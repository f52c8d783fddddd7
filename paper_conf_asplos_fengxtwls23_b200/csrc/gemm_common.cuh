// Shared pieces of the tcgen05 GEMM kernels (gemm_tc.cu: 1-CTA, batched /
// causal; gemm_tc2.cu: 2-CTA cta_group::2 persistent kernel with a
// Stream-K tail): tile constants, kernel parameters, the fused epilogue and
// the TMA tensor-map encoder.  Included by exactly those two files.
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdlib>
#include <cstring>
#include <mutex>

#include "common.h"
#include "gemm.h"
#include "ptx.cuh"

namespace mobius {

namespace gemm_detail {

constexpr int BM = 128;
constexpr int BK = 64;
constexpr int NUM_THREADS = 192;
constexpr int NUM_THREADS2 = 320;  // 2-CTA kernel: producer, MMA, 8 epilogue warps

template <int BN>
struct Cfg {
  static constexpr int STAGES = BN == 256 ? 4 : (BN == 128 ? 6 : 8);
  static constexpr int A_BYTES = BM * BK * 2;
  static constexpr int B_BYTES = BN * BK * 2;
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int TMEM_COLS = 2 * BN;
  static constexpr int SMEM = 1024 /*align slack*/ + STAGES * STAGE_BYTES + 256;
};

struct Params {
  int M, N, K;
  int nb1, nb2;
  int tiles_m, tiles_n, num_kb;
  int causal;
  int epi;
  int c_f32;
  int accumulate;
  float alpha;
  __nv_bfloat16* C;
  int64_t ldc, cbs1, cbs2;
  const __nv_bfloat16* bias;
  const __nv_bfloat16* R;
  int64_t ldr, rbs1, rbs2;
  __nv_bfloat16* AUX;
  int64_t ldx, xbs1, xbs2;
  // Stream-K tail (2-CTA kernel only; sk_tiles == 0 disables): the first
  // sk_tiles tiles' k-blocks are split evenly over all clusters; partial
  // accumulators go to sk_ws, the last-arriving segment reduces them in
  // segment order (deterministic) and runs the fused epilogue.
  // sk_slices > 0 selects the k-aligned variant: the sk_tiles remainder
  // tiles are cut into sk_slices equal k-slices, unit u = (slice u / sk_tiles,
  // tile u % sk_tiles) goes to cluster u % clusters, so all clusters of the
  // Stream-K round stream the same k range of their panels (L2 reuse); the
  // contiguous variant gives each cluster a different k phase.
  int sk_tiles, sk_maxseg, sk_slices;
  int64_t sk_units;
  float* sk_ws;
  int* sk_cnt;
  // ones row (2-CTA kernel, A_MN): the 64-row A box starting at M row
  // ones_m0p1 - 1 is loaded from the ones map (tmX) instead of A (0 = off)
  int ones_m0p1;
  // split-K with reduce-add (2-CTA kernel, EPI_ACCUM + accumulate): the
  // sk_tiles * sk_slices units of the k-aligned schedule cover every tile
  // and each unit reduce-adds its partial straight into C (no workspace).
  int splitk_reduce;
  // 2-CTA kernel: M tiles per rasterisation group (tiles of a group share
  // their B panels in L2); chosen on the host from the shape
  int group_m;
};

__device__ __forceinline__ float tanh_fast(float x) {
  float y;
  asm("tanh.approx.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
// tanh GeLU, 0.5 u (1 + tanh(c (u + a u^3))), in FMA form: u (c + c a u^2)
// then 0.5u + 0.5u t (5 FP32 ops + one MUFU.TANH per element; the epilogue
// of the bias+GeLU forward GEMM evaluates it for every output element)
__device__ __forceinline__ float gelu_f(float u) {
  const float c = 0.7978845608028654f, ca = 0.7978845608028654f * 0.044715f;
  const float t = tanh_fast(u * fmaf(ca, u * u, c));
  const float hu = 0.5f * u;
  return fmaf(hu, t, hu);
}
__device__ __forceinline__ float gelu_grad_f(float u) {
  const float c = 0.7978845608028654f, a = 0.044715f;
  float t = tanh_fast(c * (u + a * u * u * u));
  return 0.5f * (1.f + t) + 0.5f * u * (1.f - t * t) * c * (1.f + 3.f * a * u * u);
}

// tile index -> (b1, b2, mt, nt), grouped along M for L2 reuse of B tiles
__device__ __forceinline__ void decode_tile(const Params& p, int t, int& b1, int& b2, int& mt, int& nt) {
  int per_batch = p.tiles_m * p.tiles_n;
  int b = t / per_batch;
  int r = t - b * per_batch;
  b1 = b / p.nb2;
  b2 = b - b1 * p.nb2;
  constexpr int GROUP = 8;
  int group_span = GROUP * p.tiles_n;
  int g = r / group_span;
  int first_m = g * GROUP;
  int gm = min(GROUP, p.tiles_m - first_m);
  int rr = r - g * group_span;
  mt = first_m + rr % gm;
  nt = rr / gm;
}

template <int BN>
__device__ __forceinline__ bool tile_active(const Params& p, int mt, int nt) {
  if (p.causal == CAUSAL_SKIP_UPPER) return nt * BN <= mt * BM + BM - 1;
  return true;
}

__device__ __forceinline__ void kb_range(const Params& p, int mt, int& kb0, int& kb1) {
  kb0 = 0;
  kb1 = p.num_kb;
  if (p.causal == CAUSAL_K_LT_MEND) {
    int kend = min(p.K, mt * BM + BM);
    kb1 = (kend + BK - 1) / BK;
  } else if (p.causal == CAUSAL_K_GE_M0) {
    kb0 = (mt * BM) / BK;
  }
}

// 8 bf16 (16 bytes) <-> floats
__device__ __forceinline__ void ld_bf16x8(const __nv_bfloat16* g, float* f) {
  const uint4 pk = *reinterpret_cast<const uint4*>(g);
  const __nv_bfloat162* h2 = reinterpret_cast<const __nv_bfloat162*>(&pk);
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    const float2 x = __bfloat1622float2(h2[j]);
    f[2 * j] = x.x;
    f[2 * j + 1] = x.y;
  }
}
__device__ __forceinline__ void st_bf16x8(__nv_bfloat16* g, const float* f) {
  uint4 pk;
  __nv_bfloat162* h2 = reinterpret_cast<__nv_bfloat162*>(&pk);
#pragma unroll
  for (int j = 0; j < 4; ++j) h2[j] = __floats2bfloat162_rn(f[2 * j], f[2 * j + 1]);
  *reinterpret_cast<uint4*>(g) = pk;
}

// Fused epilogue of one W-column chunk (W = 32 or 64) of output row m: v[]
// holds alpha * acc for columns [n0, n0 + W); applies bias / GeLU /
// residual / GeLU' / fp32 accumulate and stores.  A full chunk issues every
// global load it needs (bias, R, old C) before any arithmetic, so a warp has
// W/8 (W/4 for fp32 C) 16-byte loads in flight instead of one dependent
// chain per 8 columns - the epilogue is latency-bound otherwise.  All
// indices are compile-time (nothing spills); a ragged last chunk takes the
// predicated scalar path.
// EPI, the C type and accumulate are compile-time so each variant keeps only
// the registers it needs; epi_vals<W> dispatches on the runtime values.
template <int W, int EPI, bool CF32, bool ACC>
__device__ __forceinline__ void epi_vals_t(const Params& p, float (&v)[W], int m, int b1, int b2, int n0) {
  if (m >= p.M || n0 >= p.N) return;
  const int64_t crow = (int64_t)b1 * p.cbs1 + (int64_t)b2 * p.cbs2 + (int64_t)m * p.ldc;
  constexpr bool has_bias = EPI == EPI_BIAS || EPI == EPI_BIAS_GELU || EPI == EPI_BIAS_RESID;
  constexpr bool has_r = EPI == EPI_BIAS_RESID || EPI == EPI_GELU_BWD;
  constexpr bool accum = EPI == EPI_ACCUM && ACC;
  const __nv_bfloat16* rrow = has_r ? p.R + (int64_t)b1 * p.rbs1 + (int64_t)b2 * p.rbs2 + (int64_t)m * p.ldr + n0 : nullptr;
  // AUX: the pre-activation u (EPI_BIAS_GELU), or, when set for
  // EPI_GELU_BWD, g = gelu(R) - the forward's activation recomputed from the
  // R (= u) values this epilogue reads anyway
  __nv_bfloat16* aux = (EPI == EPI_BIAS_GELU || (EPI == EPI_GELU_BWD && p.AUX))
                           ? p.AUX + (int64_t)b1 * p.xbs1 + (int64_t)b2 * p.xbs2 + (int64_t)m * p.ldx + n0
                           : nullptr;
  if (n0 + W <= p.N) {
    uint4 lb[W / 8], lr[W / 8];
    float4 lc[W / 4];
    if constexpr (has_bias) {
#pragma unroll
      for (int i = 0; i < W / 8; ++i) lb[i] = __ldg(reinterpret_cast<const uint4*>(p.bias + n0) + i);
    }
    if constexpr (has_r) {
#pragma unroll
      for (int i = 0; i < W / 8; ++i) lr[i] = *(reinterpret_cast<const uint4*>(rrow) + i);
    }
    float* cpf = reinterpret_cast<float*>(p.C) + crow + n0;
    if constexpr (accum && CF32) {
#pragma unroll
      for (int i = 0; i < W / 4; ++i) lc[i] = *(reinterpret_cast<const float4*>(cpf) + i);
    }
    if constexpr (has_bias) {
#pragma unroll
      for (int i = 0; i < W / 8; ++i) {
        const __nv_bfloat162* h2 = reinterpret_cast<const __nv_bfloat162*>(&lb[i]);
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const float2 x = __bfloat1622float2(h2[j]);
          v[8 * i + 2 * j] += x.x;
          v[8 * i + 2 * j + 1] += x.y;
        }
      }
    }
    if constexpr (EPI == EPI_BIAS_GELU) {
#pragma unroll
      for (int i = 0; i < W; i += 8) st_bf16x8(aux + i, v + i);
      // GeLU of the bf16-rounded pre-activation (what backward will see)
#pragma unroll
      for (int i = 0; i < W; ++i) v[i] = gelu_f(__bfloat162float(__float2bfloat16_rn(v[i])));
    }
    if constexpr (EPI == EPI_GELU_BWD) {
      if (aux) {
#pragma unroll
        for (int i = 0; i < W / 8; ++i) {
          float gf[8];
          const __nv_bfloat162* h2 = reinterpret_cast<const __nv_bfloat162*>(&lr[i]);
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            const float2 x = __bfloat1622float2(h2[j]);
            gf[2 * j] = gelu_f(x.x);
            gf[2 * j + 1] = gelu_f(x.y);
          }
          st_bf16x8(aux + 8 * i, gf);
        }
      }
    }
    if constexpr (has_r) {
#pragma unroll
      for (int i = 0; i < W / 8; ++i) {
        const __nv_bfloat162* h2 = reinterpret_cast<const __nv_bfloat162*>(&lr[i]);
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const float2 x = __bfloat1622float2(h2[j]);
          if constexpr (EPI == EPI_BIAS_RESID) {
            v[8 * i + 2 * j] += x.x;
            v[8 * i + 2 * j + 1] += x.y;
          } else {
            v[8 * i + 2 * j] *= gelu_grad_f(x.x);
            v[8 * i + 2 * j + 1] *= gelu_grad_f(x.y);
          }
        }
      }
    }
    if constexpr (CF32) {
#pragma unroll
      for (int i = 0; i < W / 4; ++i) {
        float4 o = make_float4(v[4 * i], v[4 * i + 1], v[4 * i + 2], v[4 * i + 3]);
        if constexpr (accum) {
          o.x += lc[i].x;
          o.y += lc[i].y;
          o.z += lc[i].z;
          o.w += lc[i].w;
        }
        *(reinterpret_cast<float4*>(cpf) + i) = o;
      }
    } else {
      __nv_bfloat16* cp = p.C + crow + n0;
#pragma unroll
      for (int i = 0; i < W; i += 8) st_bf16x8(cp + i, v + i);
    }
  } else {
    const int cnt = p.N - n0;
#pragma unroll
    for (int i = 0; i < W; ++i) {
      if (i < cnt) {
        float x = v[i];
        if constexpr (has_bias) x += __bfloat162float(p.bias[n0 + i]);
        if (EPI == EPI_BIAS_GELU) {
          aux[i] = __float2bfloat16_rn(x);
          x = gelu_f(__bfloat162float(__float2bfloat16_rn(x)));
        }
        if (EPI == EPI_BIAS_RESID) x += __bfloat162float(rrow[i]);
        if (EPI == EPI_GELU_BWD) {
          const float u = __bfloat162float(rrow[i]);
          if (aux) aux[i] = __float2bfloat16_rn(gelu_f(u));
          x *= gelu_grad_f(u);
        }
        if constexpr (CF32) {
          float* cp = reinterpret_cast<float*>(p.C) + crow + n0;
          cp[i] = x + (accum ? cp[i] : 0.f);
        } else {
          p.C[crow + n0 + i] = __float2bfloat16_rn(x);
        }
      }
    }
  }
}

template <int W, int EPI>
__device__ __forceinline__ void epi_vals_c(const Params& p, float (&v)[W], int m, int b1, int b2, int n0) {
  if (p.c_f32)
    epi_vals_t<W, EPI, true, false>(p, v, m, b1, b2, n0);
  else
    epi_vals_t<W, EPI, false, false>(p, v, m, b1, b2, n0);
}
template <int W>
__device__ __forceinline__ void epi_vals(const Params& p, float (&v)[W], int m, int b1, int b2, int n0) {
  switch (p.epi) {
    case EPI_BIAS: epi_vals_c<W, EPI_BIAS>(p, v, m, b1, b2, n0); break;
    case EPI_BIAS_GELU: epi_vals_c<W, EPI_BIAS_GELU>(p, v, m, b1, b2, n0); break;
    case EPI_BIAS_RESID: epi_vals_c<W, EPI_BIAS_RESID>(p, v, m, b1, b2, n0); break;
    case EPI_GELU_BWD: epi_vals_c<W, EPI_GELU_BWD>(p, v, m, b1, b2, n0); break;
    case EPI_ACCUM:
      if (p.accumulate && p.c_f32)
        epi_vals_t<W, EPI_ACCUM, true, true>(p, v, m, b1, b2, n0);
      else
        epi_vals_c<W, EPI_STORE>(p, v, m, b1, b2, n0);
      break;
    default: epi_vals_c<W, EPI_STORE>(p, v, m, b1, b2, n0);
  }
}

// Epilogue of one accumulator tile row-slice (1-CTA kernel): this thread
// owns output row m (TMEM lane), columns [nt*BN, nt*BN + BN); TMEM ->
// registers -> epi_vals.  tmem_row = tmem base + lane quadrant + accumulator
// column base.
template <int BN>
__device__ __forceinline__ void epi_tile(const Params& p, uint32_t tmem_row, int m, int b1, int b2, int nt) {
#pragma unroll 1
  for (int c = 0; c < BN; c += 32) {
    uint32_t r[32];
    __syncwarp();
    ptx::tmem_ld32(tmem_row + c, r);
    ptx::tmem_ld_wait();
    float v[32];
#pragma unroll
    for (int i = 0; i < 32; ++i) v[i] = __uint_as_float(r[i]) * p.alpha;
    epi_vals<32>(p, v, m, b1, b2, nt * BN + c);
  }
}


// TMA map over a bf16 MatView (gemm_tc.cu)
int make_map(CUtensorMap* map, const MatView& v, int64_t inner, int64_t outer, int nb1, int nb2, int box_outer);
// plain 2-D (as 4-D) row-major map [outer][inner] with row stride ld
// elements, bf16 or fp32, box {box_inner, box_outer}, SWIZZLE_128B
int make_map_2d(CUtensorMap* map, const void* ptr, bool f32, int64_t ld, int64_t inner, int64_t outer, int box_inner,
                int box_outer);

}  // namespace gemm_detail
}  // namespace mobius
