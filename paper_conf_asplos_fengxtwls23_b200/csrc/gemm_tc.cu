// Persistent warp-specialised tcgen05 GEMM for sm_100a (bf16 in, fp32
// accumulate in TMEM), TMA 128B-swizzled operand tiles, mbarrier rings.
//
//   warp 0      : TMA producer (one elected lane)
//   warp 1      : TMEM allocator + MMA issuer (one elected lane)
//   warps 2..5  : epilogue, TMEM -> registers -> fused bias / GeLU /
//                 residual / GeLU' / fp32 accumulate -> global
//
// Tile 128 x BN x 64, BN in {64, 128, 256}; two TMEM accumulators so the
// epilogue of tile i overlaps the mainloop of tile i+1.  Operands may be
// K-major or MN-major (UMMA descriptor major bits), so forward (X W),
// dX (dY W^T) and dW (X^T dY) read the same stored tensors without
// transposes.  Used for every dense contraction of the block, attention
// (batched over (batch, head) via 4-D tensor maps) and the LM head.
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdlib>
#include <cstring>
#include <mutex>

#include "common.h"
#include "gemm.h"
#include "ptx.cuh"

namespace mobius {

namespace {

constexpr int BM = 128;
constexpr int BK = 64;
constexpr int NUM_THREADS = 192;

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
  int sk_tiles, sk_maxseg;
  int64_t sk_units;
  float* sk_ws;
  int* sk_cnt;
};

__device__ __forceinline__ float tanh_fast(float x) {
  float y;
  asm("tanh.approx.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
__device__ __forceinline__ float gelu_f(float u) {
  const float c = 0.7978845608028654f, a = 0.044715f;
  float t = tanh_fast(c * (u + a * u * u * u));
  return 0.5f * u * (1.f + t);
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

// Fused epilogue of one 32-column chunk of output row m: v[] holds
// alpha * acc for columns [n0, n0 + 32); applies bias / GeLU / residual /
// GeLU' / fp32 accumulate and stores.  Full chunks use 16-byte vector
// accesses only (all indices compile-time, nothing spills); a ragged last
// chunk takes the predicated scalar path.
__device__ __forceinline__ void epi_vals(const Params& p, float (&v)[32], int m, int b1, int b2, int n0) {
  if (m >= p.M || n0 >= p.N) return;
  const int64_t crow = (int64_t)b1 * p.cbs1 + (int64_t)b2 * p.cbs2 + (int64_t)m * p.ldc;
  const bool has_bias = p.epi == EPI_BIAS || p.epi == EPI_BIAS_GELU || p.epi == EPI_BIAS_RESID;
  const bool has_r = p.epi == EPI_BIAS_RESID || p.epi == EPI_GELU_BWD;
  const bool accum = p.epi == EPI_ACCUM && p.accumulate;
  const __nv_bfloat16* rrow = has_r ? p.R + (int64_t)b1 * p.rbs1 + (int64_t)b2 * p.rbs2 + (int64_t)m * p.ldr + n0 : nullptr;
  __nv_bfloat16* aux = p.epi == EPI_BIAS_GELU
                           ? p.AUX + (int64_t)b1 * p.xbs1 + (int64_t)b2 * p.xbs2 + (int64_t)m * p.ldx + n0
                           : nullptr;
  if (n0 + 32 <= p.N) {
    if (has_bias) {
#pragma unroll
      for (int i = 0; i < 32; i += 8) {
        float bb[8];
        ld_bf16x8(p.bias + n0 + i, bb);
#pragma unroll
        for (int j = 0; j < 8; ++j) v[i + j] += bb[j];
      }
    }
    if (p.epi == EPI_BIAS_GELU) {
#pragma unroll
      for (int i = 0; i < 32; i += 8) st_bf16x8(aux + i, v + i);
      // GeLU of the bf16-rounded pre-activation (what backward will see)
#pragma unroll
      for (int i = 0; i < 32; ++i) v[i] = gelu_f(__bfloat162float(__float2bfloat16_rn(v[i])));
    }
    if (has_r) {
#pragma unroll
      for (int i = 0; i < 32; i += 8) {
        float rv[8];
        ld_bf16x8(rrow + i, rv);
        if (p.epi == EPI_BIAS_RESID) {
#pragma unroll
          for (int j = 0; j < 8; ++j) v[i + j] += rv[j];
        } else {
#pragma unroll
          for (int j = 0; j < 8; ++j) v[i + j] *= gelu_grad_f(rv[j]);
        }
      }
    }
    if (p.c_f32) {
      float* cp = reinterpret_cast<float*>(p.C) + crow + n0;
#pragma unroll
      for (int i = 0; i < 32; i += 4) {
        float4 o = make_float4(v[i], v[i + 1], v[i + 2], v[i + 3]);
        if (accum) {
          const float4 old = *reinterpret_cast<const float4*>(cp + i);
          o.x += old.x;
          o.y += old.y;
          o.z += old.z;
          o.w += old.w;
        }
        *reinterpret_cast<float4*>(cp + i) = o;
      }
    } else {
      __nv_bfloat16* cp = p.C + crow + n0;
#pragma unroll
      for (int i = 0; i < 32; i += 8) st_bf16x8(cp + i, v + i);
    }
  } else {
    const int cnt = p.N - n0;
#pragma unroll
    for (int i = 0; i < 32; ++i) {
      if (i < cnt) {
        float x = v[i];
        if (has_bias) x += __bfloat162float(p.bias[n0 + i]);
        if (p.epi == EPI_BIAS_GELU) {
          aux[i] = __float2bfloat16_rn(x);
          x = gelu_f(__bfloat162float(__float2bfloat16_rn(x)));
        }
        if (p.epi == EPI_BIAS_RESID) x += __bfloat162float(rrow[i]);
        if (p.epi == EPI_GELU_BWD) x *= gelu_grad_f(__bfloat162float(rrow[i]));
        if (p.c_f32) {
          float* cp = reinterpret_cast<float*>(p.C) + crow + n0;
          cp[i] = x + (accum ? cp[i] : 0.f);
        } else {
          p.C[crow + n0 + i] = __float2bfloat16_rn(x);
        }
      }
    }
  }
}

// Epilogue of one accumulator tile row-slice: this thread owns output row m
// (TMEM lane), columns [nt*BN, nt*BN + BN); TMEM -> registers -> epi_vals.
// tmem_row = tmem base + lane quadrant + accumulator column base.
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
    epi_vals(p, v, m, b1, b2, nt * BN + c);
  }
}

template <int BN, bool A_MN, bool B_MN>
__global__ void __launch_bounds__(NUM_THREADS, 1)
    gemm_tc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB, const Params p) {
  using C = Cfg<BN>;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* smA = smem;
  uint8_t* smB = smem + C::STAGES * C::A_BYTES;
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + C::STAGES * C::STAGE_BYTES);
  uint64_t* empty = full + C::STAGES;
  uint64_t* tfull = empty + C::STAGES;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);

  const int warp = threadIdx.x / 32;
  const int lane = threadIdx.x % 32;

  if (warp == 0 && lane == 0) {
    ptx::tma_prefetch_desc(&tmA);
    ptx::tma_prefetch_desc(&tmB);
    for (int s = 0; s < C::STAGES; ++s) {
      ptx::mbar_init(&full[s], 1);
      ptx::mbar_init(&empty[s], 1);
    }
    for (int a = 0; a < 2; ++a) {
      ptx::mbar_init(&tfull[a], 1);
      ptx::mbar_init(&tempty[a], 4);
    }
    ptx::fence_mbar_init();
  }
  if (warp == 1) ptx::tmem_alloc<C::TMEM_COLS>(tmem_slot);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  const int total = p.nb1 * p.nb2 * p.tiles_m * p.tiles_n;

  if (warp == 0) {
    // ===================== TMA producer =====================
    if (lane == 0) {
      int stage = 0;
      uint32_t phase = 0;
      for (int t = blockIdx.x; t < total; t += gridDim.x) {
        int b1, b2, mt, nt;
        decode_tile(p, t, b1, b2, mt, nt);
        if (!tile_active<BN>(p, mt, nt)) continue;
        int kb0, kb1;
        kb_range(p, mt, kb0, kb1);
        const int m0 = mt * BM, n0 = nt * BN;
        for (int kb = kb0; kb < kb1; ++kb) {
          ptx::mbar_wait(&empty[stage], phase ^ 1);
          ptx::mbar_arrive_expect_tx(&full[stage], C::STAGE_BYTES);
          uint8_t* a = smA + stage * C::A_BYTES;
          uint8_t* b = smB + stage * C::B_BYTES;
          const int k0 = kb * BK;
          if (A_MN) {
#pragma unroll
            for (int i = 0; i < BM / 64; ++i) ptx::tma_load_4d(a + i * 8192, &tmA, &full[stage], m0 + 64 * i, k0, b2, b1);
          } else {
            ptx::tma_load_4d(a, &tmA, &full[stage], k0, m0, b2, b1);
          }
          if (B_MN) {
#pragma unroll
            for (int i = 0; i < BN / 64; ++i) ptx::tma_load_4d(b + i * 8192, &tmB, &full[stage], n0 + 64 * i, k0, b2, b1);
          } else {
            ptx::tma_load_4d(b, &tmB, &full[stage], k0, n0, b2, b1);
          }
          if (++stage == C::STAGES) {
            stage = 0;
            phase ^= 1;
          }
        }
      }
    }
  } else if (warp == 1) {
    // ===================== MMA issuer (lane 0) =====================
    if (lane == 0) {
      constexpr uint32_t IDESC = ptx::idesc_bf16(BM, BN, A_MN ? 1 : 0, B_MN ? 1 : 0);
      int stage = 0;
      uint32_t phase = 0;
      int acc = 0;
      uint32_t aphase = 0;
      for (int t = blockIdx.x; t < total; t += gridDim.x) {
        int b1, b2, mt, nt;
        decode_tile(p, t, b1, b2, mt, nt);
        if (!tile_active<BN>(p, mt, nt)) continue;
        int kb0, kb1;
        kb_range(p, mt, kb0, kb1);
        ptx::mbar_wait(&tempty[acc], aphase ^ 1);
        ptx::tc_fence_after();
        const uint32_t tmem_d = tmem_base + acc * BN;
        for (int kb = kb0; kb < kb1; ++kb) {
          ptx::mbar_wait(&full[stage], phase);
          ptx::tc_fence_after();
          const uint32_t a_base = ptx::smem_u32(smA + stage * C::A_BYTES);
          const uint32_t b_base = ptx::smem_u32(smB + stage * C::B_BYTES);
#pragma unroll
          for (int k = 0; k < BK / 16; ++k) {
            uint64_t ad = A_MN ? ptx::sdesc_sw128(a_base + k * 2048, 8192, 1024)
                               : ptx::sdesc_sw128(a_base + k * 32, 16, 1024);
            uint64_t bd = B_MN ? ptx::sdesc_sw128(b_base + k * 2048, 8192, 1024)
                               : ptx::sdesc_sw128(b_base + k * 32, 16, 1024);
            ptx::mma_bf16(tmem_d, ad, bd, IDESC, (kb > kb0 || k > 0) ? 1u : 0u);
          }
          ptx::mma_commit(&empty[stage]);  // frees the smem slot when these MMAs complete
          if (++stage == C::STAGES) {
            stage = 0;
            phase ^= 1;
          }
        }
        ptx::mma_commit(&tfull[acc]);      // accumulator ready for the epilogue
        if (++acc == 2) {
          acc = 0;
          aphase ^= 1;
        }
      }
    }
  } else {
    // ===================== epilogue (warps 2..5) =====================
    const int q = warp & 3;  // TMEM lane quadrant accessible to this warp
    int acc = 0;
    uint32_t aphase = 0;
    for (int t = blockIdx.x; t < total; t += gridDim.x) {
      int b1, b2, mt, nt;
      decode_tile(p, t, b1, b2, mt, nt);
      if (!tile_active<BN>(p, mt, nt)) continue;
      ptx::mbar_wait(&tfull[acc], aphase);
      ptx::tc_fence_after();
      epi_tile<BN>(p, tmem_base + ((uint32_t)(q * 32) << 16) + acc * BN, mt * BM + q * 32 + lane, b1, b2, nt);
      ptx::tc_fence_before();
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive(&tempty[acc]);
      if (++acc == 2) {
        acc = 0;
        aphase ^= 1;
      }
    }
  }

  __syncthreads();
  if (warp == 1) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc<C::TMEM_COLS>(tmem_base);
  }
}


// ======================================================================
// 2-CTA variant (cta_group::2): a cluster of two CTAs on the two SMs of a
// TPC computes a 256 x BN tile; each CTA loads its 128 rows of A and half of
// B (BN/2 rows) into its own smem, the leader CTA issues
// tcgen05.mma.cta_group::2 (M = 256) and multicasts the commits, each CTA's
// epilogue drains its own 128 TMEM lanes.  Halves per-SM operand traffic.
// Used for plain (non-batched, non-causal) GEMMs with N >= 256.
template <int BN>
struct Cfg2 {
  static constexpr int A_BYTES = 128 * BK * 2;
  static constexpr int B_BYTES = (BN / 2) * BK * 2;
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int STAGES = (200 * 1024) / STAGE_BYTES > 8 ? 8 : (200 * 1024) / STAGE_BYTES;
  static constexpr int TMEM_COLS = 2 * BN;
  static constexpr int SMEM = 1024 + STAGES * STAGE_BYTES + 256;
};

// One unit of work of a cluster: k-blocks [k0, k1) of tile t, which is
// segment seg of nseg (nseg == 1: a whole tile, no fixup).
struct Work {
  int t, k0, k1, seg, nseg;
};

__device__ __forceinline__ int64_t sk_start(const Params& p, int c, int ncl) {
  return (int64_t)c * p.sk_units / ncl;
}
// cluster whose Stream-K range holds unit g
__device__ __forceinline__ int sk_owner(const Params& p, int64_t g, int ncl) {
  int c = (int)(g * ncl / p.sk_units);
  while (c + 1 < ncl && sk_start(p, c + 1, ncl) <= g) ++c;
  while (c > 0 && sk_start(p, c, ncl) > g) --c;
  return c;
}

// Per-cluster schedule: its Stream-K range over the first sk_tiles tiles
// (cut at tile boundaries), then whole tiles sk_tiles + cl, + ncl, ...
// The producer, MMA issuer and epilogue walk identical sequences.
struct Sched {
  int64_t g, gend;
  int t, cl, ncl;
  __device__ __forceinline__ Sched(const Params& p, int cl_, int ncl_) : cl(cl_), ncl(ncl_) {
    g = p.sk_tiles ? sk_start(p, cl, ncl) : 0;
    gend = p.sk_tiles ? sk_start(p, cl + 1, ncl) : 0;
    t = p.sk_tiles + cl;
  }
  __device__ __forceinline__ bool next(const Params& p, int total, Work& w) {
    if (g < gend) {
      const int nkb = p.num_kb;
      const int tt = (int)(g / nkb);
      w.t = tt;
      w.k0 = (int)(g - (int64_t)tt * nkb);
      w.k1 = (int)min((int64_t)nkb, (int64_t)w.k0 + (gend - g));
      const int first = sk_owner(p, (int64_t)tt * nkb, ncl);
      const int last = sk_owner(p, (int64_t)(tt + 1) * nkb - 1, ncl);
      w.seg = cl - first;
      w.nseg = last - first + 1;
      g += w.k1 - w.k0;
      return true;
    }
    if (t < total) {
      w.t = t;
      w.k0 = 0;
      w.k1 = p.num_kb;
      w.seg = 0;
      w.nseg = 1;
      t += ncl;
      return true;
    }
    return false;
  }
};

// NP pairs per cluster (cluster = 2*NP CTAs along x).  Pairs of one cluster
// compute horizontally adjacent 256 x BN tiles (same rows): with NP = 2 the
// A tile is loaded once per cluster - each CTA loads half of its 128 A rows
// and TMA-multicasts them to its counterpart in the other pair - cutting the
// L2 -> SM operand traffic by a quarter.
template <int BN, bool A_MN, bool B_MN, int NP>
__global__ void __launch_bounds__(NUM_THREADS, 1)
    gemm_tc2_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB, const Params p) {
  using C = Cfg2<BN>;
  constexpr int BM2 = 256;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* smA = smem;
  uint8_t* smB = smem + C::STAGES * C::A_BYTES;
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + C::STAGES * C::STAGE_BYTES);
  uint64_t* empty = full + C::STAGES;
  uint64_t* tfull = empty + C::STAGES;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);

  const int warp = threadIdx.x / 32;
  const int lane = threadIdx.x % 32;
  const uint32_t rank = ptx::cluster_ctarank();
  const uint32_t pair = rank >> 1, r2 = rank & 1;
  const bool leader = r2 == 0;  // MMA-issuing CTA of this pair
  const int cl = blockIdx.x / (2 * NP), ncl = gridDim.x / (2 * NP);
  const int tiles_n2 = (p.tiles_n + NP - 1) / NP;  // column groups of NP tiles

  if (warp == 0 && lane == 0) {
    ptx::tma_prefetch_desc(&tmA);
    ptx::tma_prefetch_desc(&tmB);
    for (int s = 0; s < C::STAGES; ++s) {
      ptx::mbar_init(&full[s], 1);
      ptx::mbar_init(&empty[s], NP);  // one commit per pair that reads this CTA's slot
    }
    for (int a = 0; a < 2; ++a) {
      ptx::mbar_init(&tfull[a], 1);
      ptx::mbar_init(&tempty[a], 8);  // 4 epilogue warps x 2 CTAs of the pair (leader's copy)
    }
    ptx::fence_mbar_init();
  }
  if (warp == 1) ptx::tmem_alloc_2sm<C::TMEM_COLS>(tmem_slot);
  ptx::tc_fence_before();
  ptx::cluster_sync();
  ptx::tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  const int total = p.tiles_m * tiles_n2;

  auto tile_of = [&](int t, int& mt, int& nt) {  // grouped along M for L2 reuse
    constexpr int GROUP = 8;
    const int span = GROUP * tiles_n2;
    const int g = t / span, first_m = g * GROUP;
    const int gm = min(GROUP, p.tiles_m - first_m);
    const int rr = t - g * span;
    mt = first_m + rr % gm;
    nt = (rr / gm) * NP + (int)pair;
  };

  if (warp == 0) {
    if (lane == 0) {  // TMA producer (every CTA)
      int stage = 0;
      uint32_t phase = 0;
      const uint16_t amask = (uint16_t)((1u << r2) | (NP == 2 ? (1u << (r2 + 2)) : 0u));
      Sched sc(p, cl, ncl);
      Work w;
      while (sc.next(p, total, w)) {
        int mt, nt;
        tile_of(w.t, mt, nt);
        const int m0 = mt * BM2 + (int)r2 * 128, n0 = nt * BN + (int)r2 * (BN / 2);
        for (int kb = w.k0; kb < w.k1; ++kb) {
          ptx::mbar_wait_cluster(&empty[stage], phase ^ 1);
          if (leader) ptx::mbar_arrive_expect_tx(&full[stage], 2 * C::STAGE_BYTES);
          uint8_t* a = smA + stage * C::A_BYTES;
          uint8_t* b = smB + stage * C::B_BYTES;
          const int k0 = kb * BK;
          if (NP == 1) {
            if (A_MN) {
#pragma unroll
              for (int i = 0; i < 2; ++i) ptx::tma_load_4d_2sm(a + i * 8192, &tmA, &full[stage], m0 + 64 * i, k0, 0, 0);
            } else {
              ptx::tma_load_4d_2sm(a, &tmA, &full[stage], k0, m0, 0, 0);
            }
          } else {  // this pair loads half h = pair of the 128 A rows and multicasts it
            const int h = (int)pair;
            if (A_MN)
              ptx::tma_load_4d_2sm_mc(a + h * 8192, &tmA, &full[stage], amask, m0 + 64 * h, k0, 0, 0);
            else
              ptx::tma_load_4d_2sm_mc(a + h * 8192, &tmA, &full[stage], amask, k0, m0 + 64 * h, 0, 0);
          }
          if (B_MN) {
#pragma unroll
            for (int i = 0; i < BN / 128; ++i)
              ptx::tma_load_4d_2sm(b + i * 8192, &tmB, &full[stage], n0 + 64 * i, k0, 0, 0);
          } else {
            ptx::tma_load_4d_2sm(b, &tmB, &full[stage], k0, n0, 0, 0);
          }
          if (++stage == C::STAGES) {
            stage = 0;
            phase ^= 1;
          }
        }
      }
    }
  } else if (warp == 1) {
    if (leader && lane == 0) {  // MMA issuer (pair leader)
      constexpr uint32_t IDESC = ptx::idesc_bf16(BM2, BN, A_MN ? 1 : 0, B_MN ? 1 : 0);
      const uint16_t all_mask = (uint16_t)((1u << (2 * NP)) - 1);
      const uint16_t pair_mask = (uint16_t)(3u << (2 * pair));
      int stage = 0;
      uint32_t phase = 0;
      int acc = 0;
      uint32_t aphase = 0;
      Sched sc(p, cl, ncl);
      Work w;
      while (sc.next(p, total, w)) {
        ptx::mbar_wait_cluster(&tempty[acc], aphase ^ 1);
        ptx::tc_fence_after();
        const uint32_t tmem_d = tmem_base + acc * BN;
        for (int kb = w.k0; kb < w.k1; ++kb) {
          ptx::mbar_wait_cluster(&full[stage], phase);
          ptx::tc_fence_after();
          const uint32_t a_base = ptx::smem_u32(smA + stage * C::A_BYTES);
          const uint32_t b_base = ptx::smem_u32(smB + stage * C::B_BYTES);
#pragma unroll
          for (int k = 0; k < BK / 16; ++k) {
            uint64_t ad = A_MN ? ptx::sdesc_sw128(a_base + k * 2048, 8192, 1024)
                               : ptx::sdesc_sw128(a_base + k * 32, 16, 1024);
            uint64_t bd = B_MN ? ptx::sdesc_sw128(b_base + k * 2048, 8192, 1024)
                               : ptx::sdesc_sw128(b_base + k * 32, 16, 1024);
            ptx::mma_bf16_2sm(tmem_d, ad, bd, IDESC, (kb > w.k0 || k > 0) ? 1u : 0u);
          }
          // the slot may be refilled by this pair's producers and (A halves)
          // by the other pair's: free it in every CTA of the cluster
          ptx::mma_commit_2sm(&empty[stage], all_mask);
          if (++stage == C::STAGES) {
            stage = 0;
            phase ^= 1;
          }
        }
        ptx::mma_commit_2sm(&tfull[acc], pair_mask);  // accumulator ready in both CTAs of the pair
        if (++acc == 2) {
          acc = 0;
          aphase ^= 1;
        }
      }
    }
  } else {
    // epilogue (warps 2..5): rows mt*256 + r2*128 + lane quadrant
    const int q = warp & 3;
    const uint32_t tempty_leader = ptx::mapa_shared(ptx::smem_u32(&tempty[0]), pair * 2);
    int acc = 0;
    uint32_t aphase = 0;
    Sched sc(p, cl, ncl);
    Work w;
    while (sc.next(p, total, w)) {
      int mt, nt;
      tile_of(w.t, mt, nt);
      const int m = mt * BM2 + (int)r2 * 128 + q * 32 + lane;
      const uint32_t tmem_row = tmem_base + ((uint32_t)(q * 32) << 16) + acc * BN;
      ptx::mbar_wait_cluster(&tfull[acc], aphase);
      ptx::tc_fence_after();
      if (w.nseg == 1) {
        epi_tile<BN>(p, tmem_row, m, 0, 0, nt);
        ptx::tc_fence_before();
        __syncwarp();
        if (lane == 0) ptx::mbar_arrive_cluster(tempty_leader + acc * 8);
      } else {
        // Stream-K segment: raw partial (32 rows x BN fp32 per warp) to the
        // workspace, lane-interleaved so every store is 512 contiguous bytes
        const int wq = (int)r2 * 4 + q;
        constexpr int SLOT = 32 * BN;  // floats per warp slot
        float* base = p.sk_ws + ((int64_t)w.t * p.sk_maxseg * 8 + wq) * SLOT;
        const int64_t seg_stride = 8 * (int64_t)SLOT;
        float4* mine = reinterpret_cast<float4*>(base + w.seg * seg_stride) + lane;
#pragma unroll 1
        for (int c = 0; c < BN; c += 32) {
          uint32_t r[32];
          __syncwarp();
          ptx::tmem_ld32(tmem_row + c, r);
          ptx::tmem_ld_wait();
#pragma unroll
          for (int i = 0; i < 8; ++i)
            __stcg(mine + ((c / 32) * 8 + i) * 32, make_float4(__uint_as_float(r[4 * i]), __uint_as_float(r[4 * i + 1]),
                                                              __uint_as_float(r[4 * i + 2]), __uint_as_float(r[4 * i + 3])));
        }
        ptx::tc_fence_before();
        __syncwarp();
        if (lane == 0) ptx::mbar_arrive_cluster(tempty_leader + acc * 8);  // accumulator free: MMA runs on
        __threadfence();
        __syncwarp();
        int old = 0;
        int* cnt = p.sk_cnt + (int64_t)w.t * 8 + wq;
        if (lane == 0) old = atomicAdd(cnt, 1);
        old = __shfl_sync(0xffffffffu, old, 0);
        if (old == w.nseg - 1) {  // last segment to arrive: reduce in segment order
          __threadfence();
#pragma unroll 1
          for (int c = 0; c < BN; c += 32) {
            float v[32];
#pragma unroll
            for (int i = 0; i < 32; ++i) v[i] = 0.f;
#pragma unroll 1
            for (int sgi = 0; sgi < w.nseg; ++sgi) {
              const float4* src = reinterpret_cast<const float4*>(base + sgi * seg_stride) + lane;
#pragma unroll
              for (int i = 0; i < 8; ++i) {
                const float4 x = __ldcg(src + ((c / 32) * 8 + i) * 32);
                v[4 * i] += x.x;
                v[4 * i + 1] += x.y;
                v[4 * i + 2] += x.z;
                v[4 * i + 3] += x.w;
              }
            }
#pragma unroll
            for (int i = 0; i < 32; ++i) v[i] *= p.alpha;
            epi_vals(p, v, m, 0, 0, nt * BN + c);
          }
          if (lane == 0) *cnt = 0;  // self-cleaning for the next launch
        }
      }
      if (++acc == 2) {
        acc = 0;
        aphase ^= 1;
      }
    }
  }

  __syncthreads();
  ptx::cluster_sync();
  if (warp == 1) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc_2sm<C::TMEM_COLS>(tmem_base);
  }
}

// ------------------------------------------------------------ host side
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

EncodeTiledFn get_encode() {
  static EncodeTiledFn fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<EncodeTiledFn>(p);
  });
  return fn;
}

// 4-D map {inner, outer, nb2, nb1} over a bf16 MatView; box {64, box_outer, 1, 1}
int make_map(CUtensorMap* map, const MatView& v, int64_t inner, int64_t outer, int nb1, int nb2, int box_outer) {
  EncodeTiledFn enc = get_encode();
  if (!enc) MOBIUS_FAIL(MOBIUS_ECUDA, "cuTensorMapEncodeTiled unavailable");
  if ((reinterpret_cast<uintptr_t>(v.ptr) & 15) != 0) MOBIUS_FAIL(MOBIUS_EINVAL, "TMA base not 16B aligned");
  int64_t s1 = v.ld * 2;
  int64_t s2 = nb2 > 1 ? v.bs2 * 2 : s1 * outer;
  int64_t s3 = nb1 > 1 ? v.bs1 * 2 : s2 * nb2;
  if (s1 % 16 || s2 % 16 || s3 % 16) MOBIUS_FAIL(MOBIUS_EINVAL, "TMA strides must be multiples of 16 bytes");
  cuuint64_t dims[4] = {(cuuint64_t)inner, (cuuint64_t)outer, (cuuint64_t)nb2, (cuuint64_t)nb1};
  cuuint64_t strides[3] = {(cuuint64_t)s1, (cuuint64_t)s2, (cuuint64_t)s3};
  cuuint32_t box[4] = {64, (cuuint32_t)box_outer, 1, 1};
  cuuint32_t estr[4] = {1, 1, 1, 1};
  CUresult r = enc(map, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, const_cast<void*>(v.ptr), dims, strides, box, estr,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) MOBIUS_FAIL(MOBIUS_ECUDA, "cuTensorMapEncodeTiled failed (%d)", (int)r);
  return MOBIUS_OK;
}

template <int BN, bool A_MN, bool B_MN>
int launch(const CUtensorMap& ta, const CUtensorMap& tb, const Params& p, int total, cudaStream_t s) {
  auto k = gemm_tc_kernel<BN, A_MN, B_MN>;
  static bool attr_set = false;  // per instantiation
  if (!attr_set) {
    if (cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg<BN>::SMEM) != cudaSuccess)
      MOBIUS_FAIL(MOBIUS_ECUDA, "cudaFuncSetAttribute(smem) failed");
    attr_set = true;
  }
  int grid = total < num_sms() ? total : num_sms();
  if (grid < 1) grid = 1;
  k<<<grid, NUM_THREADS, Cfg<BN>::SMEM, s>>>(ta, tb, p);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) MOBIUS_FAIL(MOBIUS_ECUDA, "gemm_tc launch: %s", cudaGetErrorString(e));
  return MOBIUS_OK;
}

template <int BN>
int dispatch_major(bool amn, bool bmn, const CUtensorMap& ta, const CUtensorMap& tb, const Params& p, int total,
                   cudaStream_t s) {
  if (!amn && !bmn) return launch<BN, false, false>(ta, tb, p, total, s);
  if (!amn && bmn) return launch<BN, false, true>(ta, tb, p, total, s);
  if (amn && !bmn) return launch<BN, true, false>(ta, tb, p, total, s);
  return launch<BN, true, true>(ta, tb, p, total, s);
}

template <int BN, bool A_MN, bool B_MN, int NP>
int launch2(const CUtensorMap& ta, const CUtensorMap& tb, const Params& p, cudaStream_t s) {
  auto k = gemm_tc2_kernel<BN, A_MN, B_MN, NP>;
  static bool attr_set = false;
  if (!attr_set) {
    if (cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg2<BN>::SMEM) != cudaSuccess)
      MOBIUS_FAIL(MOBIUS_ECUDA, "cudaFuncSetAttribute(smem, 2cta) failed");
    attr_set = true;
  }
  const int total = p.tiles_m * ((p.tiles_n + NP - 1) / NP);
  int clusters = num_sms() / (2 * NP);
  if (total < clusters && p.sk_tiles == 0) clusters = total;  // Stream-K needs every cluster
  if (clusters < 1) clusters = 1;
  cudaLaunchConfig_t cfg;
  std::memset(&cfg, 0, sizeof(cfg));
  cfg.gridDim = dim3(2 * NP * clusters);
  cfg.blockDim = dim3(NUM_THREADS);
  cfg.dynamicSmemBytes = Cfg2<BN>::SMEM;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = 2 * NP;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  cudaError_t e = cudaLaunchKernelEx(&cfg, k, ta, tb, p);
  if (e != cudaSuccess) MOBIUS_FAIL(MOBIUS_ECUDA, "gemm_tc2 launch: %s", cudaGetErrorString(e));
  return MOBIUS_OK;
}

}  // namespace

int num_sms() {
  static int n = 0;
  if (!n) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    if (n <= 0) n = 148;
  }
  return n;
}

// pairs per cluster for the 2-CTA kernel (MOBIUS_GEMM_NP=2 enables the A
// multicast across two pairs; measured slower on the 1.5B shapes - the pairs
// run in lock-step on every smem slot - so it is off by default)
static int g_gemm_np = -1;
static int g_gemm_sk = -1;  // Stream-K tail: env MOBIUS_GEMM_SK=0 disables

// Stream-K workspace, one per stream (GEMMs on different streams may run
// concurrently).  Grows on demand; counters start at zero and are reset by
// the reducing warp, so consecutive launches on one stream reuse them.
struct SkWs {
  cudaStream_t s;
  float* ws;
  size_t ws_bytes;
  int* cnt;
  size_t cnt_n;
};
static std::mutex g_sk_mu;
static SkWs g_sk[16];
static int g_sk_n = 0;

static int sk_workspace(cudaStream_t s, size_t ws_bytes, size_t cnt_n, float** ws, int** cnt) {
  std::lock_guard<std::mutex> lk(g_sk_mu);
  SkWs* e = nullptr;
  for (int i = 0; i < g_sk_n; ++i)
    if (g_sk[i].s == s) e = &g_sk[i];
  if (!e) {
    if (g_sk_n == 16) MOBIUS_FAIL(MOBIUS_ENOMEM, "gemm: too many streams for Stream-K workspaces");
    e = &g_sk[g_sk_n++];
    std::memset(e, 0, sizeof(*e));
    e->s = s;
  }
  if (e->ws_bytes < ws_bytes) {
    if (e->ws) {
      cudaStreamSynchronize(s);
      cudaFree(e->ws);
    }
    e->ws = nullptr;
    e->ws_bytes = 0;
    if (cudaMalloc(&e->ws, ws_bytes) != cudaSuccess) MOBIUS_FAIL(MOBIUS_ENOMEM, "gemm: Stream-K workspace");
    e->ws_bytes = ws_bytes;
  }
  if (e->cnt_n < cnt_n) {
    if (e->cnt) {
      cudaStreamSynchronize(s);
      cudaFree(e->cnt);
    }
    e->cnt = nullptr;
    e->cnt_n = 0;
    if (cudaMalloc(&e->cnt, cnt_n * sizeof(int)) != cudaSuccess) MOBIUS_FAIL(MOBIUS_ENOMEM, "gemm: Stream-K counters");
    if (cudaMemset(e->cnt, 0, cnt_n * sizeof(int)) != cudaSuccess) MOBIUS_FAIL(MOBIUS_ECUDA, "gemm: counter memset");
    e->cnt_n = cnt_n;
  }
  *ws = e->ws;
  *cnt = e->cnt;
  return MOBIUS_OK;
}

// host copy of the device owner function (same integer arithmetic)
static int sk_owner_h(int64_t units, int64_t g, int ncl) {
  auto start = [&](int c) { return (int64_t)c * units / ncl; };
  int c = (int)(g * ncl / units);
  while (c + 1 < ncl && start(c + 1) <= g) ++c;
  while (c > 0 && start(c) > g) --c;
  return c;
}

// Wave quantisation: T tiles over P clusters take ceil(T/P) tile-times.
// Stream-K keeps floor(T/P)-1 whole waves and spreads the remaining tiles'
// k-blocks evenly (cost ~ T/P + fixup); used when that saves >= 5% of a
// wave and every cluster gets a reasonable k-range.
static void plan_stream_k(Params& p, int P) {
  p.sk_tiles = 0;
  p.sk_units = 0;
  p.sk_maxseg = 0;
  if (g_gemm_sk < 0) {
    const char* e = getenv("MOBIUS_GEMM_SK");
    g_gemm_sk = (e && e[0] == '0') ? 0 : 1;
  }
  if (!g_gemm_sk) return;
  const int T = p.tiles_m * p.tiles_n, nkb = p.num_kb;
  if (T % P == 0) return;
  const int waves = (T + P - 1) / P;
  const int dp_waves = T / P >= 1 ? T / P - 1 : 0;
  const int sk_tiles = T - dp_waves * P;
  const double cost = dp_waves + (double)sk_tiles / P + 0.25;
  if (cost > waves - 0.05) return;
  const int64_t units = (int64_t)sk_tiles * nkb;
  const int64_t per = units / P;
  if (per < 4 || per * 4 < nkb) return;
  int maxseg = 1;
  for (int t = 0; t < sk_tiles; ++t) {
    const int n = sk_owner_h(units, (int64_t)(t + 1) * nkb - 1, P) - sk_owner_h(units, (int64_t)t * nkb, P) + 1;
    if (n > maxseg) maxseg = n;
  }
  p.sk_tiles = sk_tiles;
  p.sk_units = units;
  p.sk_maxseg = maxseg;
}

template <int BN>
static int gemm_bf16_2cta_bn(const GemmDesc& d, cudaStream_t s) {
  if (g_gemm_np < 0) {
    const char* e = getenv("MOBIUS_GEMM_NP");
    g_gemm_np = (e && e[0] == '2') ? 2 : 1;
  }
  const bool mc = g_gemm_np == 2 && (d.N + BN - 1) / BN >= 2;
  CUtensorMap ta, tb;
  int rc;
  if (d.a_mn)
    rc = make_map(&ta, d.A, d.M, d.K, d.nb1, d.nb2, BK);
  else
    rc = make_map(&ta, d.A, d.K, d.M, d.nb1, d.nb2, mc ? 64 : 128);
  if (rc) return rc;
  if (d.b_mn)
    rc = make_map(&tb, d.B, d.N, d.K, d.nb1, d.nb2, BK);
  else
    rc = make_map(&tb, d.B, d.K, d.N, d.nb1, d.nb2, BN / 2);
  if (rc) return rc;
  Params p;
  std::memset(&p, 0, sizeof(p));
  p.M = d.M; p.N = d.N; p.K = d.K; p.nb1 = 1; p.nb2 = 1;
  p.tiles_m = (d.M + 255) / 256;
  p.tiles_n = (d.N + BN - 1) / BN;
  p.num_kb = (d.K + BK - 1) / BK;
  p.causal = CAUSAL_NONE;
  p.epi = d.epi; p.c_f32 = d.c_f32 ? 1 : 0; p.accumulate = d.accumulate ? 1 : 0; p.alpha = d.alpha;
  p.C = (__nv_bfloat16*)d.C.ptr; p.ldc = d.C.ld;
  p.bias = (const __nv_bfloat16*)d.bias;
  p.R = (const __nv_bfloat16*)d.R.ptr; p.ldr = d.R.ld;
  p.AUX = (__nv_bfloat16*)d.AUX.ptr; p.ldx = d.AUX.ld;
  if (g_gemm_np != 2) {
    plan_stream_k(p, num_sms() / 2);
    if (p.sk_tiles) {
      const size_t ws = (size_t)p.sk_tiles * p.sk_maxseg * 8 * 32 * BN * sizeof(float);
      int rc2 = sk_workspace(s, ws, (size_t)p.sk_tiles * 8, &p.sk_ws, &p.sk_cnt);
      if (rc2) return rc2;
    }
  }
  if (g_gemm_np == 2 && p.tiles_n >= 2) {  // A multicast across two pairs
    if (!d.a_mn && !d.b_mn) return launch2<BN, false, false, 2>(ta, tb, p, s);
    if (!d.a_mn && d.b_mn) return launch2<BN, false, true, 2>(ta, tb, p, s);
    if (d.a_mn && !d.b_mn) return launch2<BN, true, false, 2>(ta, tb, p, s);
    return launch2<BN, true, true, 2>(ta, tb, p, s);
  }
  if (!d.a_mn && !d.b_mn) return launch2<BN, false, false, 1>(ta, tb, p, s);
  if (!d.a_mn && d.b_mn) return launch2<BN, false, true, 1>(ta, tb, p, s);
  if (d.a_mn && !d.b_mn) return launch2<BN, true, false, 1>(ta, tb, p, s);
  return launch2<BN, true, true, 1>(ta, tb, p, s);
}

// 256 x 256 tiles: at 64 B/clk/SM of operand traffic this is the only 2-CTA
// shape that stays under the L2->SM feed rate (256 x 128 measured slower even
// where it quantises better over the 74 SM pairs)
static int gemm_bf16_2cta(const GemmDesc& d, cudaStream_t s) { return gemm_bf16_2cta_bn<256>(d, s); }

static int g_gemm_mode = -1;  // -1 auto (env MOBIUS_GEMM_2CTA, default on), 0 off, 1 on

void gemm_set_config(int two_cta, int stream_k) {
  g_gemm_mode = two_cta;
  g_gemm_sk = stream_k;
}

int gemm_bf16(const GemmDesc& d, cudaStream_t s) {
  if (g_gemm_mode < 0) {
    const char* e = getenv("MOBIUS_GEMM_2CTA");
    g_gemm_mode = (e && e[0] == '0') ? 0 : 1;
  }
  if (g_gemm_mode == 1 && d.causal == CAUSAL_NONE && d.nb1 == 1 && d.nb2 == 1 && d.N >= 256 && d.M >= 256 &&
      d.K >= 64)
    return gemm_bf16_2cta(d, s);
  MOBIUS_CHECK_ARG(d.M > 0 && d.N > 0 && d.K > 0, "gemm: empty shape %d x %d x %d", d.M, d.N, d.K);
  MOBIUS_CHECK_ARG(d.N % 8 == 0 || !true, "gemm: N must be a multiple of 8");
  int BN = d.N >= 256 ? 256 : (d.N > 64 ? 128 : 64);
  if (d.N > 128 && d.N < 256) BN = 128;
  CUtensorMap ta, tb;
  int rc;
  if (d.a_mn)
    rc = make_map(&ta, d.A, d.M, d.K, d.nb1, d.nb2, BK);
  else
    rc = make_map(&ta, d.A, d.K, d.M, d.nb1, d.nb2, BM);
  if (rc) return rc;
  if (d.b_mn)
    rc = make_map(&tb, d.B, d.N, d.K, d.nb1, d.nb2, BK);
  else
    rc = make_map(&tb, d.B, d.K, d.N, d.nb1, d.nb2, BN);
  if (rc) return rc;
  Params p;
  std::memset(&p, 0, sizeof(p));
  p.M = d.M;
  p.N = d.N;
  p.K = d.K;
  p.nb1 = d.nb1;
  p.nb2 = d.nb2;
  p.tiles_m = (d.M + BM - 1) / BM;
  p.tiles_n = (d.N + BN - 1) / BN;
  p.num_kb = (d.K + BK - 1) / BK;
  p.causal = d.causal;
  p.epi = d.epi;
  p.c_f32 = d.c_f32 ? 1 : 0;
  p.accumulate = d.accumulate ? 1 : 0;
  p.alpha = d.alpha;
  p.C = (__nv_bfloat16*)d.C.ptr;
  p.ldc = d.C.ld;
  p.cbs1 = d.C.bs1;
  p.cbs2 = d.C.bs2;
  p.bias = (const __nv_bfloat16*)d.bias;
  p.R = (const __nv_bfloat16*)d.R.ptr;
  p.ldr = d.R.ld;
  p.rbs1 = d.R.bs1;
  p.rbs2 = d.R.bs2;
  p.AUX = (__nv_bfloat16*)d.AUX.ptr;
  p.ldx = d.AUX.ld;
  p.xbs1 = d.AUX.bs1;
  p.xbs2 = d.AUX.bs2;
  int total = d.nb1 * d.nb2 * p.tiles_m * p.tiles_n;
  if (BN == 256) return dispatch_major<256>(d.a_mn, d.b_mn, ta, tb, p, total, s);
  if (BN == 128) return dispatch_major<128>(d.a_mn, d.b_mn, ta, tb, p, total, s);
  return dispatch_major<64>(d.a_mn, d.b_mn, ta, tb, p, total, s);
}

}  // namespace mobius
