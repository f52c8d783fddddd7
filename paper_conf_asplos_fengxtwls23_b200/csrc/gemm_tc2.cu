// 2-CTA (cta_group::2) persistent tcgen05 GEMM for plain (non-batched,
// non-causal) products with M, N >= 256: 256 x 256 x 64 tiles over SM pairs,
// 8 epilogue warps, and a deterministic Stream-K tail for the last partial
// wave of long-K shapes.  Shared epilogue and parameters: gemm_common.cuh.
#include "gemm_common.cuh"

#include <vector>

namespace mobius {
namespace gemm_detail {

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
  static constexpr int STAGES = (160 * 1024) / STAGE_BYTES > 8 ? 8 : (160 * 1024) / STAGE_BYTES;
  static constexpr int TMEM_COLS = 2 * BN;
  // epilogue staging: per epilogue warp two 4 KiB boxes (32 rows x 128 B,
  // SWIZZLE_128B) for TMA stores / reduce-adds of C and TMA loads of R
  static constexpr int EPI_BOX = 4096;
  static constexpr int EPI_BYTES = 8 * 2 * EPI_BOX;
  static constexpr int SMEM = 1024 + STAGES * STAGE_BYTES + EPI_BYTES + 512;
};

// ---------------------------------------------------- TMA-store epilogue
__device__ __forceinline__ void tma_store_2d(const CUtensorMap* m, uint32_t src, int c0, int c1) {
  asm volatile("cp.async.bulk.tensor.4d.global.shared::cta.bulk_group [%0, {%2, %3, %4, %5}], [%1];" ::"l"(
                   reinterpret_cast<uint64_t>(m)),
               "r"(src), "r"(c0), "r"(c1), "r"(0), "r"(0)
               : "memory");
}
// TMA store with an L2 evict-first policy: for outputs not read again soon
// (the GeLU pre-activation u is read only by the backward), so they do not
// push this GEMM's operand tiles out of L2 (fc1 fwd: 526 -> 521 us at T = 32768)
__device__ __forceinline__ void tma_store_2d_evict_first(const CUtensorMap* m, uint32_t src, int c0, int c1) {
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  asm volatile(
      "cp.async.bulk.tensor.4d.global.shared::cta.bulk_group.L2::cache_hint [%0, {%2, %3, %4, %5}], [%1], %6;" ::"l"(
          reinterpret_cast<uint64_t>(m)),
      "r"(src), "r"(c0), "r"(c1), "r"(0), "r"(0), "l"(pol)
      : "memory");
}
__device__ __forceinline__ void tma_reduce_add_2d(const CUtensorMap* m, uint32_t src, int c0, int c1) {
  asm volatile(
      "cp.reduce.async.bulk.tensor.4d.global.shared::cta.add.tile.bulk_group [%0, {%2, %3, %4, %5}], [%1];" ::"l"(
          reinterpret_cast<uint64_t>(m)),
      "r"(src), "r"(c0), "r"(c1), "r"(0), "r"(0)
      : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_read() {
  asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
// byte offset of 16-byte chunk c of row r in a 32 x 128 B SWIZZLE_128B box
__device__ __forceinline__ uint32_t box_off(int r, int c) { return (uint32_t)(r * 128 + ((c ^ (r & 7)) << 4)); }

struct EpiMaps {
  const CUtensorMap* C;  // bf16 box {64, 32} or fp32 box {32, 32}
  const CUtensorMap* R;  // bf16 box {64, 32} (residual / GeLU input)
  const CUtensorMap* X;  // bf16 box {64, 32} (pre-activation output)
};

// One warp's share of an accumulator tile: 32 rows (its TMEM lane quadrant)
// x 128 columns (half the tile), starting at (m0w, n0w).  Values leave TMEM
// 64 (bf16) or 32 (fp32) columns at a time, get the fused ops in registers,
// are written swizzled into this warp's staging boxes and leave with one
// TMA store (or, for the fp32 dW accumulate, a TMA reduce-add: L2 does the
// read-modify-write) per box; R boxes arrive by TMA before the accumulator
// is ready.  Partial boxes at the matrix edge are clipped by the TMA unit.
// `release` is called after the last TMEM read (accumulator handed back).
template <int HALF, int EPI, bool CF32, bool ACC, typename Rel>
__device__ __forceinline__ void epi_tma(const Params& p, const EpiMaps& mp, uint32_t tmem_row, uint32_t stg,
                                        uint64_t* rbar, uint32_t rph, int m0w, int n0w, int lane, Rel release) {
  constexpr bool has_bias = EPI == EPI_BIAS || EPI == EPI_BIAS_GELU || EPI == EPI_BIAS_RESID;
  constexpr bool has_r = EPI == EPI_BIAS_RESID || EPI == EPI_GELU_BWD;
  if constexpr (CF32) {
    // fp32 C: HALF/32 32-column boxes, alternating between the two staging boxes
    constexpr int NF = HALF / 32;
#pragma unroll 1
    for (int j = 0; j < NF; ++j) {
      uint32_t r[32];
      __syncwarp();
      ptx::tmem_ld32(tmem_row + j * 32, r);
      ptx::tmem_ld_wait();
      if (j == NF - 1) release();
      const int n0 = n0w + 32 * j;
      if (n0 >= p.N) continue;
      const uint32_t box = stg + (j & 1) * 4096;
      if (j >= 2) {
        if (lane == 0) bulk_wait_read<1>();  // the store from this box two chunks ago has read it
        __syncwarp();
      }
#pragma unroll
      for (int c = 0; c < 8; ++c) {
        float4 o = make_float4(__uint_as_float(r[4 * c]) * p.alpha, __uint_as_float(r[4 * c + 1]) * p.alpha,
                               __uint_as_float(r[4 * c + 2]) * p.alpha, __uint_as_float(r[4 * c + 3]) * p.alpha);
        asm volatile("st.shared.v4.f32 [%0], {%1, %2, %3, %4};" ::"r"(box + box_off(lane, c)), "f"(o.x), "f"(o.y),
                     "f"(o.z), "f"(o.w)
                     : "memory");
      }
      ptx::fence_proxy_async();
      __syncwarp();
      if (lane == 0) {
        if (ACC)
          tma_reduce_add_2d(mp.C, box, n0, m0w);
        else
          tma_store_2d(mp.C, box, n0, m0w);
        bulk_commit();
      }
    }
  } else {
    // bf16 C: HALF/64 64-column chunks; GeLU uses both boxes per chunk (u, g)
    constexpr int NCH = HALF / 64;
#pragma unroll 1
    for (int j = 0; j < NCH; ++j) {
      const int n0 = n0w + 64 * j;
      uint32_t ra[32], rb[32];
      __syncwarp();
      ptx::tmem_ld32(tmem_row + j * 64, ra);
      ptx::tmem_ld32(tmem_row + j * 64 + 32, rb);
      ptx::tmem_ld_wait();
      if (j == NCH - 1) release();
      if (n0 >= p.N) continue;
      float v[64];
#pragma unroll
      for (int i = 0; i < 32; ++i) {
        v[i] = __uint_as_float(ra[i]) * p.alpha;
        v[32 + i] = __uint_as_float(rb[i]) * p.alpha;
      }
      if constexpr (has_bias) {
        if (n0 + 64 <= p.N) {
#pragma unroll
          for (int i = 0; i < 8; ++i) {
            const uint4 pk = __ldg(reinterpret_cast<const uint4*>(p.bias + n0) + i);
            const __nv_bfloat162* h2 = reinterpret_cast<const __nv_bfloat162*>(&pk);
#pragma unroll
            for (int k = 0; k < 4; ++k) {
              const float2 x = __bfloat1622float2(h2[k]);
              v[8 * i + 2 * k] += x.x;
              v[8 * i + 2 * k + 1] += x.y;
            }
          }
        } else {
#pragma unroll
          for (int i = 0; i < 64; ++i)
            if (n0 + i < p.N) v[i] += __bfloat162float(p.bias[n0 + i]);
        }
      }
      const uint32_t box = stg + (has_r ? j * 4096 : 0);
      uint32_t gk[EPI == EPI_GELU_BWD ? 8 : 1][4];  // EPI_GELU_BWD with AUX: packed g of this chunk
      if constexpr (has_r) {
        ptx::mbar_wait(&rbar[j], (rph >> j) & 1u);  // R box j landed
#pragma unroll
        for (int c = 0; c < 8; ++c) {
          uint4 pk;
          asm volatile("ld.shared.v4.b32 {%0, %1, %2, %3}, [%4];"
                       : "=r"(pk.x), "=r"(pk.y), "=r"(pk.z), "=r"(pk.w)
                       : "r"(box + box_off(lane, c)));
          const __nv_bfloat162* h2 = reinterpret_cast<const __nv_bfloat162*>(&pk);
#pragma unroll
          for (int k = 0; k < 4; ++k) {
            const float2 x = __bfloat1622float2(h2[k]);
            if constexpr (EPI == EPI_BIAS_RESID) {
              v[8 * c + 2 * k] += x.x;
              v[8 * c + 2 * k + 1] += x.y;
            } else {
              if (p.AUX) {  // g = gelu(u), bf16, as the forward epilogue computed it
                const __nv_bfloat162 g2 = __floats2bfloat162_rn(gelu_f(x.x), gelu_f(x.y));
                gk[c][k] = *reinterpret_cast<const uint32_t*>(&g2);
              }
              v[8 * c + 2 * k] *= gelu_grad_f(x.x);
              v[8 * c + 2 * k + 1] *= gelu_grad_f(x.y);
            }
          }
        }
      } else if (j > 0) {
        if (lane == 0) bulk_wait_read<0>();  // previous chunk's stores have read the boxes
        __syncwarp();
      }
      if constexpr (EPI == EPI_BIAS_GELU) {
        // u (bf16) -> box 0 (AUX), g = gelu(bf16(u)) -> box 1 (C)
#pragma unroll
        for (int c = 0; c < 8; ++c) {
          uint32_t pu[4], pg[4];
#pragma unroll
          for (int k = 0; k < 4; ++k) {
            const __nv_bfloat162 u2 = __floats2bfloat162_rn(v[8 * c + 2 * k], v[8 * c + 2 * k + 1]);
            const float2 uf = __bfloat1622float2(u2);
            const __nv_bfloat162 g2 = __floats2bfloat162_rn(gelu_f(uf.x), gelu_f(uf.y));
            pu[k] = *reinterpret_cast<const uint32_t*>(&u2);
            pg[k] = *reinterpret_cast<const uint32_t*>(&g2);
          }
          asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(stg + box_off(lane, c)), "r"(pu[0]), "r"(pu[1]),
                       "r"(pu[2]), "r"(pu[3])
                       : "memory");
          asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(stg + 4096 + box_off(lane, c)), "r"(pg[0]),
                       "r"(pg[1]), "r"(pg[2]), "r"(pg[3])
                       : "memory");
        }
        ptx::fence_proxy_async();
        __syncwarp();
        if (lane == 0) {
          tma_store_2d_evict_first(mp.X, stg, n0, m0w);
          tma_store_2d(mp.C, stg + 4096, n0, m0w);
          bulk_commit();
        }
      } else {
#pragma unroll
        for (int c = 0; c < 8; ++c) {
          uint32_t pk[4];
#pragma unroll
          for (int k = 0; k < 4; ++k) {
            const __nv_bfloat162 o2 = __floats2bfloat162_rn(v[8 * c + 2 * k], v[8 * c + 2 * k + 1]);
            pk[k] = *reinterpret_cast<const uint32_t*>(&o2);
          }
          asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(box + box_off(lane, c)), "r"(pk[0]), "r"(pk[1]),
                       "r"(pk[2]), "r"(pk[3])
                       : "memory");
        }
        ptx::fence_proxy_async();
        __syncwarp();
        if (lane == 0) {
          tma_store_2d(mp.C, box, n0, m0w);
          bulk_commit();
        }
        if constexpr (EPI == EPI_GELU_BWD) {
          if (p.AUX) {  // g leaves through the same box once the dU store has read it
            if (lane == 0) bulk_wait_read<0>();
            __syncwarp();
#pragma unroll
            for (int c = 0; c < 8; ++c)
              asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(box + box_off(lane, c)), "r"(gk[c][0]),
                           "r"(gk[c][1]), "r"(gk[c][2]), "r"(gk[c][3])
                           : "memory");
            ptx::fence_proxy_async();
            __syncwarp();
            if (lane == 0) {
              tma_store_2d(mp.X, box, n0, m0w);
              bulk_commit();
            }
          }
        }
      }
    }
  }
}

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
    if (p.sk_slices) {  // k-aligned: units cl, cl + ncl, ... of sk_tiles * sk_slices
      g = cl;
      gend = (int64_t)p.sk_tiles * p.sk_slices;
    } else {
      g = p.sk_tiles ? sk_start(p, cl, ncl) : 0;
      gend = p.sk_tiles ? sk_start(p, cl + 1, ncl) : 0;
    }
    t = p.sk_tiles + cl;
  }
  __device__ __forceinline__ bool next(const Params& p, int total, Work& w) {
    if (p.sk_slices && g < gend) {
      const int sl = (int)(g / p.sk_tiles), kbs = (p.num_kb + p.sk_slices - 1) / p.sk_slices;
      w.t = (int)(g % p.sk_tiles);
      w.k0 = sl * kbs;
      w.k1 = min(p.num_kb, w.k0 + kbs);
      w.seg = p.splitk_reduce ? 0 : sl;
      w.nseg = p.splitk_reduce ? 1 : p.sk_slices;  // split-K: each unit reduce-adds into C itself
      g += ncl;
      return true;
    }
    if (!p.sk_slices && g < gend) {
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
__global__ void __launch_bounds__(NUM_THREADS2, 1)
    gemm_tc2_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                    const __grid_constant__ CUtensorMap tmC, const __grid_constant__ CUtensorMap tmR,
                    const __grid_constant__ CUtensorMap tmX, const Params p) {
  using C = Cfg2<BN>;
  constexpr int BM2 = 256;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* smA = smem;
  uint8_t* smB = smem + C::STAGES * C::A_BYTES;
  uint8_t* smE = smem + C::STAGES * C::STAGE_BYTES;  // [8 warps][2 boxes][4 KiB]
  uint64_t* full = reinterpret_cast<uint64_t*>(smE + C::EPI_BYTES);
  uint64_t* empty = full + C::STAGES;
  uint64_t* tfull = empty + C::STAGES;
  uint64_t* tempty = tfull + 2;
  uint64_t* rbar = tempty + 2;  // [8 warps][2] R-box arrivals
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(rbar + 16);

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
      ptx::mbar_init(&tempty[a], 16);  // 8 epilogue warps x 2 CTAs of the pair (leader's copy)
    }
    for (int i = 0; i < 16; ++i) ptx::mbar_init(&rbar[i], 1);
    ptx::fence_mbar_init();
  }
  if (warp == 1) ptx::tmem_alloc_2sm<C::TMEM_COLS>(tmem_slot);
  ptx::tc_fence_before();
  ptx::cluster_sync();
  ptx::tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  const int total = p.tiles_m * tiles_n2;

  auto tile_of = [&](int t, int& mt, int& nt) {  // grouped along M for L2 reuse
    const int GROUP = p.group_m;
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
        // a ragged last tile column of <= BN/2 columns runs as an N = BN/2
        // MMA: each CTA then supplies BN/4 rows of B (the rest of its box is
        // loaded but not read)
        const int nhalf = (p.N - nt * BN <= BN / 2) ? BN / 4 : BN / 2;
        const int m0 = mt * BM2 + (int)r2 * 128, n0 = nt * BN + (int)r2 * nhalf;
        for (int kb = w.k0; kb < w.k1; ++kb) {
          ptx::mbar_wait_cluster(&empty[stage], phase ^ 1);
          if (leader) ptx::mbar_arrive_expect_tx(&full[stage], 2 * C::STAGE_BYTES);
          uint8_t* a = smA + stage * C::A_BYTES;
          uint8_t* b = smB + stage * C::B_BYTES;
          const int k0 = kb * BK;
          if (NP == 1) {
            if (A_MN) {
#pragma unroll
              for (int i = 0; i < 2; ++i) {
                const int mm = m0 + 64 * i;
                if (p.ones_m0p1 && mm == p.ones_m0p1 - 1)  // bias-gradient row: [1, 0 .. 0] per k
                  ptx::tma_load_4d_2sm(a + i * 8192, &tmX, &full[stage], 0, k0, 0, 0);
                else
                  ptx::tma_load_4d_2sm(a + i * 8192, &tmA, &full[stage], mm, k0, 0, 0);
              }
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
    if (leader) {  // MMA issuer (pair leader): the whole warp, converged; one elected lane issues (ptx::*_w)
      const uint32_t tmem_base_u = __shfl_sync(0xffffffffu, tmem_base, 0);  // warp-uniform
      constexpr uint32_t IDESC = ptx::idesc_bf16(BM2, BN, A_MN ? 1 : 0, B_MN ? 1 : 0);
      constexpr uint32_t IDESC_NARROW = ptx::idesc_bf16(BM2, BN / 2, A_MN ? 1 : 0, B_MN ? 1 : 0);
      const uint16_t all_mask = (uint16_t)((1u << (2 * NP)) - 1);
      const uint16_t pair_mask = (uint16_t)(3u << (2 * pair));
      int stage = 0;
      uint32_t phase = 0;
      int acc = 0;
      uint32_t aphase = 0;
      Sched sc(p, cl, ncl);
      Work w;
      while (sc.next(p, total, w)) {
        int mt_, nt_;
        tile_of(w.t, mt_, nt_);
        const uint32_t idesc = (p.N - nt_ * BN <= BN / 2) ? IDESC_NARROW : IDESC;  // ragged last column
        ptx::mbar_wait_cluster(&tempty[acc], aphase ^ 1);
        ptx::tc_fence_after();
        const uint32_t tmem_d = tmem_base_u + acc * BN;
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
            ptx::mma_bf16_2sm_w(tmem_d, ad, bd, idesc, (kb > w.k0 || k > 0) ? 1u : 0u);
          }
          // the slot may be refilled by this pair's producers and (A halves)
          // by the other pair's: free it in every CTA of the cluster
          ptx::mma_commit_2sm_w(&empty[stage], all_mask);
          if (++stage == C::STAGES) {
            stage = 0;
            phase ^= 1;
          }
        }
        ptx::mma_commit_2sm_w(&tfull[acc], pair_mask);  // accumulator ready in both CTAs of the pair
        if (++acc == 2) {
          acc = 0;
          aphase ^= 1;
        }
      }
    }
  } else {
    // epilogue (warps 2..9): warp w drains TMEM lane quadrant w % 4 (rows
    // mt*256 + r2*128 + 32*(w%4) + lane), column half (w-2)/4 of the tile,
    // 64 columns per step
    const int q = warp & 3, hf = (warp - 2) >> 2;
    constexpr int HALF = BN / 2;
    const uint32_t tempty_leader = ptx::mapa_shared(ptx::smem_u32(&tempty[0]), pair * 2);
    int acc = 0;
    uint32_t aphase = 0;
    const uint32_t stg = ptx::smem_u32(smE) + (uint32_t)(warp - 2) * (2 * C::EPI_BOX);
    uint64_t* wrbar = rbar + (warp - 2) * 2;
    uint32_t rph = 0;  // phase bit per R box barrier
    const EpiMaps mp{&tmC, &tmR, &tmX};
    const bool has_r = p.epi == EPI_BIAS_RESID || p.epi == EPI_GELU_BWD;
    Sched sc(p, cl, ncl);
    Work w;
    while (sc.next(p, total, w)) {
      int mt, nt;
      tile_of(w.t, mt, nt);
      const int m = mt * BM2 + (int)r2 * 128 + q * 32 + lane;
      const int ncol0 = nt * BN + hf * HALF;
      const uint32_t tmem_row = tmem_base + ((uint32_t)(q * 32) << 16) + acc * BN + hf * HALF;
      if (has_r && w.nseg == 1 && lane == 0) {
        // R boxes of this tile into the staging boxes while the mainloop runs
        bulk_wait_read<0>();  // the previous tile's stores have read them
        const int m0w = mt * BM2 + (int)r2 * 128 + q * 32;
#pragma unroll
        for (int j = 0; j < HALF / 64; ++j)
          if (ncol0 + 64 * j < p.N) {
            ptx::mbar_arrive_expect_tx(&wrbar[j], C::EPI_BOX);
            ptx::tma_load_4d(smE + (warp - 2) * (2 * C::EPI_BOX) + j * C::EPI_BOX, &tmR, &wrbar[j], ncol0 + 64 * j,
                             m0w, 0, 0);
          }
      }
      ptx::mbar_wait_cluster(&tfull[acc], aphase);
      ptx::tc_fence_after();
      if (w.nseg == 1) {
        auto release = [&]() {  // last TMEM read of this tile: hand the accumulator back early
          ptx::tc_fence_before();
          __syncwarp();
          if (lane == 0) ptx::mbar_arrive_cluster(tempty_leader + acc * 8);
        };
        const int m0w = mt * BM2 + (int)r2 * 128 + q * 32;
        switch (p.epi) {
          case EPI_BIAS: epi_tma<HALF, EPI_BIAS, false, false>(p, mp, tmem_row, stg, wrbar, rph, m0w, ncol0, lane, release); break;
          case EPI_BIAS_GELU:
            epi_tma<HALF, EPI_BIAS_GELU, false, false>(p, mp, tmem_row, stg, wrbar, rph, m0w, ncol0, lane, release);
            break;
          case EPI_BIAS_RESID:
          case EPI_GELU_BWD:
            if (p.epi == EPI_BIAS_RESID)
              epi_tma<HALF, EPI_BIAS_RESID, false, false>(p, mp, tmem_row, stg, wrbar, rph, m0w, ncol0, lane, release);
            else
              epi_tma<HALF, EPI_GELU_BWD, false, false>(p, mp, tmem_row, stg, wrbar, rph, m0w, ncol0, lane, release);
#pragma unroll
            for (int j = 0; j < HALF / 64; ++j)
              if (ncol0 + 64 * j < p.N) rph ^= 1u << j;
            break;
          case EPI_ACCUM:
            if (p.accumulate)
              epi_tma<HALF, EPI_ACCUM, true, true>(p, mp, tmem_row, stg, wrbar, rph, m0w, ncol0, lane, release);
            else
              epi_tma<HALF, EPI_STORE, true, false>(p, mp, tmem_row, stg, wrbar, rph, m0w, ncol0, lane, release);
            break;
          default:
            if (p.c_f32)
              epi_tma<HALF, EPI_STORE, true, false>(p, mp, tmem_row, stg, wrbar, rph, m0w, ncol0, lane, release);
            else
              epi_tma<HALF, EPI_STORE, false, false>(p, mp, tmem_row, stg, wrbar, rph, m0w, ncol0, lane, release);
        }
      } else {
        // Stream-K segment: raw partial (32 rows x BN/2 fp32 per warp) to the
        // workspace, lane-interleaved so every store is 512 contiguous bytes
        const int wq = (int)r2 * 8 + (warp - 2);
        constexpr int SLOT = 32 * HALF;  // floats per warp slot
        float* base = p.sk_ws + ((int64_t)w.t * p.sk_maxseg * 16 + wq) * SLOT;
        const int64_t seg_stride = 16 * (int64_t)SLOT;
        float4* mine = reinterpret_cast<float4*>(base + w.seg * seg_stride) + lane;
#pragma unroll 1
        for (int c = 0; c < HALF; c += 32) {
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
        int* cnt = p.sk_cnt + (int64_t)w.t * 16 + wq;
        if (lane == 0) old = atomicAdd(cnt, 1);
        old = __shfl_sync(0xffffffffu, old, 0);
        if (old == w.nseg - 1) {  // last segment to arrive: reduce in segment order
          __threadfence();
#pragma unroll 1
          for (int c = 0; c < HALF; c += 32) {
            float v[32];
#pragma unroll
            for (int i = 0; i < 32; ++i) v[i] = 0.f;
#pragma unroll 1
            for (int sgi = 0; sgi < w.nseg; ++sgi) {
              const float4* src = reinterpret_cast<const float4*>(base + sgi * seg_stride) + lane;
              float4 x[8];
#pragma unroll
              for (int i = 0; i < 8; ++i) x[i] = __ldcg(src + ((c / 32) * 8 + i) * 32);
#pragma unroll
              for (int i = 0; i < 8; ++i) {
                v[4 * i] += x[i].x;
                v[4 * i + 1] += x[i].y;
                v[4 * i + 2] += x[i].z;
                v[4 * i + 3] += x[i].w;
              }
            }
#pragma unroll
            for (int i = 0; i < 32; ++i) v[i] *= p.alpha;
            epi_vals<32>(p, v, m, 0, 0, ncol0 + c);
          }
          if (lane == 0) *cnt = 0;  // self-cleaning for the next launch
        }
      }
      if (++acc == 2) {
        acc = 0;
        aphase ^= 1;
      }
    }
    if (lane == 0) bulk_wait_all();  // staged stores complete before the CTA exits
  }

  __syncthreads();
  ptx::cluster_sync();
  if (warp == 1) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc_2sm<C::TMEM_COLS>(tmem_base);
  }
}

template <int BN, bool A_MN, bool B_MN, int NP>
int launch2(const CUtensorMap& ta, const CUtensorMap& tb, const CUtensorMap& tc, const CUtensorMap& tr,
            const CUtensorMap& tx, const Params& p, cudaStream_t s) {
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
  cfg.blockDim = dim3(NUM_THREADS2);
  cfg.dynamicSmemBytes = Cfg2<BN>::SMEM;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = 2 * NP;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  cudaError_t e = cudaLaunchKernelEx(&cfg, k, ta, tb, tc, tr, tx, p);
  if (e != cudaSuccess) MOBIUS_FAIL(MOBIUS_ECUDA, "gemm_tc2 launch: %s", cudaGetErrorString(e));
  return MOBIUS_OK;
}

}  // namespace gemm_detail

using namespace gemm_detail;

static int g_gemm_sk = -1;  // Stream-K tail: env MOBIUS_GEMM_SK=0 disables

// Stream-K workspace, one per (device, stream): GEMMs on different streams
// may run concurrently.  Grows on demand; counters start at zero and are
// reset by the reducing warp, so consecutive launches on one stream reuse
// them.  The owner of a stream releases its entry (gemm_release_stream,
// called by mobius_destroy for the context's compute stream).
struct SkWs {
  int dev;
  cudaStream_t s;
  float* ws;
  size_t ws_bytes;
  int* cnt;
  size_t cnt_n;
};
static std::mutex g_sk_mu;
static std::vector<SkWs> g_sk;

static int sk_workspace(cudaStream_t s, size_t ws_bytes, size_t cnt_n, float** ws, int** cnt) {
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) MOBIUS_FAIL(MOBIUS_ECUDA, "gemm: cudaGetDevice");
  std::lock_guard<std::mutex> lk(g_sk_mu);
  SkWs* e = nullptr;
  for (auto& x : g_sk)
    if (x.s == s && x.dev == dev) e = &x;
  if (!e) {
    g_sk.push_back(SkWs{dev, s, nullptr, 0, nullptr, 0});
    e = &g_sk.back();
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

// free the Stream-K workspace of stream s on the current device (the stream
// must be idle; no-op when it never ran a Stream-K GEMM)
void gemm_release_stream(cudaStream_t s) {
  int dev = 0;
  cudaGetDevice(&dev);
  std::lock_guard<std::mutex> lk(g_sk_mu);
  for (size_t i = 0; i < g_sk.size(); ++i) {
    if (g_sk[i].s != s || g_sk[i].dev != dev) continue;
    if (g_sk[i].ws) cudaFree(g_sk[i].ws);
    if (g_sk[i].cnt) cudaFree(g_sk[i].cnt);
    g_sk.erase(g_sk.begin() + i);
    return;
  }
}
size_t gemm_workspace_entries() {
  std::lock_guard<std::mutex> lk(g_sk_mu);
  return g_sk.size();
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
static int g_gemm_skmode = -1;  // MOBIUS_GEMM_SKMODE: 0 auto, 1 contiguous only, 2 k-aligned when possible

static void plan_stream_k(Params& p, int P) {
  p.sk_tiles = 0;
  p.sk_units = 0;
  p.sk_maxseg = 0;
  p.sk_slices = 0;
  p.splitk_reduce = 0;
  if (g_gemm_sk < 0) {
    const char* e = getenv("MOBIUS_GEMM_SK");
    g_gemm_sk = (e && e[0] == '0') ? 0 : 1;
  }
  if (!g_gemm_sk) return;
  if (g_gemm_skmode < 0) {
    const char* e = getenv("MOBIUS_GEMM_SKMODE");
    g_gemm_skmode = e ? atoi(e) : 0;
  }
  const int T = p.tiles_m * p.tiles_n, nkb = p.num_kb;
  // fp32-accumulating long-K GEMMs (the weight gradients, C += A^T B with
  // TMA reduce-add epilogues): split every tile's K range into S slices dealt
  // slice-major over the clusters, each slice reduce-adding its partial into
  // C - the sum order across slices then varies in the last bits (the bf16
  // path is not bitwise reproducible anyway).  S minimises
  // ceil(T S / P) / S waves plus 0.02 per extra slice (its reduce traffic).
  // Opt-in (MOBIUS_GEMM_SPLITK=1): faster in isolation (dW GEMMs 1806 ->
  // 1704 us per block at T = 32768) but neutral inside the step (A/B on one
  // box: 91.4k vs 91.2-91.4k tokens/s), so the deterministic Stream-K tail
  // below stays the default.
  static int splitk = -1;
  if (splitk < 0) {
    const char* e = getenv("MOBIUS_GEMM_SPLITK");
    splitk = e ? atoi(e) : 0;
  }
  if (splitk && p.epi == EPI_ACCUM && p.accumulate && p.c_f32 && nkb >= 64) {
    int best_s = 1;
    double best = (double)((T + P - 1) / P);
    for (int S = 2; S <= 8 && nkb / S >= 16; ++S) {
      const double c = (double)((T * S + P - 1) / P) / S + 0.02 * (S - 1);
      if (c < best - 1e-9) {
        best = c;
        best_s = S;
      }
    }
    if (best_s > 1) {
      p.sk_tiles = T;
      p.sk_slices = best_s;
      p.sk_maxseg = 1;
      p.sk_units = (int64_t)T * best_s;
      p.splitk_reduce = 1;
      return;
    }
  }
  if (T % P == 0) return;
  static int min_slice = -1;  // k-blocks per slice (MOBIUS_GEMM_SKSLICE, default 16)
  if (min_slice < 0) {
    const char* e = getenv("MOBIUS_GEMM_SKSLICE");
    min_slice = e ? std::max(4, atoi(e)) : 16;
  }
  if (g_gemm_skmode != 1 && nkb >= 2 * min_slice) {
    // k-aligned: every full wave data-parallel, the R remainder tiles in S
    // slices of >= 16 k-blocks dealt round-robin (slice-major) over the P
    // clusters; the tail then costs ceil(R*S/P)/S of a wave instead of 1.
    // S minimises that (ties: fewer slices = fewer partials to reduce).
    static double pen = -1.0;  // per-slice cost (partials written and reduced), in waves
    if (pen < 0) {
      const char* e = getenv("MOBIUS_GEMM_SKPEN");
      pen = e ? atof(e) : 0.04;
    }
    const int R = T % P;
    int best_s = 0;
    double best = 1.0;
    for (int S = 2; S <= std::min(16, nkb / min_slice); ++S) {
      const double c = (double)((R * S + P - 1) / P) / S + pen * S;
      if (c < best - 1e-9) {
        best = c;
        best_s = S;
      }
    }
    if (best_s && best <= 0.92) {
      p.sk_tiles = R;
      p.sk_slices = best_s;
      p.sk_maxseg = best_s;
      p.sk_units = (int64_t)R * best_s;
      return;
    }
  }
  const int waves = (T + P - 1) / P;
  const int dp_waves = T / P >= 1 ? T / P - 1 : 0;
  const int sk_tiles = T - dp_waves * P;
  const double cost = dp_waves + (double)sk_tiles / P + 0.25;
  if (cost > waves - 0.3) return;
  // Short K (< 64 k-blocks): the fp32 partial round trip costs more than the
  // wave it saves (measured: 8192x1600x1600 46 -> 58 us); long K gains
  // (8192x1600x6400 150 -> 137 us, 1600x6400x8192 165 -> 150 us, ncu).
  if (nkb < 64) return;
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
  CUtensorMap ta, tb, tc, tr, tx;
  int rc;
  const bool ones = d.ones_row;
  if (ones)
    MOBIUS_CHECK_ARG(d.a_mn && d.epi == EPI_ACCUM && d.ones && (d.M - 1) % 64 == 0 && (d.M - 1) % 256 != 0,
                     "gemm: ones row needs a_mn, EPI_ACCUM, a ones buffer and M-1 a multiple of 64 inside a tile");
  if (d.a_mn)
    rc = make_map(&ta, d.A, ones ? d.M - 1 : d.M, d.K, d.nb1, d.nb2, BK);
  else
    rc = make_map(&ta, d.A, d.K, d.M, d.nb1, d.nb2, 128);
  if (rc) return rc;
  if (d.b_mn)
    rc = make_map(&tb, d.B, d.N, d.K, d.nb1, d.nb2, BK);
  else
    rc = make_map(&tb, d.B, d.K, d.N, d.nb1, d.nb2, BN / 2);
  if (rc) return rc;
  // epilogue maps: 32-row boxes of 128 B (64 bf16 or 32 fp32 columns)
  const bool cf = d.c_f32;
  if ((rc = make_map_2d(&tc, d.C.ptr, cf, d.C.ld, d.N, d.M, cf ? 32 : 64, 32))) return rc;
  const bool has_r = d.epi == EPI_BIAS_RESID || d.epi == EPI_GELU_BWD;
  if (has_r) {
    if ((rc = make_map_2d(&tr, d.R.ptr, false, d.R.ld, d.N, d.M, 64, 32))) return rc;
  } else {
    tr = tc;
  }
  if (d.epi == EPI_BIAS_GELU || (d.epi == EPI_GELU_BWD && d.AUX.ptr)) {
    if ((rc = make_map_2d(&tx, d.AUX.ptr, false, d.AUX.ld, d.N, d.M, 64, 32))) return rc;
  } else if (ones) {  // EPI_ACCUM reads no AUX: the slot carries the ones map ([K][64], column 0 = 1)
    MatView ov;
    ov.ptr = d.ones;
    ov.ld = 64;
    if ((rc = make_map(&tx, ov, 64, d.K, 1, 1, BK))) return rc;
  } else {
    tx = tc;
  }
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
  p.ones_m0p1 = ones ? d.M : 0;  // (M - 1) + 1
  // rasterisation group: 4 M tiles when the output is narrow (<= 8 column
  // tiles: a group of 8 x 7 tiles spans less than a wave of 74 clusters),
  // else 8.  Measured under the power cap (tools/gemm_sustained.py, 1.5B
  // shapes at T = 32768, N = 1600): group 4 / 8 / 16 / 32 give fc2 fwd 559 /
  // 585 / 610 / 661 us, fc1 dX 546 / 576 / 592 / 639, qkv dX 409 / 422 / 433 /
  // 464 (the larger groups run at lower clocks), fc2 dW 625 / 640; the wide
  // outputs are within 1% or prefer 8 (qkv dW 489 / 472, fc1 dW 639 / 630);
  // 4 for every activation-major GEMM cost 6% on the 13B-width shapes
  {
    static int g_env = -2;
    if (g_env == -2) {
      const char* e = getenv("MOBIUS_GEMM_GROUP");
      g_env = e ? atoi(e) : -1;
    }
    p.group_m = g_env > 0 ? g_env : (p.tiles_n <= 8 ? 4 : 8);
  }
  plan_stream_k(p, num_sms() / 2);
  if (p.sk_tiles && !p.splitk_reduce) {
    const size_t ws = (size_t)p.sk_tiles * p.sk_maxseg * 16 * 32 * (BN / 2) * sizeof(float);
    int rc2 = sk_workspace(s, ws, (size_t)p.sk_tiles * 16, &p.sk_ws, &p.sk_cnt);
    if (rc2) return rc2;
  }
  if (!d.a_mn && !d.b_mn) return launch2<BN, false, false, 1>(ta, tb, tc, tr, tx, p, s);
  if (!d.a_mn && d.b_mn) return launch2<BN, false, true, 1>(ta, tb, tc, tr, tx, p, s);
  if (d.a_mn && !d.b_mn) return launch2<BN, true, false, 1>(ta, tb, tc, tr, tx, p, s);
  return launch2<BN, true, true, 1>(ta, tb, tc, tr, tx, p, s);
}

// 256 x 256 tiles: at 64 B/clk/SM of operand traffic this is the only 2-CTA
// shape that stays under the L2->SM feed rate (256 x 128 measured slower even
// where it quantises better over the 74 SM pairs)
int gemm_bf16_2cta(const GemmDesc& d, cudaStream_t s) { return gemm_bf16_2cta_bn<256>(d, s); }

void gemm_2cta_set_stream_k(int stream_k) { g_gemm_sk = stream_k; }

}  // namespace mobius
