// Fused causal attention (flash-style) on tcgen05 for sm_100a (SURVEY
// §8(f) f1; replaces the materialised S / P of K3/K4).
//
// All kernels are persistent (one CTA per SM walking a heaviest-first item
// list in snake order) with warp-specialised roles and mbarrier hand-offs.
// At dh 64 (the 1.5B shape) two 16-warp kernels written for it run by default
// (flash_fwd64_kernel: two query tiles in flight per CTA, per-stream TMA /
// MMA issuers, an epilogue warpgroup; flash_bwd64_kernel: a drain warpgroup
// for dQ / dV / dK, K / V double-buffered, next-item score prefetch - see
// their headers); the generic kernels below serve dh 128 (and dh 64 with
// MOBIUS_FLASH_FWD_V1 / MOBIUS_FLASH_BWD_V1 = 1).
//
// Generic forward, item = (batch, head, 128-query tile):
//   warp 0     TMA producer: Q (double buffered across items), K_j / V_j
//              tiles through a 4-deep ring (dh 64)
//   warp 1     MMA issuer:   S_j = Q K_j^T -> TMEM (double buffered);
//                            O += P_j V_j  -> TMEM (O double buffered across
//                            items; dh 64: P_j from TMEM as a TS-MMA operand)
//   warps 2-9  softmax:      (lane quadrant x column half) per S row; online
//                            max / sum in the log2 domain, lazy O rescale,
//                            P_j (bf16) -> TMEM (dh 64) or smem (dh 128); the
//                            O / l read-out of an item is deferred until the
//                            next item's first P tile is issued and leaves
//                            through smem + TMA stores (dh 64); writes lse.
// Generic backward, item = (batch, head, 128-key tile kt), query tiles i >= kt:
//   S^T = K Q_i^T, dP^T = V dO_i^T (TMEM); thread = key row computes
//   P^T = 2^(S^T*c - lse_q) (-> TMEM, dh 64) and dS^T = P^T (dP^T - D_q)
//   (-> smem); then dV += P^T dO_i, dK += dS^T Q_i (TMEM accumulators),
//   dQ_i = dS K_j (TMEM, drained one tile behind by TMA reduce-add into an
//   fp32 buffer); the 1/sqrt(dh) of dS is applied to dK at its store and to
//   dQ in the final cast; dV / dK leave through smem + TMA stores.  The same
//   smem tiles serve as K-major and MN-major UMMA operands, so no transposes
//   are materialised.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <cstring>

#include "common.h"
#include "flash.h"
#include "ptx.cuh"

namespace mobius {

namespace {

constexpr int BQ = 128;
constexpr int BKV = 128;

__device__ __forceinline__ void named_bar(int id, int n) { asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory"); }

// byte offset of 16-byte chunk `c` (8 bf16) of row `r` in a K-major SW128
// tile of 128 rows whose K extent is split in 64-element atoms of 16 KiB
__device__ __forceinline__ uint32_t sw128_off(int r, int c) {
  return (uint32_t)((c >> 3) * 16384 + (r >> 3) * 1024 + (r & 7) * 128 + (((c & 7) ^ (r & 7)) << 4));
}

__device__ __forceinline__ uint32_t pack_bf16(float a, float b) {
  __nv_bfloat162 h = __floats2bfloat162_rn(a, b);
  return *reinterpret_cast<uint32_t*>(&h);
}

__device__ __forceinline__ void st_shared_v4(uint32_t addr, uint32_t a, uint32_t b, uint32_t c, uint32_t d) {
  asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(addr), "r"(a), "r"(b), "r"(c), "r"(d) : "memory");
}

__device__ __forceinline__ void sts_f32(uint32_t addr, float v) {
  asm volatile("st.shared.f32 [%0], %1;" ::"r"(addr), "f"(v) : "memory");
}
__device__ __forceinline__ float lds_f32(uint32_t addr) {
  float v;
  asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(addr) : "memory");
  return v;
}

__device__ __forceinline__ float4 lds_f32x4(uint32_t addr) {
  float4 v;
  asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(addr)
               : "memory");
  return v;
}

__device__ __forceinline__ float ex2(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}

__device__ __forceinline__ uint32_t pack_bf16x2(float2 v) { return pack_bf16(v.x, v.y); }

// 2^x for a pair on the FMA pipe instead of the MUFU unit (the forward
// softmax issues one ex2 per score, which makes MUFU its busiest pipe):
// 2^x = 2^round(x) * q(f), f = x - round(x) in [-1/2, 1/2], q a degree-3
// fit of 2^f (max relative error 1.8e-4, far below the bf16 rounding of P;
// coefficients from a relative-error least-squares fit on Chebyshev nodes).
// round(x) comes from the 1.5 * 2^23 magic-number add, whose low mantissa
// bits then hold it as an integer that is shifted into the exponent.
// Arguments below -125 (masked scores: -inf) give exactly 0, like ex2.approx.ftz.
__device__ __forceinline__ float2 ex2_poly2(float2 x0) {
  float2 x;
  x.x = fmaxf(x0.x, -125.f);
  x.y = fmaxf(x0.y, -125.f);
  const float2 magic = make_float2(12582912.f, 12582912.f);
  const float2 j = __fadd2_rn(x, magic);
  const float2 t = __fadd2_rn(j, make_float2(-12582912.f, -12582912.f));  // round(x)
  const float2 f = __fadd2_rn(x, make_float2(-t.x, -t.y));
  float2 q = __ffma2_rn(make_float2(0.053241830319166183f, 0.053241830319166183f), f,
                        make_float2(0.24228397011756897f, 0.24228397011756897f));
  q = __ffma2_rn(q, f, make_float2(0.6935495138168335f, 0.6935495138168335f));
  q = __ffma2_rn(q, f, make_float2(0.9999545216560364f, 0.9999545216560364f));
  return make_float2(x0.x < -125.f ? 0.f : __int_as_float(__float_as_int(q.x) + (__float_as_int(j.x) << 23)),
                     x0.y < -125.f ? 0.f : __int_as_float(__float_as_int(q.y) + (__float_as_int(j.y) << 23)));
}
#ifdef MOBIUS_BWD_PROF  // debug: per-phase clock64 totals of one CTA's MMA / softmax-gradient warps (printf)
#define BPROF_DECL long long bprof[8] = {0, 0, 0, 0, 0, 0, 0, 0}; long long bprof_t0 = clock64();
#define BPROF(k, ...) do { long long t0_ = clock64(); __VA_ARGS__; bprof[k] += clock64() - t0_; } while (0)
#define BPROF_DUMP(tag) if ((blockIdx.x == 0 || blockIdx.x == 77) && lane == 0) printf("%s blk %d warp %d total %lld: %lld %lld %lld %lld %lld %lld %lld %lld\n", tag, blockIdx.x, warp, clock64() - bprof_t0, bprof[0], bprof[1], bprof[2], bprof[3], bprof[4], bprof[5], bprof[6], bprof[7]);
#else
#define BPROF_DECL
#define BPROF(k, ...) __VA_ARGS__
#define BPROF_DUMP(tag)
#endif
#ifndef MOBIUS_FLASH_POLY_PAIRS
#define MOBIUS_FLASH_POLY_PAIRS 2  // of every 16 pairs of scores, this many use ex2_poly2 (forward)
#endif
// score pair e/2 of a 32-column slab: polynomial or MUFU
__device__ __forceinline__ float2 ex2_pair(float a, float b, int pair) {
  if ((pair & 15) < MOBIUS_FLASH_POLY_PAIRS) return ex2_poly2(make_float2(a, b));
  return make_float2(ex2(a), ex2(b));
}

// (Polynomial exp2 for part of the backward's P^T was measured slower: 2 / 4 /
// 6 of 16 pairs: 672 / 740 / 734 us against 665 us at mbs 32, dh 64.)
// Softmax-gradient math of one 32-query slab of a key row (flash bwd):
//   P^T[r, q]  = 2^(S^T[r, q] * c - lse_q)          (masked to q >= r on the diagonal tile)
//   dS^T[r, q] = P^T[r, q] * (dP^T[r, q] - D_q)      (the 1/sqrt(dh) factor is applied to
//                                                     dK / dQ after accumulation)
// sLDq: smem address of lse[q0..q0+31] (fp32), followed 512 bytes later by -D.
// Packed f32x2 arithmetic (FADD2/FMUL2); the non-diagonal instantiation
// carries no masking code at all.
template <bool DIAG>
__device__ __forceinline__ void bwd_slab_math(const uint32_t (&vs)[32], const uint32_t (&vd)[32], uint32_t sLDq,
                                              int q0, int r, float sl2, uint32_t (&ppk)[16], uint32_t (&dpk)[16]) {
#pragma unroll
  for (int e = 0; e < 32; e += 4) {
    const float4 L = lds_f32x4(sLDq + e * 4), nD = lds_f32x4(sLDq + 512 + e * 4);  // broadcast reads
    float p0 = ex2(fmaf(__uint_as_float(vs[e]), sl2, -L.x));
    float p1 = ex2(fmaf(__uint_as_float(vs[e + 1]), sl2, -L.y));
    float p2 = ex2(fmaf(__uint_as_float(vs[e + 2]), sl2, -L.z));
    float p3 = ex2(fmaf(__uint_as_float(vs[e + 3]), sl2, -L.w));
    if (DIAG) {  // key r attends only from queries >= r
      const int q = q0 + e;
      if (q < r) p0 = 0.f;
      if (q + 1 < r) p1 = 0.f;
      if (q + 2 < r) p2 = 0.f;
      if (q + 3 < r) p3 = 0.f;
    }
    const float2 P01 = make_float2(p0, p1), P23 = make_float2(p2, p3);
    const float2 t01 = __fadd2_rn(make_float2(__uint_as_float(vd[e]), __uint_as_float(vd[e + 1])), make_float2(nD.x, nD.y));
    const float2 t23 =
        __fadd2_rn(make_float2(__uint_as_float(vd[e + 2]), __uint_as_float(vd[e + 3])), make_float2(nD.z, nD.w));
    ppk[e >> 1] = pack_bf16x2(P01);
    ppk[(e >> 1) + 1] = pack_bf16x2(P23);
    dpk[e >> 1] = pack_bf16x2(__fmul2_rn(P01, t01));
    dpk[(e >> 1) + 1] = pack_bf16x2(__fmul2_rn(P23, t23));
  }
}

// The same math for the dh 64 kernel, software-pipelined: the lse / -D
// values of the next 4 queries (two broadcast LDS.128) are requested before
// the current 4 are computed, so the shared-memory latency overlaps the MUFU
// work instead of stalling the FFMA that consumes them (ncu: short-scoreboard
// stalls on exactly those FFMAs were the largest stall in the slab math); the
// scale-subtract runs as packed FFMA2 (computing -x, negated for free in the
// MUFU operand).
template <bool DIAG>
__device__ __forceinline__ void bwd_slab_math_pl(const uint32_t (&vs)[32], const uint32_t (&vd)[32], uint32_t sLDq,
                                                 int q0, int r, float sl2, uint32_t (&ppk)[16], uint32_t (&dpk)[16]) {
  float4 L = lds_f32x4(sLDq), nD = lds_f32x4(sLDq + 512);
  const float2 nsl = make_float2(-sl2, -sl2);
#pragma unroll
  for (int e = 0; e < 32; e += 4) {
    float4 Ln = L, nDn = nD;
    if (e + 4 < 32) {
      Ln = lds_f32x4(sLDq + (e + 4) * 4);
      nDn = lds_f32x4(sLDq + 512 + (e + 4) * 4);
    }
    // -x = L - s sl2 (FFMA2), P = 2^x with the negation folded into MUFU.EX2's operand
    const float2 y01 = __ffma2_rn(make_float2(__uint_as_float(vs[e]), __uint_as_float(vs[e + 1])), nsl, make_float2(L.x, L.y));
    const float2 y23 =
        __ffma2_rn(make_float2(__uint_as_float(vs[e + 2]), __uint_as_float(vs[e + 3])), nsl, make_float2(L.z, L.w));
    float p0 = ex2(-y01.x), p1 = ex2(-y01.y), p2 = ex2(-y23.x), p3 = ex2(-y23.y);
    if (DIAG) {  // key r attends only from queries >= r
      const int q = q0 + e;
      if (q < r) p0 = 0.f;
      if (q + 1 < r) p1 = 0.f;
      if (q + 2 < r) p2 = 0.f;
      if (q + 3 < r) p3 = 0.f;
    }
    const float2 P01 = make_float2(p0, p1), P23 = make_float2(p2, p3);
    const float2 t01 = __fadd2_rn(make_float2(__uint_as_float(vd[e]), __uint_as_float(vd[e + 1])), make_float2(nD.x, nD.y));
    const float2 t23 =
        __fadd2_rn(make_float2(__uint_as_float(vd[e + 2]), __uint_as_float(vd[e + 3])), make_float2(nD.z, nD.w));
    ppk[e >> 1] = pack_bf16x2(P01);
    ppk[(e >> 1) + 1] = pack_bf16x2(P23);
    dpk[e >> 1] = pack_bf16x2(__fmul2_rn(P01, t01));
    dpk[(e >> 1) + 1] = pack_bf16x2(__fmul2_rn(P23, t23));
    L = Ln;
    nD = nDn;
  }
}
#ifndef MOBIUS_BWD_MATH
#define MOBIUS_BWD_MATH 1  // dh 64 kernel: 1 = bwd_slab_math_pl, 0 = bwd_slab_math
#endif

constexpr int NT_FWD = 320;  // 10 warps: TMA, MMA, 8 softmax warps (4 lane quadrants x 2 column halves)

template <int DH>
struct FwdCfg {
  static constexpr int Q_BYTES = BQ * DH * 2;
  static constexpr int KV_BYTES = BKV * DH * 2;
  // dh 64: P (bf16, 64 packed columns per buffer) lives in TMEM columns
  // 384 / 448 and feeds O += P V as the A operand of a TS-MMA, so PV reads
  // only V from smem and the softmax warps write P with tcgen05.st; dh 128
  // has no TMEM left (O[2] takes 256 columns) and stages P in smem
  static constexpr bool P_TMEM = DH == 64;
  static constexpr int P_BYTES = P_TMEM ? 0 : BQ * BKV * 2;
  static constexpr int KVS = DH == 64 ? 4 : 1;  // K/V ring depth (smem budget)
  // dh 64: O leaves through a staging tile (4 KB per 32-row quadrant) and
  // TMA stores; dh 128 has no smem left for it and stores row per thread
  static constexpr int O_STG = DH == 64 ? 128 * 128 : 0;
  static constexpr int SMEM = 1024 + 2 * Q_BYTES + 2 * KVS * KV_BYTES + 2 * P_BYTES + O_STG + 8192;  // + sMax/sSum (<= 6 KB at CP 4), barriers
};

struct FwdParams {
  __nv_bfloat16* O;  // [mbs*s, h] (head view)
  float* lse;        // [mbs, nh, s], log2 domain
  int s, nh, h, mbs;
  float scale_log2;  // log2(e) / sqrt(dh)
  int group;         // (batch, head) pairs per item chunk (see chunked_item)
};

// Item order of the persistent kernels: the (batch, head) pairs are taken
// `group` at a time and each chunk's items are listed heaviest tile first.
// All tiles of a pair then run within a few waves of each other, so the
// pair's fp32 dQ accumulator (backward) stays in L2 between its key tiles;
// ordering the whole list heaviest first (one tile level for every pair,
// then the next; group = all pairs, still the forward's order) re-reads it
// from DRAM (ncu: flash bwd moved 3.1 GB per call at mbs 32, five times its
// algorithmic bytes).
// Returns the tile level (0 = heaviest) and the pair index.
__device__ __forceinline__ void chunked_item(int i, int n_t, int nbh, int group, int& level, int& pair) {
  const int per = group * n_t;
  const int c = i / per, idx = i - c * per;
  const int gc = min(group, nbh - c * group);  // pairs in this (possibly partial) chunk
  level = idx / gc;
  pair = c * group + idx % gc;
}

// Persistent item order: pass k visits CTAs left-to-right for even k and
// right-to-left for odd k over a list sorted heaviest first, so per-CTA
// work balances (static round robin leaves the first CTAs ~9% heavier)
__device__ __forceinline__ int snake_item(int pass, int ncta, int cta) {
  return pass * ncta + ((pass & 1) ? ncta - 1 - cta : cta);
}

__device__ __forceinline__ void fwd_item(const FwdParams& p, int i, int& qt, int& hd, int& b) {
  const int n_qt = p.s / BQ, nb = p.nh * p.mbs;
  int level, r;
  chunked_item(i, n_qt, nb, p.group, level, r);
  qt = n_qt - 1 - level;  // heaviest (most kv tiles) first within a chunk
  hd = r % p.nh;
  b = r / p.nh;
}

// Persistent: one CTA per SM loops over (batch, head, 128-query tile) items.
// The TMA warp runs ahead into the next item (Q and O double-buffered), S_j
// is double-buffered in TMEM so the tensor core computes S_{j+1} while the
// softmax warps process S_j, P_j is double-buffered in smem, O accumulates in
// TMEM with lazy rescaling.  Each query row is handled by two softmax warps
// (column halves) that exchange only the row max.  All barrier phases run on
// global step counters across items.
template <int DH, int CP>
__global__ void __launch_bounds__((2 + 4 * CP) * 32, 1)
    flash_fwd_kernel(const __grid_constant__ CUtensorMap tm, const __grid_constant__ CUtensorMap tmo,
                     const FwdParams p) {
  using C = FwdCfg<DH>;
  constexpr int NSW = 4 * CP;  // softmax warps
  constexpr int KVS = C::KVS;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sQ = smem;                     // [2]
  uint8_t* sK = sQ + 2 * C::Q_BYTES;      // [KVS]
  uint8_t* sV = sK + KVS * C::KV_BYTES;   // [KVS]
  uint8_t* sP = sV + KVS * C::KV_BYTES;   // [2]
  uint8_t* sO = sP + 2 * C::P_BYTES;      // O staging (dh 64)
  float* sMax = reinterpret_cast<float*>(sO + C::O_STG);  // [2 iters][CP parts][128]
  float* sSum = sMax + 2 * CP * 128;                              // [CP parts][128]
  uint64_t* bars = reinterpret_cast<uint64_t*>(sSum + CP * 128);
  uint64_t* q_full = bars;                  // [2]
  uint64_t* q_empty = bars + 2;             // [2]
  uint64_t* s_full = bars + 4;              // [2]
  uint64_t* s_empty = bars + 6;             // [2] (count 8)
  uint64_t* p_full = bars + 8;              // [2] (count 8)
  uint64_t* pv_done = bars + 10;            // [2] PV of global step g commits pv_done[g & 1]
  uint64_t* o_ready = bars + 12;            // [2] all PVs of an item done
  uint64_t* o_empty = bars + 14;            // [2] (count 8) O read out
  uint64_t* k_full = bars + 16;             // [KVS]
  uint64_t* k_empty = k_full + KVS;         // [KVS]
  uint64_t* v_full = k_empty + KVS;         // [KVS]
  uint64_t* v_empty = v_full + KVS;         // [KVS]
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(v_empty + KVS);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int n_items = (p.s / BQ) * p.nh * p.mbs;

  if (threadIdx.x == 0) {
    ptx::tma_prefetch_desc(&tm);
    for (int i = 0; i < KVS; ++i) {
      ptx::mbar_init(&k_full[i], 1);
      ptx::mbar_init(&k_empty[i], 1);
      ptx::mbar_init(&v_full[i], 1);
      ptx::mbar_init(&v_empty[i], 1);
    }
    for (int i = 0; i < 2; ++i) {
      ptx::mbar_init(&q_full[i], 1);
      ptx::mbar_init(&q_empty[i], 1);
      ptx::mbar_init(&s_full[i], 1);
      ptx::mbar_init(&s_empty[i], NSW);
      ptx::mbar_init(&p_full[i], NSW);
      ptx::mbar_init(&pv_done[i], 1);
      ptx::mbar_init(&o_ready[i], 1);
      ptx::mbar_init(&o_empty[i], NSW);
    }
    ptx::fence_mbar_init();
  }
  if (warp == 1) ptx::tmem_alloc<512>(tmem_slot);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem_k = *tmem_slot;
  const uint32_t tmem = tmem_k;
  // TMEM: S[2] at 0 / 128, O[2] at 256 / 256 + DH, P[2] at 384 / 448 (dh 64)
  if (warp == 0) {
    if (lane == 0) {
      int g = 0, it = 0;
      for (int pass = 0; pass * (int)gridDim.x < n_items; ++pass) {
        const int i = snake_item(pass, (int)gridDim.x, (int)blockIdx.x);
        if (i >= n_items) continue;
        int qt, hd, b;
        fwd_item(p, i, qt, hd, b);
        const int qb = it & 1;
        ptx::mbar_wait(&q_empty[qb], ((it >> 1) & 1) ^ 1);
        ptx::mbar_arrive_expect_tx(&q_full[qb], C::Q_BYTES);
#pragma unroll
        for (int c = 0; c < DH / 64; ++c)
          ptx::tma_load_4d(sQ + qb * C::Q_BYTES + c * 16384, &tm, &q_full[qb], 64 * c, qt * BQ, hd, b);
        for (int j = 0; j <= qt; ++j, ++g) {
          const int st = g % KVS, kph = (g / KVS) & 1;
          ptx::mbar_wait(&k_empty[st], kph ^ 1);
          ptx::mbar_arrive_expect_tx(&k_full[st], C::KV_BYTES);
#pragma unroll
          for (int c = 0; c < DH / 64; ++c)
            ptx::tma_load_4d(sK + st * C::KV_BYTES + c * 16384, &tm, &k_full[st], 64 * c, j * BKV, p.nh + hd, b);
          ptx::mbar_wait(&v_empty[st], kph ^ 1);
          ptx::mbar_arrive_expect_tx(&v_full[st], C::KV_BYTES);
#pragma unroll
          for (int c = 0; c < DH / 64; ++c)
            ptx::tma_load_4d(sV + st * C::KV_BYTES + c * 16384, &tm, &v_full[st], 64 * c, j * BKV, 2 * p.nh + hd, b);
        }
        ++it;
      }
    }
  } else if (warp == 1) {
    {  // whole warp, converged: every MMA / commit is issued by one elected lane (ptx::*_w)
      const uint32_t tmem = __shfl_sync(0xffffffffu, tmem_k, 0);  // warp-uniform TMEM base
      constexpr uint32_t ID_S = ptx::idesc_bf16(BQ, BKV, 0, 0);
      constexpr uint32_t ID_O = ptx::idesc_bf16(BQ, DH, 0, 1);
      int gs = 0, gp = 0, it = 0;  // global S-issue step, global PV step, local item count
      for (int pass = 0; pass * (int)gridDim.x < n_items; ++pass) {
        const int i = snake_item(pass, (int)gridDim.x, (int)blockIdx.x);
        if (i >= n_items) continue;
        int qt, hd, b;
        fwd_item(p, i, qt, hd, b);
        const int nkv = qt + 1, ob = it & 1;
        ptx::mbar_wait(&q_full[ob], (it >> 1) & 1);
        const uint32_t aq = ptx::smem_u32(sQ + ob * C::Q_BYTES);
        auto issue_s = [&](int last) {
          const int st = gs % KVS, kph = (gs / KVS) & 1, sb = gs & 1;
          ptx::mbar_wait(&k_full[st], kph);
          ptx::mbar_wait(&s_empty[sb], ((gs >> 1) & 1) ^ 1);
          ptx::tc_fence_after();
          const uint32_t ak = ptx::smem_u32(sK + st * C::KV_BYTES);
#pragma unroll
          for (int k = 0; k < DH / 16; ++k) {
            const uint32_t off = (k >> 2) * 16384 + (k & 3) * 32;
            ptx::mma_bf16_w(tmem + sb * 128, ptx::sdesc_sw128(aq + off, 16, 1024), ptx::sdesc_sw128(ak + off, 16, 1024),
                          ID_S, k > 0);
          }
          ptx::mma_commit_w(&s_full[sb]);
          ptx::mma_commit_w(&k_empty[st]);
          if (last) ptx::mma_commit_w(&q_empty[ob]);
          ++gs;
        };
        issue_s(nkv == 1);
        ptx::mbar_wait(&o_empty[ob], ((it >> 1) & 1) ^ 1);  // O[ob] read out (item it-2)
        for (int j = 0; j < nkv; ++j) {
          if (j + 1 < nkv) issue_s(j + 2 == nkv);
          const int st = gp % KVS, kph = (gp / KVS) & 1, pb = gp & 1;
          ptx::mbar_wait(&p_full[pb], (gp >> 1) & 1);
          ptx::mbar_wait(&v_full[st], kph);
          ptx::tc_fence_after();
          const uint32_t ap = ptx::smem_u32(sP + pb * C::P_BYTES), av = ptx::smem_u32(sV + st * C::KV_BYTES);
          if constexpr (C::P_TMEM) {
#pragma unroll
            for (int k = 0; k < BKV / 16; ++k)  // 16 keys = 8 packed TMEM columns of P
              ptx::mma_bf16_ts_w(tmem + 256 + ob * DH, tmem + 384 + pb * 64 + 8 * k,
                               ptx::sdesc_sw128(av + k * 2048, 16384, 1024), ID_O, (j > 0 || k > 0) ? 1u : 0u);
          } else {
#pragma unroll
            for (int k = 0; k < BKV / 16; ++k) {
              const uint32_t offp = (k >> 2) * 16384 + (k & 3) * 32;
              ptx::mma_bf16_w(tmem + 256 + ob * DH, ptx::sdesc_sw128(ap + offp, 16, 1024),
                            ptx::sdesc_sw128(av + k * 2048, 16384, 1024), ID_O, (j > 0 || k > 0) ? 1u : 0u);
            }
          }
          ptx::mma_commit_w(&pv_done[pb]);
          ptx::mma_commit_w(&v_empty[st]);
          ++gp;
        }
        ptx::mma_commit_w(&o_ready[ob]);
        ++it;
      }
    }
  } else {
    // ------------------------------------------------ softmax warps
    // 4 * CP warps: (TMEM lane quadrant q4) x (column part cq of CP); a
    // thread owns row `row` of S, columns [cq SC, cq SC + SC), and OC
    // columns of O
    constexpr int SC = 128 / CP, NG = SC / 32, OC = DH / CP;
    const int q4 = warp & 3;           // TMEM lane quadrant
    const int cq = (warp - 2) >> 2;    // column part of S (and of O)
    const int row = q4 * 32 + lane;
    const uint32_t lb = (uint32_t)(q4 * 32) << 16;
    const float sc = p.scale_log2;
    int g = 0, it = 0;
    // deferred O epilogue of the previous item
    bool pend = false;
    int pd_ob = 0;
    uint32_t pd_ph = 0;
    float pd_l = 1.f, pd_m = 0.f;
    __nv_bfloat16* pd_orow = nullptr;
    float* pd_lse = nullptr;
    int pd_qt = 0, pd_hd = 0, pd_b = 0;
    const bool o_issuer = cq == 0 && lane == 0;  // issues this quadrant's O TMA stores (dh 64)
    const uint32_t o_slab = ptx::smem_u32(sO) + q4 * 4096;
    // OC columns of O in TMEM (oc0: first column of this part) <-> registers
    auto o_pack_store = [&](uint32_t base, float inv_l) {
      // base: TMEM address of this part's O columns; writes bf16(O * inv_l)
      if constexpr (OC == 16) {
        uint32_t v[16];
        __syncwarp();
        ptx::tmem_ld16(base, v);
        ptx::tmem_ld_wait();
        uint32_t pk[8];
#pragma unroll
        for (int e = 0; e < 16; e += 2)
          pk[e / 2] = pack_bf16(__uint_as_float(v[e]) * inv_l, __uint_as_float(v[e + 1]) * inv_l);
        static_assert(DH == 64, "OC 16 only at dh 64");
#pragma unroll
        for (int k = 0; k < 2; ++k)
          st_shared_v4(o_slab + lane * 128 + (((cq * 2 + k) ^ (lane & 7)) << 4), pk[4 * k], pk[4 * k + 1],
                       pk[4 * k + 2], pk[4 * k + 3]);
      } else {
#pragma unroll
        for (int c = 0; c < OC / 32; ++c) {
          uint32_t v[32];
          __syncwarp();
          ptx::tmem_ld32(base + c * 32, v);
          ptx::tmem_ld_wait();
          uint32_t pk[16];
#pragma unroll
          for (int e = 0; e < 32; e += 2)
            pk[e / 2] = pack_bf16(__uint_as_float(v[e]) * inv_l, __uint_as_float(v[e + 1]) * inv_l);
          if constexpr (DH == 64) {  // row `lane` of the quadrant's 32-row slab, 16-byte chunks, SW128
#pragma unroll
            for (int k = 0; k < 4; ++k)
              st_shared_v4(o_slab + lane * 128 + (((cq * (OC / 8) + c * 4 + k) ^ (lane & 7)) << 4), pk[4 * k],
                           pk[4 * k + 1], pk[4 * k + 2], pk[4 * k + 3]);
          } else {
#pragma unroll
            for (int k = 0; k < 4; ++k)
              *reinterpret_cast<uint4*>(pd_orow + c * 32 + k * 8) =
                  make_uint4(pk[4 * k], pk[4 * k + 1], pk[4 * k + 2], pk[4 * k + 3]);
          }
        }
      }
    };
    auto store_o = [&]() {
      if (!pend) return;
      pend = false;
      ptx::mbar_wait(&o_ready[pd_ob], pd_ph);
      ptx::tc_fence_after();
      const float inv_l = 1.f / pd_l;
      if constexpr (DH == 64) {
        if (o_issuer) asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");  // previous store read the slab
        named_bar(2 + q4, 32 * CP);
      }
      o_pack_store(tmem + 256 + pd_ob * DH + cq * OC + lb, inv_l);
      if constexpr (DH == 64) {
        ptx::fence_proxy_async();
        named_bar(2 + q4, 32 * CP);
        if (o_issuer) {
          asm volatile("cp.async.bulk.tensor.4d.global.shared::cta.bulk_group [%0, {%2, %3, %4, %5}], [%1];" ::"l"(
                           reinterpret_cast<uint64_t>(&tmo)),
                       "r"(o_slab), "r"(0), "r"(pd_qt * BQ + q4 * 32), "r"(pd_hd), "r"(pd_b)
                       : "memory");
          asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        }
      }
      if (cq == 0) *pd_lse = pd_m + __log2f(pd_l);
      ptx::tc_fence_before();
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive(&o_empty[pd_ob]);
    };
    for (int pass = 0; pass * (int)gridDim.x < n_items; ++pass) {
      const int i = snake_item(pass, (int)gridDim.x, (int)blockIdx.x);
      if (i >= n_items) continue;
      int qt, hd, b;
      fwd_item(p, i, qt, hd, b);
      const int nkv = qt + 1, ob = it & 1;
      const int qrow = qt * BQ + row;
      float m_run = -INFINITY, l_run = 0.f;
      for (int j = 0; j < nkv; ++j, ++g) {
        const int sb = g & 1;
        const bool diag = (j == qt);
        const uint32_t TS = tmem + sb * 128 + cq * SC + lb;
        ptx::mbar_wait(&s_full[sb], (g >> 1) & 1);
        ptx::tc_fence_after();
        uint32_t v[NG][32];
        __syncwarp();
#pragma unroll
        for (int gi = 0; gi < NG; ++gi) ptx::tmem_ld32(TS + gi * 32, v[gi]);
        ptx::tmem_ld_wait();
        ptx::tc_fence_before();
        __syncwarp();
        if (lane == 0) ptx::mbar_arrive(&s_empty[sb]);  // S values are in registers
        const int cbase = cq * SC;  // first key column of this part
        if (diag) {  // mask keys > query (only on the diagonal tile)
#pragma unroll
          for (int gi = 0; gi < NG; ++gi)
#pragma unroll
            for (int e = 0; e < 32; ++e)
              if (cbase + gi * 32 + e > row) v[gi][e] = __float_as_uint(-INFINITY);
        }
        // pass A: part-row max of raw scores, combined across the CP warps of the row
        float mx;
        {  // four independent max chains (one serial chain was 32 dependent FMNMX3)
          float m4[4] = {-INFINITY, -INFINITY, -INFINITY, -INFINITY};
#pragma unroll
          for (int gi = 0; gi < NG; ++gi)
#pragma unroll
            for (int e = 0; e < 32; e += 2)
              m4[(e >> 1) & 3] =
                  fmaxf(m4[(e >> 1) & 3], fmaxf(__uint_as_float(v[gi][e]), __uint_as_float(v[gi][e + 1])));
          mx = fmaxf(fmaxf(m4[0], m4[1]), fmaxf(m4[2], m4[3]));
        }
        float* smx = sMax + (g & 1) * (CP * 128);
        sts_f32(ptx::smem_u32(smx + cq * 128 + row), mx);
        named_bar(2 + q4, 32 * CP);
#pragma unroll
        for (int c = 0; c < CP; ++c)
          if (c != cq) mx = fmaxf(mx, lds_f32(ptx::smem_u32(smx + c * 128 + row)));
        // lazy rescaling: keep the running max unless it grows by > 8 (log2)
        const float m_cand = fmaxf(m_run, mx * sc);
        const bool grow = m_cand > m_run + 8.f;
        const float m_new = grow ? m_cand : m_run;
        const float alpha = ex2(m_run - m_new);  // 1 when not growing; 0 at j = 0
        if (j >= 1 && __any_sync(0xffffffffu, grow)) {  // rescale this part of O (PV of step g-1 done)
          ptx::mbar_wait(&pv_done[(g - 1) & 1], ((g - 1) >> 1) & 1);
          ptx::tc_fence_after();
          const uint32_t TO = tmem + 256 + ob * DH + cq * OC + lb;
          if constexpr (OC == 16) {
            uint32_t o[16];
            ptx::tmem_ld16(TO, o);
            ptx::tmem_ld_wait();
#pragma unroll
            for (int e = 0; e < 16; ++e) o[e] = __float_as_uint(__uint_as_float(o[e]) * alpha);
            ptx::tmem_st16(TO, o);
          } else {
#pragma unroll
            for (int c = 0; c < OC / 32; ++c) {
              uint32_t o[32];
              ptx::tmem_ld32(TO + c * 32, o);
              ptx::tmem_ld_wait();
#pragma unroll
              for (int e = 0; e < 32; ++e) o[e] = __float_as_uint(__uint_as_float(o[e]) * alpha);
              ptx::tmem_st32(TO + c * 32, o);
            }
          }
          ptx::tmem_st_wait();
        }
        // P buffer sb is free once the PV of global step g-2 completed
        if (g >= 2) ptx::mbar_wait(&pv_done[sb], ((g - 2) >> 1) & 1);
        // pass B: P = 2^(x*sc - m_new) -> TMEM / smem (bf16), part-row sum
        const uint32_t sp = ptx::smem_u32(sP + sb * C::P_BYTES);
        // packed f32x2 scale-subtract and two interleaved f32x2 row-sum
        // accumulators (a scalar sum was one 64-long dependent FADD chain)
        float2 rsa = make_float2(0.f, 0.f), rsb = make_float2(0.f, 0.f);
        const float2 sc2 = make_float2(sc, sc), nm2 = make_float2(-m_new, -m_new);
#pragma unroll
        for (int gi = 0; gi < NG; ++gi) {
          uint32_t pk[16];
#pragma unroll
          for (int e = 0; e < 32; e += 2) {
            const float2 xx =
                __ffma2_rn(make_float2(__uint_as_float(v[gi][e]), __uint_as_float(v[gi][e + 1])), sc2, nm2);
            const float2 pp = ex2_pair(xx.x, xx.y, (e >> 1) + gi * 8);
            if ((e >> 1) & 1)
              rsb = __fadd2_rn(rsb, pp);
            else
              rsa = __fadd2_rn(rsa, pp);
            pk[e >> 1] = pack_bf16(pp.x, pp.y);
          }
          if constexpr (C::P_TMEM) {  // keys cq*SC + gi*32 .. -> packed columns cq*SC/2 + gi*16 ..
            ptx::tmem_st16(tmem + 384 + sb * 64 + cq * (SC / 2) + gi * 16 + lb, pk);
          } else {
#pragma unroll
            for (int k = 0; k < 4; ++k)
              st_shared_v4(sp + sw128_off(row, cq * (SC / 8) + gi * 4 + k), pk[4 * k], pk[4 * k + 1], pk[4 * k + 2],
                           pk[4 * k + 3]);
          }
        }
        if constexpr (C::P_TMEM) ptx::tmem_st_wait();
        const float rs = (rsa.x + rsa.y) + (rsb.x + rsb.y);
        l_run = l_run * alpha + rs;
        m_run = m_new;
        ptx::tc_fence_before();
        if constexpr (!C::P_TMEM) ptx::fence_proxy_async();  // P in smem feeds the PV MMA
        __syncwarp();
        if (lane == 0) ptx::mbar_arrive(&p_full[sb]);
        if (j == 0) store_o();  // previous item's O while this tile's PV runs
      }
      // output: O / l  (l = sum over the CP parts).  The O read-out waits for
      // the item's last PV, so it is deferred until the next item's first P
      // tile is handed to the tensor core (O is double-buffered in TMEM)
      sts_f32(ptx::smem_u32(sSum + cq * 128 + row), l_run);
      named_bar(2 + q4, 32 * CP);
      float l_tot = 0.f;
#pragma unroll
      for (int c = 0; c < CP; ++c) l_tot += lds_f32(ptx::smem_u32(sSum + c * 128 + row));
      named_bar(2 + q4, 32 * CP);  // partners read sSum before the next item overwrites it
      pend = true;
      pd_ob = ob;
      pd_ph = (it >> 1) & 1;
      pd_l = l_tot;
      pd_m = m_run;
      pd_orow = p.O + ((int64_t)b * p.s + qrow) * p.h + hd * DH + cq * OC;
      pd_lse = p.lse + ((int64_t)b * p.nh + hd) * p.s + qrow;
      pd_qt = qt;
      pd_hd = hd;
      pd_b = b;
      ++it;
    }
    store_o();
    if (DH == 64 && o_issuer) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");  // O stores complete
  }
  __syncthreads();
  if (warp == 1) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc<512>(tmem);
  }
}

// ---------------------------------------------------------------- fwd, dh 64
// Ping-pong forward for dh 64 (the 1.5B shape): two query tiles in flight per
// CTA, one per stream, so one softmax warpgroup's row max / exponentials
// overlap the other's and the tensor core interleaves both tiles' MMAs.
// 16 warps:
//   warps 0, 2  TMA of stream A / B: Q of the stream's items (double
//               buffered, the next item's Q prefetched at the current item's
//               last S), K / V tiles through the stream's 4-deep ring
//   warps 1, 3  MMA of stream A / B: S(r) = Q K_r^T as soon as the softmax
//               warps hold S(r-1) in registers, then O += P(r-1) V_{r-1};
//               each issuer commits its own MMAs, so neither stream's
//               issue order waits on the other's softmax
//   warps 4-7   softmax, stream A; warps 8-11 softmax, stream B: thread =
//               query row, all 128 key columns of the tile (no cross-warp
//               max / sum exchange); P (bf16) -> TMEM, feeds PV as a TS-MMA
//   warps 12-15 epilogue: O / l of a finished item -> bf16 -> 32-row smem
//               slab per warp -> TMA store; lse
// The CTA's persistent item list (heaviest first, snake order) is dealt
// alternately to the two streams.  setmaxnreg: 56 / 192 / 192 / 72.
// TMEM per stream X: S at 256 X (128 cols), P at 256 X + 128 (64 packed
// cols), O at 256 X + 192 (64 cols).
#ifndef MOBIUS_FWD_POLL_NS
#define MOBIUS_FWD_POLL_NS 256  // epilogue warps' back-off between o_ready polls (ns, 0 = spin)
#endif
#ifndef MOBIUS_FWD_MMA_BATCH
#define MOBIUS_FWD_MMA_BATCH 1
#endif
// register split of the dh-64 forward (per thread; 4 warpgroups, sum 512)
#ifndef MOBIUS_FWD_REG_WG0
#define MOBIUS_FWD_REG_WG0 56
#endif
#ifndef MOBIUS_FWD_REG_SMX
#define MOBIUS_FWD_REG_SMX 192
#endif
#ifndef MOBIUS_FWD_REG_EPI
#define MOBIUS_FWD_REG_EPI 72
#endif
static_assert(MOBIUS_FWD_REG_WG0 + 2 * MOBIUS_FWD_REG_SMX + MOBIUS_FWD_REG_EPI <= 512, "fwd64 register split");
struct Fwd64Cfg {
  static constexpr int T_BYTES = 128 * 64 * 2;  // Q / K / V tile
  static constexpr int KVR = 4;                 // K / V ring per stream (16 KB entries)
  static constexpr int SMEM = 1024 + 4 * T_BYTES + 2 * KVR * T_BYTES + 4 * 4096 + 2 * 2 * 2 * 128 * 4 + 512;
};

// per-stream walk over the CTA's items (stream X takes local items X, X+2, ...)
struct FwdStream {
  int k;              // items of this stream started so far - 1
  int nkv, qt, hd, b;
  int r;              // round within the item: S(r) if r < nkv, PV(r-1) if r >= 1
  bool act;
};

__global__ void __launch_bounds__(512, 1) flash_fwd64_kernel(const __grid_constant__ CUtensorMap tm,
                                                          const __grid_constant__ CUtensorMap tmo, const FwdParams p) {
  using C = Fwd64Cfg;
  constexpr int DH = 64, KVR = C::KVR;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sQ = smem;                         // [stream][buf]
  uint8_t* sKV = sQ + 4 * C::T_BYTES;         // [stream][KVR]
  uint8_t* sO = sKV + 2 * KVR * C::T_BYTES;   // [4 warps] 32-row O staging slabs (4 KB)
  float* sLM = reinterpret_cast<float*>(sO + 4 * 4096);  // [stream][item parity][l | m][128]
  uint64_t* bars = reinterpret_cast<uint64_t*>(sLM + 2 * 2 * 2 * 128);
  uint64_t* q_full = bars;         // [stream * 2 + buf]
  uint64_t* q_empty = bars + 4;    // [stream * 2 + buf]
  uint64_t* kv_full = bars + 8;    // [stream * KVR + e]
  uint64_t* kv_empty = bars + 8 + 2 * KVR;
  uint64_t* s_full = bars + 8 + 4 * KVR;  // [stream]
  uint64_t* s_free = s_full + 2;          // [stream] (count 4)
  uint64_t* p_full = s_full + 4;          // [stream] (count 4)
  uint64_t* pv_done = s_full + 6;         // [stream]
  uint64_t* o_ready = s_full + 8;         // [stream]
  uint64_t* o_empty = s_full + 10;        // [stream] (count 4)
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(s_full + 12);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int n_items = (p.s / BQ) * p.nh * p.mbs;
  const int ncta = (int)gridDim.x, cta = (int)blockIdx.x;
  // stream-local item k of stream X -> (qt, hd, b); false past the CTA's list
  auto item_of = [&](int X, int k, FwdStream& x) {
    const int li = 2 * k + X;
    const int i = snake_item(li, ncta, cta);
    x.act = i < n_items;
    if (x.act) {
      fwd_item(p, i, x.qt, x.hd, x.b);
      x.nkv = x.qt + 1;
    }
  };
  auto stream_init = [&](int X, FwdStream& x) {
    x.k = 0;
    x.r = 0;
    item_of(X, 0, x);
  };
  auto stream_advance = [&](int X, FwdStream& x) {  // after a round
    if (++x.r > x.nkv) {
      ++x.k;
      x.r = 0;
      item_of(X, x.k, x);
    }
  };

  if (threadIdx.x == 0) {
    ptx::tma_prefetch_desc(&tm);
    ptx::tma_prefetch_desc(&tmo);
    for (int i = 0; i < 4; ++i) {
      ptx::mbar_init(&q_full[i], 1);
      ptx::mbar_init(&q_empty[i], 1);
    }
    for (int i = 0; i < 2 * KVR; ++i) {
      ptx::mbar_init(&kv_full[i], 1);
      ptx::mbar_init(&kv_empty[i], 1);
    }
    for (int x = 0; x < 2; ++x) {
      ptx::mbar_init(&s_full[x], 1);
      ptx::mbar_init(&s_free[x], 4);
      ptx::mbar_init(&p_full[x], 4);
      ptx::mbar_init(&pv_done[x], 1);
      ptx::mbar_init(&o_ready[x], 1);
      ptx::mbar_init(&o_empty[x], 4);
    }
    ptx::fence_mbar_init();
  }
  if (warp == 1) ptx::tmem_alloc<512>(tmem_slot);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_slot;

  if (warp == 0 || warp == 2) {
    asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(MOBIUS_FWD_REG_WG0));
    const int X = warp >> 1;
    if (lane == 0) {
      FwdStream x;
      stream_init(X, x);
      int op = 0;  // ring entries issued
      uint64_t* kvf = kv_full + X * KVR;
      uint64_t* kve = kv_empty + X * KVR;
      uint8_t* ring = sKV + X * KVR * C::T_BYTES;
      auto load_q = [&](int k, int qt, int hd, int b) {
        const int qb = X * 2 + (k & 1);
        ptx::mbar_wait(&q_empty[qb], ((k >> 1) & 1) ^ 1);
        ptx::mbar_arrive_expect_tx(&q_full[qb], C::T_BYTES);
        ptx::tma_load_4d(sQ + qb * C::T_BYTES, &tm, &q_full[qb], 0, qt * BQ, hd, b);
      };
      auto load_kv = [&](int slot_nh, int j, int hd, int b) {  // slot_nh: nh (K) or 2 nh (V)
        const int e = op % KVR;
        ptx::mbar_wait(&kve[e], ((op / KVR) & 1) ^ 1);
        ptx::mbar_arrive_expect_tx(&kvf[e], C::T_BYTES);
        ptx::tma_load_4d(ring + e * C::T_BYTES, &tm, &kvf[e], 0, j * BKV, slot_nh + hd, b);
        ++op;
      };
      if (x.act) load_q(0, x.qt, x.hd, x.b);
      while (x.act) {
        if (x.r < x.nkv) {
          load_kv(p.nh, x.r, x.hd, x.b);
          if (x.r == x.nkv - 1) {  // last S of the item: prefetch the stream's next Q
            FwdStream nx;
            item_of(X, x.k + 1, nx);
            if (nx.act) load_q(x.k + 1, nx.qt, nx.hd, nx.b);
          }
        }
        if (x.r >= 1) load_kv(2 * p.nh, x.r - 1, x.hd, x.b);
        stream_advance(X, x);
      }
    }
  } else if (warp == 1 || warp == 3) {
    asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(MOBIUS_FWD_REG_WG0));
    const int X = warp >> 1;
    const uint32_t tm0 = __shfl_sync(0xffffffffu, tmem, 0) + X * 256;  // warp-uniform TMEM base of the stream
    constexpr uint32_t ID_S = ptx::idesc_bf16(BQ, BKV, 0, 0);
    constexpr uint32_t ID_O = ptx::idesc_bf16(BQ, DH, 0, 1);
    uint64_t* kvf = kv_full + X * KVR;
    uint64_t* kve = kv_empty + X * KVR;
    const uint32_t ring = ptx::smem_u32(sKV + X * KVR * C::T_BYTES);
    FwdStream x;
    stream_init(X, x);
    int op = 0, gs = 0, gp = 0;
    BPROF_DECL
    while (x.act) {
      if (x.r < x.nkv) {  // S(r) = Q K_r^T
        const int e = op % KVR, qb = X * 2 + (x.k & 1);
        if (x.r == 0) BPROF(0, ptx::mbar_wait(&q_full[qb], (x.k >> 1) & 1));
        BPROF(1, ptx::mbar_wait(&kvf[e], (op / KVR) & 1));
        if (gs >= 1) BPROF(2, ptx::mbar_wait(&s_free[X], (gs - 1) & 1));  // softmax holds the previous S
        ptx::tc_fence_after();
        const uint32_t aq = ptx::smem_u32(sQ + qb * C::T_BYTES), ak = ring + e * C::T_BYTES;
#if MOBIUS_FWD_MMA_BATCH  // 4 MMAs (K = 64) in one issue block, descriptors advanced by 32 bytes
        ptx::mma_bf16_ss4_w(tm0, ptx::sdesc_sw128(aq, 16, 1024), ptx::sdesc_sw128(ak, 16, 1024), ID_S, 0u, 2ull);
#else
#pragma unroll
        for (int t = 0; t < DH / 16; ++t)
          ptx::mma_bf16_w(tm0, ptx::sdesc_sw128(aq + t * 32, 16, 1024), ptx::sdesc_sw128(ak + t * 32, 16, 1024), ID_S,
                          t > 0);
#endif
        ptx::mma_commit_w(&s_full[X]);
        ptx::mma_commit_w(&kve[e]);
        if (x.r == x.nkv - 1) ptx::mma_commit_w(&q_empty[qb]);
        ++op;
        ++gs;
      }
      if (x.r >= 1) {  // O += P(r-1) V_{r-1}
        const int j = x.r - 1, e = op % KVR;
        BPROF(3, ptx::mbar_wait(&p_full[X], gp & 1));
        BPROF(4, ptx::mbar_wait(&kvf[e], (op / KVR) & 1));
        if (j == 0 && x.k >= 1) BPROF(5, ptx::mbar_wait(&o_empty[X], (x.k - 1) & 1));  // previous item's O read out
        ptx::tc_fence_after();
        const uint32_t av = ring + e * C::T_BYTES;
#if MOBIUS_FWD_MMA_BATCH  // 8 TS MMAs (K = 128 keys) in one issue block; V rows advance 2048 bytes per 16 keys
        ptx::mma_bf16_ts8_w(tm0 + 192, tm0 + 128, ptx::sdesc_sw128(av, 16384, 1024), ID_O, j > 0 ? 1u : 0u, 128ull);
#else
#pragma unroll
        for (int t = 0; t < BKV / 16; ++t)  // 16 keys = 8 packed TMEM columns of P
          ptx::mma_bf16_ts_w(tm0 + 192, tm0 + 128 + 8 * t, ptx::sdesc_sw128(av + t * 2048, 16384, 1024), ID_O,
                             (j > 0 || t > 0) ? 1u : 0u);
#endif
        ptx::mma_commit_w(&pv_done[X]);
        ptx::mma_commit_w(&kve[e]);
        if (j == x.nkv - 1) ptx::mma_commit_w(&o_ready[X]);
        ++op;
        ++gp;
      }
      stream_advance(X, x);
    }
    BPROF_DUMP("fmma")
  } else if (warp < 12) {
    asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;" ::"n"(MOBIUS_FWD_REG_SMX));
    // ------------------------------------------------ softmax, stream X
    const int X = (warp - 4) >> 2, q4 = warp & 3;
    const int row = q4 * 32 + lane;
    const uint32_t lb = (uint32_t)(q4 * 32) << 16;
    const uint32_t TS = tmem + lb + X * 256, TP = TS + 128, TO = TS + 192;
    const float sc = p.scale_log2;
    int g = 0;  // tiles of this stream so far (S and PV counters)
    FwdStream x;
    stream_init(X, x);
    BPROF_DECL
#ifdef MOBIUS_BWD_PROF
    long long tb;
#define FP_MARK(k) { long long t_ = clock64(); bprof[k] += t_ - tb; tb = t_; }
#else
#define FP_MARK(k)
#endif
    while (x.act) {
      const int nkv = x.nkv;
      float m_run = -INFINITY, l_run = 0.f;
      for (int j = 0; j < nkv; ++j, ++g) {
#ifdef MOBIUS_BWD_PROF
        tb = clock64();
#endif
        ptx::mbar_wait(&s_full[X], g & 1);
        FP_MARK(0)
        ptx::tc_fence_after();
        uint32_t v[4][32];
        __syncwarp();
#pragma unroll
        for (int gi = 0; gi < 4; ++gi) ptx::tmem_ld32(TS + gi * 32, v[gi]);
        ptx::tmem_ld_wait();
        ptx::tc_fence_before();
        __syncwarp();
        if (lane == 0) ptx::mbar_arrive(&s_free[X]);  // S values are in registers
        FP_MARK(1)
        if (j == x.qt) {  // diagonal tile: mask keys > query
#pragma unroll
          for (int gi = 0; gi < 4; ++gi)
#pragma unroll
            for (int e = 0; e < 32; ++e)
              if (gi * 32 + e > row) v[gi][e] = __float_as_uint(-INFINITY);
        }
        float mx;
        {  // four independent max chains
          float m4[4] = {-INFINITY, -INFINITY, -INFINITY, -INFINITY};
#pragma unroll
          for (int gi = 0; gi < 4; ++gi)
#pragma unroll
            for (int e = 0; e < 32; e += 2)
              m4[(e >> 1) & 3] = fmaxf(m4[(e >> 1) & 3], fmaxf(__uint_as_float(v[gi][e]), __uint_as_float(v[gi][e + 1])));
          mx = fmaxf(fmaxf(m4[0], m4[1]), fmaxf(m4[2], m4[3]));
        }
        // lazy rescaling: keep the running max unless it grows by > 8 (log2)
        const float m_cand = fmaxf(m_run, mx * sc);
        const bool grow = m_cand > m_run + 8.f;
        const float m_new = grow ? m_cand : m_run;
        const float alpha = ex2(m_run - m_new);  // 1 when not growing; 0 at j = 0
        // P = 2^(x sc - m_new) packed bf16, row sum (two f32x2 accumulators)
        uint32_t pk[4][16];
        float2 rsa = make_float2(0.f, 0.f), rsb = make_float2(0.f, 0.f);
        const float2 sc2 = make_float2(sc, sc), nm2 = make_float2(-m_new, -m_new);
#pragma unroll
        for (int gi = 0; gi < 4; ++gi) {
#pragma unroll
          for (int e = 0; e < 32; e += 2) {
            const float2 xx = __ffma2_rn(make_float2(__uint_as_float(v[gi][e]), __uint_as_float(v[gi][e + 1])), sc2, nm2);
            // all on MUFU: a polynomial share (2 / 4 / 6 / 8 of 16 pairs) measured
            // 232 / 246 / 258 / 281 us against 227 us at mbs 32
            const float2 pp = make_float2(ex2(xx.x), ex2(xx.y));
            if ((e >> 1) & 1)
              rsb = __fadd2_rn(rsb, pp);
            else
              rsa = __fadd2_rn(rsa, pp);
            pk[gi][e >> 1] = pack_bf16(pp.x, pp.y);
          }
        }
        const float rs = (rsa.x + rsa.y) + (rsb.x + rsb.y);
        l_run = l_run * alpha + rs;
        m_run = m_new;
        FP_MARK(2)
        // P and O of this stream are free once its previous PV completed
        if (g >= 1) {
          ptx::mbar_wait(&pv_done[X], (g - 1) & 1);
          ptx::tc_fence_after();
        }
        FP_MARK(3)
        if (j >= 1 && __any_sync(0xffffffffu, grow)) {  // rescale O (the item's PVs so far are done)
          uint32_t o[32];
#pragma unroll
          for (int c = 0; c < 2; ++c) {
            ptx::tmem_ld32(TO + c * 32, o);
            ptx::tmem_ld_wait();
#pragma unroll
            for (int e = 0; e < 32; ++e) o[e] = __float_as_uint(__uint_as_float(o[e]) * alpha);
            ptx::tmem_st32(TO + c * 32, o);
          }
        }
#pragma unroll
        for (int gi = 0; gi < 4; ++gi) ptx::tmem_st16(TP + gi * 16, pk[gi]);
        ptx::tmem_st_wait();
        if (j == nkv - 1) {  // l / m of the item for the epilogue (double-buffered by item parity)
          float* lm = sLM + (X * 2 + (x.k & 1)) * 256;
          lm[row] = l_run;
          lm[128 + row] = m_run;
        }
        ptx::tc_fence_before();
        __syncwarp();
        if (lane == 0) ptx::mbar_arrive(&p_full[X]);
        FP_MARK(4)
      }
      ++x.k;
      item_of(X, x.k, x);
    }
    BPROF_DUMP("fsmx")
  } else {
    asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(MOBIUS_FWD_REG_EPI));
    // ------------------------------------------------ epilogue
    // whichever stream's item finishes next: O / l -> bf16 -> this warp's
    // 32-row SW128 slab -> TMA store (one per warp); lse = m + log2 l
    const int q4 = warp & 3, row = q4 * 32 + lane;
    const uint32_t lb = (uint32_t)(q4 * 32) << 16;
    const uint32_t slab = ptx::smem_u32(sO) + q4 * 4096;
    FwdStream st[2];
    stream_init(0, st[0]);
    stream_init(1, st[1]);
    while (st[0].act || st[1].act) {
      int X = -1;
      while (X < 0) {  // poll: the streams finish items in an order set by the MMA interleave
        for (int c = 0; c < 2 && X < 0; ++c)
          if (st[c].act && ptx::mbar_test(&o_ready[c], st[c].k & 1)) X = c;
        X = __shfl_sync(0xffffffffu, X, 0);
        // back off between polls: a spinning warp takes issue slots from the
        // softmax warps on its SMSP (items finish every few thousand cycles)
        if (X < 0 && MOBIUS_FWD_POLL_NS) __nanosleep(MOBIUS_FWD_POLL_NS);
      }
      FwdStream& x = st[X];
      ptx::tc_fence_after();
      const float* lm = sLM + (X * 2 + (x.k & 1)) * 256;
      const float l = lm[row], m = lm[128 + row];
      uint32_t v[2][32];
      __syncwarp();
      ptx::tmem_ld32(tmem + lb + X * 256 + 192, v[0]);
      ptx::tmem_ld32(tmem + lb + X * 256 + 224, v[1]);
      ptx::tmem_ld_wait();
      ptx::tc_fence_before();
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive(&o_empty[X]);  // O of this stream may be overwritten
      const float inv_l = 1.f / l;
      if (lane == 0) asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");  // previous store read the slab
      __syncwarp();
#pragma unroll
      for (int c = 0; c < 2; ++c) {
        uint32_t pk[16];
#pragma unroll
        for (int e = 0; e < 32; e += 2)
          pk[e / 2] = pack_bf16(__uint_as_float(v[c][e]) * inv_l, __uint_as_float(v[c][e + 1]) * inv_l);
#pragma unroll
        for (int k = 0; k < 4; ++k)
          st_shared_v4(slab + lane * 128 + (((c * 4 + k) ^ (lane & 7)) << 4), pk[4 * k], pk[4 * k + 1], pk[4 * k + 2],
                       pk[4 * k + 3]);
      }
      ptx::fence_proxy_async();
      __syncwarp();
      if (lane == 0) {
        asm volatile("cp.async.bulk.tensor.4d.global.shared::cta.bulk_group [%0, {%2, %3, %4, %5}], [%1];" ::"l"(
                         reinterpret_cast<uint64_t>(&tmo)),
                     "r"(slab), "r"(0), "r"(x.qt * BQ + q4 * 32), "r"(x.hd), "r"(x.b)
                     : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      }
      p.lse[((int64_t)x.b * p.nh + x.hd) * p.s + x.qt * BQ + row] = m + __log2f(l);
      ++x.k;
      item_of(X, x.k, x);
    }
    if (lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc<512>(tmem);
  }
}

// ====================================================================== bwd
template <int DH>
struct BwdCfg {
  static constexpr int T_BYTES = 128 * DH * 2;       // one K / V / Q / dO tile
  static constexpr int QS = DH == 64 ? 2 : 1;        // Q/dO pipeline depth
  static constexpr int PT_BYTES = 128 * 128 * 2;     // P^T or dS^T tile
  static constexpr bool DQ_OWN = DH == 64;           // dQ has its own TMEM columns (else aliases S^T)
  // dh 64: P^T lives in TMEM columns 448..511 and feeds dV += P^T dO as the
  // A operand of a TS-MMA; the smem it used becomes the second dS^T buffer
  static constexpr bool PT_TMEM = DH == 64;
  // dh 64: dQ(i-1) is drained from its own staging tile while the MMAs of
  // tile i run; dh 128: staged in the P^T/dS^T tiles (smem budget)
  static constexpr int STG_BYTES = DQ_OWN ? 128 * DH * 4 : 0;
  static constexpr int SMEM = 1024 + 2 * T_BYTES + QS * 2 * T_BYTES + 2 * PT_BYTES + STG_BYTES + QS * 1024 + 256;
};

struct BwdParams {
  const float* lse;     // [mbs, nh, s] log2 domain
  const float* Dsum;    // [mbs, nh, s] -rowsum(dO * O) (negated)
  float* dQacc;         // [mbs*s, h] fp32 (head view), accumulated by TMA reduce-add
  __nv_bfloat16* dqkv;  // [mbs*s, 3h] (dh 64 kernel: dK / dV rows stored by the drain warpgroup)
  int s, nh, h, mbs;
  float scale_log2, scale;
  int group;            // (batch, head) pairs per item chunk (chunked_item)
};

__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   ptx::smem_u32(dst)),
               "l"(reinterpret_cast<uint64_t>(src)), "r"(bytes), "r"(ptx::smem_u32(bar))
               : "memory");
}

// Item = (batch, head, 128-key tile kt); it visits query tiles i >= kt.
// Persistent: one CTA per SM walks its items (snake order over the list
// sorted heaviest first, so per-CTA work balances to ~5%); all barrier
// phases run on a per-CTA global tile counter g, so the TMA warp prefetches
// the next item's Q/dO tiles and K/V while the current item finishes, and
// the next item's scores start while its predecessor's dV/dK leave TMEM.
// MMA order per query tile: [S^T, dP^T](i) ... wait P^T/dS^T(i) ... dV, dK,
// dQ(i), then [S^T, dP^T](i+1) right away (the softmax-gradient warps are
// done with S^T(i)), so the next scores overlap the dQ read-out.

template <int DH, int CP>
__global__ void __launch_bounds__((2 + 4 * CP) * 32, 1) flash_bwd_kernel(const __grid_constant__ CUtensorMap tm,
                                                              const __grid_constant__ CUtensorMap tdo,
                                                              const __grid_constant__ CUtensorMap tdq,
                                                              const __grid_constant__ CUtensorMap tdkv, const BwdParams p) {
  using C = BwdCfg<DH>;
  constexpr int QS = C::QS;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sK = smem;
  uint8_t* sV = sK + C::T_BYTES;
  uint8_t* sQ = sV + C::T_BYTES;             // [QS]
  uint8_t* sdO = sQ + QS * C::T_BYTES;       // [QS]
  uint8_t* sPT = sdO + QS * C::T_BYTES;
  uint8_t* sdST = sPT + C::PT_BYTES;
  uint8_t* sSTG = sdST + C::PT_BYTES;  // dQ staging (dh 64)
  float* sLD = reinterpret_cast<float*>(sSTG + C::STG_BYTES);  // [QS][lse 128 | -D 128]
  uint64_t* bars = reinterpret_cast<uint64_t*>(sLD + QS * 256);
  uint64_t* kv_full = bars;          // K/V of the current item landed
  uint64_t* q_full = bars + 1;       // [2] (Q, dO, lse, D)
  uint64_t* q_empty = bars + 3;      // [2]
  uint64_t* s_full = bars + 5;       // S^T and dP^T ready
  uint64_t* p_full = bars + 6;       // P^T / dS^T in smem (count 8)
  uint64_t* mm_done = bars + 7;      // dV/dK/dQ of this tile done (P^T/dS^T smem free, dQ ready)
  uint64_t* dq_empty = bars + 8;     // dQ read out (count 8)
  uint64_t* st_empty = bars + 9;     // S^T / dP^T loaded into registers (count 8)
  uint64_t* pt_free = bars + 10;     // dV MMAs of this tile done: P^T (TMEM) may be overwritten
  uint64_t* kv_empty = bars + 11;    // every MMA of an item done: K/V smem may be reloaded
  uint64_t* acc_empty = bars + 12;   // dV/dK of an item read out of TMEM (count 8)
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 13);
  // dS^T buffers: [g & 1] with P^T in TMEM, else a single tile
  uint8_t* const sdS_buf[2] = {C::PT_TMEM ? sPT : sdST, sdST};

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int n_t = p.s / 128;
  const int nbh = p.nh * p.mbs;
  const int n_items = n_t * nbh;
  const int ncta = (int)gridDim.x, cta = (int)blockIdx.x;
  // item index -> (key tile, head, batch); the list is sorted heaviest
  // first: every (b, head) with key tile 0 (n_t query tiles) before key tile 1 ...
  auto decode = [&](int item, int& kt, int& hd, int& b) {
    int r;
    chunked_item(item, n_t, nbh, p.group, kt, r);  // key tile 0 (most query tiles) first within a chunk
    hd = r % p.nh;
    b = r / p.nh;
  };

  if (threadIdx.x == 0) {
    ptx::tma_prefetch_desc(&tm);
    ptx::tma_prefetch_desc(&tdo);
    ptx::tma_prefetch_desc(&tdq);
    ptx::tma_prefetch_desc(&tdkv);
    ptx::mbar_init(kv_full, 1);
    for (int i = 0; i < 2; ++i) {
      ptx::mbar_init(&q_full[i], 1);
      ptx::mbar_init(&q_empty[i], 1);
    }
    ptx::mbar_init(s_full, 1);
    ptx::mbar_init(p_full, 4 * CP);
    ptx::mbar_init(mm_done, 1);
    ptx::mbar_init(dq_empty, 4 * CP);
    ptx::mbar_init(st_empty, 4 * CP);
    ptx::mbar_init(pt_free, 1);
    ptx::mbar_init(kv_empty, 1);
    ptx::mbar_init(acc_empty, 4 * CP);
    ptx::fence_mbar_init();
  }
  if (warp == 1) ptx::tmem_alloc<512>(tmem_slot);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  // TMEM: S^T 0..127, dP^T 128..255, dV 256.., dK 256+DH.., dQ 384.. (dh 64) or aliasing S^T (dh 128)
  const uint32_t T_S = tmem, T_DP = tmem + 128, T_DV = tmem + 256;
  const uint32_t T_DQ = C::DQ_OWN ? tmem + 384 : tmem;
  const uint32_t T_PT = tmem + 448;  // PT_TMEM only

  if (warp == 0) {
    if (lane == 0) {
      int g = 0, n = 0;  // global tile / item counters of this CTA
      for (int pass = 0; pass * ncta < n_items; ++pass) {
        const int item = snake_item(pass, ncta, cta);
        if (item >= n_items) continue;
        int kt, hd, b;
        decode(item, kt, hd, b);
        const int nq = n_t - kt;
        const int64_t ld_base = ((int64_t)b * p.nh + hd) * p.s;
        auto load_q = [&](int it) {
          const int gg = g + it, st = gg % QS, ph = (gg / QS) & 1, qi = kt + it;
          ptx::mbar_wait(&q_empty[st], ph ^ 1);
          ptx::mbar_arrive_expect_tx(&q_full[st], 2 * C::T_BYTES + 1024);
#pragma unroll
          for (int c = 0; c < DH / 64; ++c) {
            ptx::tma_load_4d(sQ + st * C::T_BYTES + c * 16384, &tm, &q_full[st], 64 * c, qi * 128, hd, b);
            ptx::tma_load_4d(sdO + st * C::T_BYTES + c * 16384, &tdo, &q_full[st], 64 * c, qi * 128, hd, b);
          }
          bulk_g2s(sLD + st * 256, p.lse + ld_base + qi * 128, 512, &q_full[st]);
          bulk_g2s(sLD + st * 256 + 128, p.Dsum + ld_base + qi * 128, 512, &q_full[st]);
        };
        load_q(0);  // its ring slot frees before the previous item's K/V do
        if (n >= 1) ptx::mbar_wait(kv_empty, (n - 1) & 1);
        ptx::mbar_arrive_expect_tx(kv_full, 2 * C::T_BYTES);
#pragma unroll
        for (int c = 0; c < DH / 64; ++c) {
          ptx::tma_load_4d(sK + c * 16384, &tm, kv_full, 64 * c, kt * 128, p.nh + hd, b);
          ptx::tma_load_4d(sV + c * 16384, &tm, kv_full, 64 * c, kt * 128, 2 * p.nh + hd, b);
        }
        for (int it = 1; it < nq; ++it) load_q(it);
        g += nq;
        ++n;
      }
    }
  } else if (warp == 1) {
    {  // whole warp, converged: every MMA / commit is issued by one elected lane (ptx::*_w)
      // TMEM addresses re-derived from a shuffled (provably warp-uniform) base so
      // the MMA operands live in uniform registers (no per-MMA waterfall loop)
      const uint32_t T_S = __shfl_sync(0xffffffffu, tmem, 0), T_DP = T_S + 128, T_DV = T_S + 256;
      const uint32_t T_DQ = C::DQ_OWN ? T_S + 384 : T_S;
      const uint32_t T_PT = T_S + 448;
      constexpr uint32_t ID_ST = ptx::idesc_bf16(128, 128, 0, 0);  // S^T, dP^T
      constexpr uint32_t ID_DV = ptx::idesc_bf16(128, DH, 0, 1);   // dV, dK
      constexpr uint32_t ID_DQ = ptx::idesc_bf16(128, DH, 1, 1);   // dQ
      const uint32_t ak = ptx::smem_u32(sK), av = ptx::smem_u32(sV);
      const uint32_t apt = ptx::smem_u32(sPT), adst = ptx::smem_u32(sdST);
      BPROF_DECL
      auto issue_st = [&](int gg) {
        const int st = gg % QS, ph = (gg / QS) & 1;
        const uint32_t aq = ptx::smem_u32(sQ + st * C::T_BYTES), ado = ptx::smem_u32(sdO + st * C::T_BYTES);
        BPROF(5, ptx::mbar_wait(&q_full[st], ph));
        if (!C::DQ_OWN && gg >= 1) ptx::mbar_wait(dq_empty, (gg - 1) & 1);  // S^T region holds dQ(gg-1)
        ptx::tc_fence_after();
#pragma unroll
        for (int t = 0; t < DH / 16; ++t) {
          const uint32_t off = (t >> 2) * 16384 + (t & 3) * 32;
          ptx::mma_bf16_w(T_S, ptx::sdesc_sw128(ak + off, 16, 1024), ptx::sdesc_sw128(aq + off, 16, 1024), ID_ST, t > 0);
        }
#pragma unroll
        for (int t = 0; t < DH / 16; ++t) {
          const uint32_t off = (t >> 2) * 16384 + (t & 3) * 32;
          ptx::mma_bf16_w(T_DP, ptx::sdesc_sw128(av + off, 16, 1024), ptx::sdesc_sw128(ado + off, 16, 1024), ID_ST,
                        t > 0);
        }
        ptx::mma_commit_w(s_full);
      };
      int g = 0, n = 0;
      for (int pass = 0; pass * ncta < n_items; ++pass) {
        const int item = snake_item(pass, ncta, cta);
        if (item >= n_items) continue;
        int kt_, hd_, b_;
        decode(item, kt_, hd_, b_);
        const int nq = n_t - kt_;
        BPROF(0, ptx::mbar_wait(kv_full, n & 1));
        // S^T / dP^T TMEM must have been read (dh 64; dh 128: issue_st waits dq_empty)
        if (C::DQ_OWN && g >= 1) ptx::mbar_wait(st_empty, (g - 1) & 1);
        issue_st(g);
        for (int it = 0; it < nq; ++it) {
          const int gg = g + it, st = gg % QS;
          const uint32_t aq = ptx::smem_u32(sQ + st * C::T_BYTES), ado = ptx::smem_u32(sdO + st * C::T_BYTES);
          // scores of the next query tile overlap this tile's softmax-gradient -
          // if its Q / dO tile has landed; otherwise this tile's dV/dK/dQ go first
          // (blocking on the load here would stall the whole chain)
          bool st_next = false;
          if (C::DQ_OWN && it + 1 < nq) {
            BPROF(1, ptx::mbar_wait(st_empty, gg & 1));
            const int sn = (gg + 1) % QS;
            const bool landed = __shfl_sync(0xffffffffu, (int)ptx::mbar_test(&q_full[sn], ((gg + 1) / QS) & 1), 0);
            if (landed) {  // warp-uniform decision
              issue_st(gg + 1);
              st_next = true;
            }
          }
          BPROF(2, ptx::mbar_wait(p_full, gg & 1));
          if (it == 0 && n >= 1) BPROF(3, ptx::mbar_wait(acc_empty, (n - 1) & 1));  // previous item's dV/dK read out
          ptx::tc_fence_after();
          if (C::PT_TMEM) {
            const uint32_t ads = ptx::smem_u32(sdS_buf[gg & 1]);
#pragma unroll
            for (int t = 0; t < 128 / 16; ++t)  // dV += P^T dO, P^T from TMEM (8 columns per 16 queries)
              ptx::mma_bf16_ts_w(T_DV, T_PT + 8 * t, ptx::sdesc_sw128(ado + t * 2048, 16384, 1024), ID_DV,
                               (it > 0 || t > 0) ? 1u : 0u);
            ptx::mma_commit_w(pt_free);
#pragma unroll
            for (int t = 0; t < 128 / 16; ++t) {  // dK += dS^T Q
              const uint32_t offa = (t >> 2) * 16384 + (t & 3) * 32;
              ptx::mma_bf16_w(T_DV + DH, ptx::sdesc_sw128(ads + offa, 16, 1024), ptx::sdesc_sw128(aq + t * 2048, 16384, 1024),
                            ID_DV, (it > 0 || t > 0) ? 1u : 0u);
            }
            ptx::mma_commit_w(&q_empty[st]);  // last reads of Q / dO (dQ needs only dS and K): refill the slot now
            if (gg >= 1) BPROF(4, ptx::mbar_wait(dq_empty, (gg - 1) & 1));  // dQ(gg-1) read out
#pragma unroll
            for (int t = 0; t < 128 / 16; ++t)  // K = 128 keys: dQ = dS K
              ptx::mma_bf16_w(T_DQ, ptx::sdesc_sw128(ads + t * 2048, 16384, 1024),
                            ptx::sdesc_sw128(ak + t * 2048, 16384, 1024), ID_DQ, t > 0);
          } else {
#pragma unroll
            for (int t = 0; t < 128 / 16; ++t) {  // K = 128 queries
              const uint32_t offa = (t >> 2) * 16384 + (t & 3) * 32;
              ptx::mma_bf16_w(T_DV, ptx::sdesc_sw128(apt + offa, 16, 1024), ptx::sdesc_sw128(ado + t * 2048, 16384, 1024),
                            ID_DV, (it > 0 || t > 0) ? 1u : 0u);  // dV += P^T dO
              ptx::mma_bf16_w(T_DV + DH, ptx::sdesc_sw128(adst + offa, 16, 1024),
                            ptx::sdesc_sw128(aq + t * 2048, 16384, 1024), ID_DV, (it > 0 || t > 0) ? 1u : 0u);  // dK += dS^T Q
            }
            ptx::mma_commit_w(&q_empty[st]);  // last reads of Q / dO
            if (C::DQ_OWN && gg >= 1) ptx::mbar_wait(dq_empty, (gg - 1) & 1);  // dQ(gg-1) read out
#pragma unroll
            for (int t = 0; t < 128 / 16; ++t)  // K = 128 keys: dQ = dS K
              ptx::mma_bf16_w(T_DQ, ptx::sdesc_sw128(adst + t * 2048, 16384, 1024),
                            ptx::sdesc_sw128(ak + t * 2048, 16384, 1024), ID_DQ, t > 0);
          }
          ptx::mma_commit_w(mm_done);
          if (C::DQ_OWN && it + 1 < nq && !st_next) issue_st(gg + 1);
          if (!C::DQ_OWN && it + 1 < nq) issue_st(gg + 1);
        }
        ptx::mma_commit_w(kv_empty);
        g += nq;
        ++n;
      }
      BPROF_DUMP("bmma")
    }
  } else {
    // ---------------------------------------- softmax-gradient warps
    // 4 CP warps: (lane quadrant q4, column part cq); thread = key row r,
    // query columns [QC cq, QC cq + QC); dQ columns [DC cq, DC cq + DC)
    constexpr int NSW = 4 * CP, QC = 128 / CP, NG = QC / 32, DC = DH / CP;
    static_assert(CP == 2 || (DH == 64 && CP == 4), "CP 4 only at dh 64");
    const int q4 = warp & 3;
    const int cq = (warp - 2) >> 2;
    const int r = q4 * 32 + lane;  // key row of this thread (TMEM lane)
    const uint32_t lane_base = (uint32_t)(q4 * 32) << 16;
    const uint32_t spt = ptx::smem_u32(sPT);
    // dQ (TMEM lane = query row) -> fp32 staging [DH/32 slabs][128 rows][128 B],
    // 16-byte chunks XOR-swizzled by row (TMA SWIZZLE_128B, conflict-free
    // stores) -> one TMA reduce-add per 32-column slab into the dQ buffer
    // The reduce is not waited for here: the staging memory is next written
    // one query tile later (stage_free() before that write), by which time
    // the bulk copy has long finished reading it - so no warp stalls on it.
    auto stage_free = [&]() {
      if (warp == 2 && lane == 0) asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
      named_bar(1, 32 * NSW);
    };
    auto dq_drain = [&](int qiq, int hd, int b, uint32_t stg) {
      if constexpr (DC == 16) {  // a quarter of a 32-column slab: chunks (cq % 2) * 4 .. +3 of slab cq / 2
        uint32_t v[16];
        __syncwarp();
        ptx::tmem_ld16(T_DQ + cq * 16 + lane_base, v);
        ptx::tmem_ld_wait();
        ptx::tc_fence_before();
        __syncwarp();
        if (lane == 0) ptx::mbar_arrive(dq_empty);  // dQ TMEM may be overwritten
        stage_free();
        const int c = cq >> 1;
#pragma unroll
        for (int k = 0; k < 4; ++k)
          st_shared_v4(stg + c * 16384 + r * 128 + ((((cq & 1) * 4 + k) ^ (r & 7)) << 4), v[4 * k], v[4 * k + 1],
                       v[4 * k + 2], v[4 * k + 3]);
      } else {
      uint32_t v[DC / 32][32];
#pragma unroll
      for (int cc = 0; cc < DC / 32; ++cc) {
        const int c = cq * (DC / 32) + cc;  // 32-column slab
        __syncwarp();
        ptx::tmem_ld32(T_DQ + c * 32 + lane_base, v[cc]);
      }
      ptx::tmem_ld_wait();
      ptx::tc_fence_before();
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive(dq_empty);  // dQ TMEM may be overwritten
      if (C::DQ_OWN) stage_free();                 // dh 128: done before the P^T / dS^T writes
#pragma unroll
      for (int cc = 0; cc < DC / 32; ++cc) {
        const int c = cq * (DC / 32) + cc;
#pragma unroll
        for (int k = 0; k < 8; ++k)
          st_shared_v4(stg + c * 16384 + r * 128 + ((k ^ (r & 7)) << 4), v[cc][4 * k], v[cc][4 * k + 1],
                       v[cc][4 * k + 2], v[cc][4 * k + 3]);
      }
      }
      ptx::fence_proxy_async();
      named_bar(1, 32 * NSW);
      if (warp == 2 && lane == 0) {
#pragma unroll
        for (int c = 0; c < DH / 32; ++c)
          asm volatile(
              "cp.reduce.async.bulk.tensor.4d.global.shared::cta.add.tile.bulk_group [%0, {%2, %3, %4, %5}], [%1];" ::"l"(
                  reinterpret_cast<uint64_t>(&tdq)),
              "r"(stg + c * 16384), "r"(c * 32), "r"(qiq * 128), "r"(hd), "r"(b)
              : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      }
    };
    int g = 0, n = 0;
    BPROF_DECL
    for (int pass = 0; pass * ncta < n_items; ++pass) {
      const int item = snake_item(pass, ncta, cta);
      if (item >= n_items) continue;
      int kt, hd, b;
      decode(item, kt, hd, b);
      const int nq = n_t - kt;
      for (int it = 0; it < nq; ++it) {
#ifdef MOBIUS_BWD_PROF
        long long tb = clock64();
#endif
        const int gg = g + it, st = gg % QS;
        const int qi = kt + it;
        const bool diag = (it == 0);
        ptx::mbar_wait(&q_full[st], (gg / QS) & 1);  // lse / D of this query tile in smem
        ptx::mbar_wait(s_full, gg & 1);
        ptx::tc_fence_after();
#ifdef MOBIUS_BWD_PROF
        bprof[0] += clock64() - tb; tb = clock64();
#endif
        uint32_t vs[NG][32], vd[NG][32];
        __syncwarp();
#pragma unroll
        for (int cc = 0; cc < NG; ++cc) {
          ptx::tmem_ld32(T_S + cq * QC + cc * 32 + lane_base, vs[cc]);
          ptx::tmem_ld32(T_DP + cq * QC + cc * 32 + lane_base, vd[cc]);
        }
        ptx::tmem_ld_wait();
        ptx::tc_fence_before();
        __syncwarp();
        if (lane == 0) ptx::mbar_arrive(st_empty);  // S^T / dP^T TMEM may be overwritten
#ifdef MOBIUS_BWD_PROF
        bprof[1] += clock64() - tb; tb = clock64();
#endif
        // P^T / dS^T smem must be free: dh 128 - the previous tile's dQ drain
        // (staged there) completed; dh 64 - the previous tile's MMAs completed
        if (C::PT_TMEM) {
          // P^T (TMEM) free once the dV MMAs of the previous tile completed;
          // dS^T buffer gg&1 was last read by the MMAs of tile gg-2, whose
          // completion the dQ drain of tile gg-2 already waited for
          if (gg >= 1) {
            ptx::mbar_wait(pt_free, (gg - 1) & 1);
            ptx::tc_fence_after();
          }
        } else if (C::DQ_OWN && gg >= 1) {
          ptx::mbar_wait(mm_done, (gg - 1) & 1);
          ptx::tc_fence_after();
        }
        if (!C::DQ_OWN && gg >= 1) stage_free();  // dQ(gg-1) staged in P^T / dS^T: reduce must have read it
        if (C::DQ_OWN && it == 0 && gg >= 1) stage_free();  // previous item's dV/dK stores read the P^T / dS^T tiles
#ifdef MOBIUS_BWD_PROF
        bprof[2] += clock64() - tb; tb = clock64();
#endif
        const uint32_t sds = ptx::smem_u32(sdS_buf[C::PT_TMEM ? (gg & 1) : 0]);
#pragma unroll
        for (int cc = 0; cc < NG; ++cc) {
          const int c = cq * NG + cc;  // 32-query slab
          uint32_t ppk[16], dpk[16];
          const uint32_t aL = ptx::smem_u32(sLD + st * 256 + c * 32);
          if (diag)
            bwd_slab_math<true>(vs[cc], vd[cc], aL, c * 32, r, p.scale_log2, ppk, dpk);
          else
            bwd_slab_math<false>(vs[cc], vd[cc], aL, c * 32, r, p.scale_log2, ppk, dpk);
          if (C::PT_TMEM) {  // P^T row r, queries c*32.. -> TMEM columns (2 bf16 per column)
            ptx::tmem_st16(T_PT + c * 16 + lane_base, ppk);
#pragma unroll
            for (int k = 0; k < 4; ++k)
              st_shared_v4(sds + sw128_off(r, c * 4 + k), dpk[4 * k], dpk[4 * k + 1], dpk[4 * k + 2], dpk[4 * k + 3]);
          } else {
#pragma unroll
            for (int k = 0; k < 4; ++k) {
              const uint32_t o = sw128_off(r, c * 4 + k);
              st_shared_v4(spt + o, ppk[4 * k], ppk[4 * k + 1], ppk[4 * k + 2], ppk[4 * k + 3]);
              st_shared_v4(sds + o, dpk[4 * k], dpk[4 * k + 1], dpk[4 * k + 2], dpk[4 * k + 3]);
            }
          }
        }
        if (C::PT_TMEM) ptx::tmem_st_wait();
        ptx::tc_fence_before();
        ptx::fence_proxy_async();
        __syncwarp();
        if (lane == 0) ptx::mbar_arrive(p_full);
#ifdef MOBIUS_BWD_PROF
        bprof[3] += clock64() - tb; tb = clock64();
#endif
        if (C::DQ_OWN) {
          // drain dQ of the previous query tile of this item while this tile's MMAs run
          if (it >= 1) {
            if (C::PT_TMEM) {
              ptx::mbar_wait(mm_done, (gg - 1) & 1);
              ptx::tc_fence_after();
            }
            dq_drain(qi - 1, hd, b, ptx::smem_u32(sSTG));
          }
        } else {
          ptx::mbar_wait(mm_done, gg & 1);
          ptx::tc_fence_after();
          dq_drain(qi, hd, b, spt);  // staged in the (now free) P^T / dS^T tiles
        }
#ifdef MOBIUS_BWD_PROF
        bprof[4] += clock64() - tb;
#endif
      }
#ifdef MOBIUS_BWD_PROF
      long long tb2 = clock64();
#endif
      const int glast = g + nq - 1;
      ptx::mbar_wait(mm_done, glast & 1);
      ptx::tc_fence_after();
      if (C::DQ_OWN)
        dq_drain(kt + nq - 1, hd, b, ptx::smem_u32(sSTG));
      else
        stage_free();  // dh 128: the last dQ was staged in the P^T / dS^T tiles
      // dV (half 0) / dK (half 1) of this key tile (rows = keys), bf16, staged
      // 128B-swizzled in the (now idle) P^T / dS^T tiles and written by two
      // TMA stores per tensor atom (row-per-thread global stores are 64 B
      // pieces 3h apart); the next item's first P^T / dS^T write waits for
      // the stores' smem reads (stage_free)
      // warp (q4, cq): tensor tv = cq / (CP/2) (0 dV, 1 dK), its 32-column chunks
      // [(cq % (CP/2)) * NCH, + NCH) of the DH / 32
      constexpr int HP = CP / 2, NCH = DH / 32 / HP;
      const int tv = cq / HP, ch0 = (cq % HP) * NCH;
      const uint32_t stg = ptx::smem_u32(sPT) + tv * (DH / 64) * 16384;
#pragma unroll
      for (int ci = 0; ci < NCH; ++ci) {
        const int c = ch0 + ci;
        uint32_t v[32];
        __syncwarp();
        ptx::tmem_ld32(T_DV + tv * DH + c * 32 + lane_base, v);
        ptx::tmem_ld_wait();
        if (ci == NCH - 1) {  // last TMEM read of this item's accumulators by this warp
          ptx::tc_fence_before();
          __syncwarp();
          if (lane == 0) ptx::mbar_arrive(acc_empty);
        }
        uint32_t pk[16];
        const float f = tv == 0 ? 1.f : p.scale;  // dK = scale * sum dS^T Q (dS^T was stored unscaled)
#pragma unroll
        for (int e = 0; e < 32; e += 2)
          pk[e / 2] = pack_bf16x2(__fmul2_rn(make_float2(__uint_as_float(v[e]), __uint_as_float(v[e + 1])), make_float2(f, f)));
#pragma unroll
        for (int k = 0; k < 4; ++k)
          st_shared_v4(stg + sw128_off(r, c * 4 + k), pk[4 * k], pk[4 * k + 1], pk[4 * k + 2], pk[4 * k + 3]);
      }
      ptx::fence_proxy_async();
      named_bar(1, 32 * NSW);
      if (warp == 2 && lane == 0) {
#pragma unroll
        for (int t = 0; t < 2; ++t)
#pragma unroll
          for (int a = 0; a < DH / 64; ++a)
            asm volatile("cp.async.bulk.tensor.4d.global.shared::cta.bulk_group [%0, {%2, %3, %4, %5}], [%1];" ::"l"(
                             reinterpret_cast<uint64_t>(&tdkv)),
                         "r"(ptx::smem_u32(sPT) + (t * (DH / 64) + a) * 16384), "r"(64 * a), "r"(kt * 128),
                         "r"((t == 0 ? 2 * p.nh : p.nh) + hd), "r"(b)
                         : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      }
#ifdef MOBIUS_BWD_PROF
      bprof[5] += clock64() - tb2;
#endif
      g += nq;
      ++n;
    }
    BPROF_DUMP("bsmx")
    if (warp == 2 && lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");  // last dQ reduce
    ptx::tc_fence_before();
  }
  __syncthreads();
  if (warp == 1) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc<512>(tmem);
  }
}

// ---------------------------------------------------------------- bwd, dh 64
// Warp-specialised backward for dh 64 (the 1.5B shape), 16 warps:
//   warp 0      TMA: K / V of an item into one of two slots (the next
//               item's K / V land while the current item runs), Q / dO /
//               lse / -D of each query tile through a 3-deep ring
//   warp 1      MMA: S^T = K Q^T and dP^T = V dO^T (TMEM), dV += P^T dO
//               (TS: P^T from TMEM), dK += dS^T Q, dQ = dS K (TMEM); the
//               scores of the next query tile - also across an item boundary
//               - are issued as soon as the softmax-gradient warps hold the
//               current ones in registers
//   warps 2, 3  idle
//   warps 4-11  softmax-gradient: thread = key row, 64 query columns;
//               P^T -> TMEM (hands dV its operand at once), dS^T kept in
//               registers and written to the single smem dS^T tile once the
//               previous tile's dK / dQ MMAs have read it
//   warps 12-15 drain: dQ of each tile (TMEM -> 16-column fp32 slabs,
//               SWIZZLE_64B, through a 3-slot 8 KB staging ring -> TMA
//               reduce-add) and dV / dK of each item (TMEM -> bf16 -> 64-row
//               halves -> TMA store), off the softmax warps' path
// setmaxnreg re-splits the register file per warpgroup: 56 / 176 / 176 / 104.
#ifndef MOBIUS_BWD_QS
#define MOBIUS_BWD_QS 3
#endif
#ifndef MOBIUS_BWD_SLAB32
#define MOBIUS_BWD_SLAB32 0
#endif
struct Bwd64Cfg {
  static constexpr int T_BYTES = 128 * 64 * 2;  // one K / V / Q / dO tile (16 KB)
  static constexpr int QS = MOBIUS_BWD_QS;      // Q / dO ring depth
  static constexpr int DS_BYTES = 128 * 128 * 2;
  // drain staging ring: 8 KB slots (an fp32 16-column dQ slab or 64 rows of
  // a bf16 dV / dK tile), or with MOBIUS_BWD_SLAB32 16 KB slots of 32-column slabs
  static constexpr int SLOT = MOBIUS_BWD_SLAB32 ? 16384 : 8192;
  static constexpr int NSTG = MOBIUS_BWD_SLAB32 ? 2 : 3;
  static constexpr int STG_BYTES = NSTG * SLOT;
  static constexpr int SMEM = 1024 + 4 * T_BYTES + QS * 2 * T_BYTES + DS_BYTES + STG_BYTES + QS * 1024 + 256;
};

__global__ void __launch_bounds__(512, 1) flash_bwd64_kernel(const __grid_constant__ CUtensorMap tm,
                                                          const __grid_constant__ CUtensorMap tdo,
                                                          const __grid_constant__ CUtensorMap tdq,
                                                          const __grid_constant__ CUtensorMap tdkv, const BwdParams p) {
  using C = Bwd64Cfg;
  constexpr int QS = C::QS, DH = 64;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sK = smem;                         // [2]
  uint8_t* sV = sK + 2 * C::T_BYTES;          // [2]
  uint8_t* sQ = sV + 2 * C::T_BYTES;          // [QS]
  uint8_t* sdO = sQ + QS * C::T_BYTES;        // [QS]
  uint8_t* sdS = sdO + QS * C::T_BYTES;       // dS^T (keys x queries, K-major SW128 atoms)
  uint8_t* sSTG = sdS + C::DS_BYTES;          // drain staging
  float* sLD = reinterpret_cast<float*>(sSTG + C::STG_BYTES);  // [QS][lse 128 | -D 128]
  uint64_t* bars = reinterpret_cast<uint64_t*>(sLD + QS * 256);
  uint64_t* kv_full = bars;             // [2]
  uint64_t* kv_empty = bars + 2;        // [2] every MMA of the slot's item done
  uint64_t* q_full = bars + 4;          // [QS] Q, dO, lse, -D
  uint64_t* q_empty = bars + 4 + QS;    // [QS]
  uint64_t* s_full = bars + 4 + 2 * QS;  // S^T and dP^T in TMEM
  uint64_t* st_empty = s_full + 1;       // S^T / dP^T in registers (count 8)
  uint64_t* pt_full = s_full + 2;        // P^T in TMEM (count 8)
  uint64_t* ds_full = s_full + 3;        // dS^T in smem (count 8)
  uint64_t* pt_free = s_full + 4;        // dV MMAs done: P^T TMEM may be overwritten
  uint64_t* mm_done = s_full + 5;        // [2] dV/dK/dQ of tile g done ([g & 1])
  uint64_t* dq_empty = s_full + 7;       // dQ read out of TMEM (count 4)
  uint64_t* acc_empty = s_full + 8;      // dV / dK of an item read out of TMEM (count 4)
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(s_full + 9);
  auto mm_wait = [&](int t) { ptx::mbar_wait(&mm_done[t & 1], (t >> 1) & 1); };

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int n_t = p.s / 128;
  const int nbh = p.nh * p.mbs;
  const int n_items = n_t * nbh;
  const int ncta = (int)gridDim.x, cta = (int)blockIdx.x;
  auto decode = [&](int item, int& kt, int& hd, int& b) {
    int r;
    chunked_item(item, n_t, nbh, p.group, kt, r);
    hd = r % p.nh;
    b = r / p.nh;
  };

  if (threadIdx.x == 0) {
    ptx::tma_prefetch_desc(&tm);
    ptx::tma_prefetch_desc(&tdo);
    ptx::tma_prefetch_desc(&tdq);
    ptx::tma_prefetch_desc(&tdkv);
    for (int i = 0; i < 2; ++i) {
      ptx::mbar_init(&kv_full[i], 1);
      ptx::mbar_init(&kv_empty[i], 1);
      ptx::mbar_init(&mm_done[i], 1);
    }
    for (int i = 0; i < QS; ++i) {
      ptx::mbar_init(&q_full[i], 1);
      ptx::mbar_init(&q_empty[i], 1);
    }
    ptx::mbar_init(s_full, 1);
    ptx::mbar_init(st_empty, 8);
    ptx::mbar_init(pt_full, 8);
    ptx::mbar_init(ds_full, 8);
    ptx::mbar_init(pt_free, 1);
    ptx::mbar_init(dq_empty, 4);
    ptx::mbar_init(acc_empty, 4);
    ptx::fence_mbar_init();
  }
  if (warp == 1) ptx::tmem_alloc<512>(tmem_slot);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  // TMEM: S^T 0..127, dP^T 128..255, dV 256..319, dK 320..383, dQ 384..447, P^T 448..511 (packed bf16)

  if (warp == 0) {
    asm volatile("setmaxnreg.dec.sync.aligned.u32 56;");
    if (lane == 0) {
      int g = 0, n = 0;
      for (int pass = 0; pass * ncta < n_items; ++pass) {
        const int item = snake_item(pass, ncta, cta);
        if (item >= n_items) continue;
        int kt, hd, b;
        decode(item, kt, hd, b);
        const int nq = n_t - kt;
        const int64_t ld_base = ((int64_t)b * p.nh + hd) * p.s;
        auto load_q = [&](int it) {
          const int gg = g + it, st = gg % QS, ph = (gg / QS) & 1, qi = kt + it;
          ptx::mbar_wait(&q_empty[st], ph ^ 1);
          ptx::mbar_arrive_expect_tx(&q_full[st], 2 * C::T_BYTES + 1024);
          ptx::tma_load_4d(sQ + st * C::T_BYTES, &tm, &q_full[st], 0, qi * 128, hd, b);
          ptx::tma_load_4d(sdO + st * C::T_BYTES, &tdo, &q_full[st], 0, qi * 128, hd, b);
          bulk_g2s(sLD + st * 256, p.lse + ld_base + qi * 128, 512, &q_full[st]);
          bulk_g2s(sLD + st * 256 + 128, p.Dsum + ld_base + qi * 128, 512, &q_full[st]);
        };
        load_q(0);
        const int kvs = n & 1;
        ptx::mbar_wait(&kv_empty[kvs], ((n >> 1) & 1) ^ 1);  // item n - 2 done with the slot
        ptx::mbar_arrive_expect_tx(&kv_full[kvs], 2 * C::T_BYTES);
        ptx::tma_load_4d(sK + kvs * C::T_BYTES, &tm, &kv_full[kvs], 0, kt * 128, p.nh + hd, b);
        ptx::tma_load_4d(sV + kvs * C::T_BYTES, &tm, &kv_full[kvs], 0, kt * 128, 2 * p.nh + hd, b);
        for (int it = 1; it < nq; ++it) load_q(it);
        g += nq;
        ++n;
      }
    }
  } else if (warp == 1) {
    asm volatile("setmaxnreg.dec.sync.aligned.u32 56;");
    const uint32_t T_S = __shfl_sync(0xffffffffu, tmem, 0), T_DP = T_S + 128, T_DV = T_S + 256;
    const uint32_t T_DK = T_S + 320, T_DQ = T_S + 384, T_PT = T_S + 448;
    constexpr uint32_t ID_ST = ptx::idesc_bf16(128, 128, 0, 0);  // S^T, dP^T
    constexpr uint32_t ID_DV = ptx::idesc_bf16(128, DH, 0, 1);   // dV, dK
    constexpr uint32_t ID_DQ = ptx::idesc_bf16(128, DH, 1, 1);   // dQ
    const uint32_t ads = ptx::smem_u32(sdS);
    BPROF_DECL
    auto issue_st = [&](int gg, int kvs) {
      const int st = gg % QS;
      const uint32_t aq = ptx::smem_u32(sQ + st * C::T_BYTES), ado = ptx::smem_u32(sdO + st * C::T_BYTES);
      const uint32_t ak = ptx::smem_u32(sK + kvs * C::T_BYTES), av = ptx::smem_u32(sV + kvs * C::T_BYTES);
      ptx::tc_fence_after();
#pragma unroll
      for (int t = 0; t < DH / 16; ++t)
        ptx::mma_bf16_w(T_S, ptx::sdesc_sw128(ak + t * 32, 16, 1024), ptx::sdesc_sw128(aq + t * 32, 16, 1024), ID_ST, t > 0);
#pragma unroll
      for (int t = 0; t < DH / 16; ++t)
        ptx::mma_bf16_w(T_DP, ptx::sdesc_sw128(av + t * 32, 16, 1024), ptx::sdesc_sw128(ado + t * 32, 16, 1024), ID_ST,
                        t > 0);
      ptx::mma_commit_w(s_full);
    };
    auto landed = [&](uint64_t* bar, uint32_t ph) {  // warp-uniform non-blocking test
      return __shfl_sync(0xffffffffu, (int)ptx::mbar_test(bar, ph), 0) != 0;
    };
    int g = 0, n = 0;
    bool pre = false;  // the current item's first scores were issued during the previous item
    for (int pass = 0; pass * ncta < n_items; ++pass) {
      const int item = snake_item(pass, ncta, cta);
      if (item >= n_items) continue;
      int kt_, hd_, b_;
      decode(item, kt_, hd_, b_);
      const int nq = n_t - kt_, kvs = n & 1;
      const bool has_next = snake_item(pass + 1, ncta, cta) < n_items;
      const uint32_t ak = ptx::smem_u32(sK + kvs * C::T_BYTES);
      if (!pre) {
        BPROF(0, ptx::mbar_wait(&kv_full[kvs], (n >> 1) & 1));
        BPROF(5, ptx::mbar_wait(&q_full[g % QS], (g / QS) & 1));
        if (g >= 1) ptx::mbar_wait(st_empty, (g - 1) & 1);
        issue_st(g, kvs);
      }
      pre = false;
      for (int it = 0; it < nq; ++it) {
        const int gg = g + it, st = gg % QS;
        const uint32_t aq = ptx::smem_u32(sQ + st * C::T_BYTES), ado = ptx::smem_u32(sdO + st * C::T_BYTES);
        // scores of the next query tile (of this item, or the next item's
        // first) overlap this tile's softmax gradient if their operands landed
        BPROF(1, ptx::mbar_wait(st_empty, gg & 1));
        const int sn = (gg + 1) % QS;
        const uint32_t qph = ((gg + 1) / QS) & 1;
        bool next_done = false;
        if (it + 1 < nq) {
          if (landed(&q_full[sn], qph)) {
            issue_st(gg + 1, kvs);
            next_done = true;
          }
        } else if (has_next) {
          if (landed(&kv_full[kvs ^ 1], ((n + 1) >> 1) & 1) && landed(&q_full[sn], qph)) {
            issue_st(gg + 1, kvs ^ 1);
            pre = true;
          }
        }
        BPROF(2, ptx::mbar_wait(pt_full, gg & 1));
        if (it == 0 && n >= 1) BPROF(3, ptx::mbar_wait(acc_empty, (n - 1) & 1));  // previous item's dV/dK read out
        ptx::tc_fence_after();
#pragma unroll
        for (int t = 0; t < 128 / 16; ++t)  // dV += P^T dO, P^T from TMEM (8 columns per 16 queries)
          ptx::mma_bf16_ts_w(T_DV, T_PT + 8 * t, ptx::sdesc_sw128(ado + t * 2048, 16384, 1024), ID_DV,
                             (it > 0 || t > 0) ? 1u : 0u);
        ptx::mma_commit_w(pt_free);
        BPROF(6, ptx::mbar_wait(ds_full, gg & 1));
        ptx::tc_fence_after();
#pragma unroll
        for (int t = 0; t < 128 / 16; ++t) {  // dK += dS^T Q
          const uint32_t offa = (t >> 2) * 16384 + (t & 3) * 32;
          ptx::mma_bf16_w(T_DK, ptx::sdesc_sw128(ads + offa, 16, 1024), ptx::sdesc_sw128(aq + t * 2048, 16384, 1024),
                          ID_DV, (it > 0 || t > 0) ? 1u : 0u);
        }
        ptx::mma_commit_w(&q_empty[st]);  // last reads of Q / dO / lse / -D
        if (gg >= 1) BPROF(4, ptx::mbar_wait(dq_empty, (gg - 1) & 1));  // dQ(gg-1) read out
        ptx::tc_fence_after();
#pragma unroll
        for (int t = 0; t < 128 / 16; ++t)  // dQ = dS K (K = 128 keys)
          ptx::mma_bf16_w(T_DQ, ptx::sdesc_sw128(ads + t * 2048, 16384, 1024), ptx::sdesc_sw128(ak + t * 2048, 16384, 1024),
                          ID_DQ, t > 0);
        ptx::mma_commit_w(&mm_done[gg & 1]);
        if (it + 1 < nq && !next_done) {
          BPROF(5, ptx::mbar_wait(&q_full[sn], qph));
          issue_st(gg + 1, kvs);
        }
      }
      ptx::mma_commit_w(&kv_empty[kvs]);
      g += nq;
      ++n;
    }
    BPROF_DUMP("bmma")
  } else if (warp < 4) {
    asm volatile("setmaxnreg.dec.sync.aligned.u32 56;");  // idle
  } else if (warp < 12) {
    asm volatile("setmaxnreg.inc.sync.aligned.u32 176;");
    // ---------------------------------------- softmax-gradient warps
    // (lane quadrant q4, column half cq); thread = key row r, queries [64 cq, 64 cq + 64)
    const int q4 = warp & 3, cq = (warp - 4) >> 2;
    const int r = q4 * 32 + lane;
    const uint32_t lane_base = (uint32_t)(q4 * 32) << 16;
    const uint32_t T_S = tmem + lane_base, T_DP = T_S + 128, T_PT = T_S + 448;
    const uint32_t sds = ptx::smem_u32(sdS);
    int g = 0;
    BPROF_DECL
    for (int pass = 0; pass * ncta < n_items; ++pass) {
      const int item = snake_item(pass, ncta, cta);
      if (item >= n_items) continue;
      int kt, hd, b;
      decode(item, kt, hd, b);
      const int nq = n_t - kt;
      for (int it = 0; it < nq; ++it) {
        const int gg = g + it, st = gg % QS;
        BPROF(0, ptx::mbar_wait(&q_full[st], (gg / QS) & 1); ptx::mbar_wait(s_full, gg & 1));
        ptx::tc_fence_after();
        uint32_t vs[2][32], vd[2][32];
        __syncwarp();
#pragma unroll
        for (int cc = 0; cc < 2; ++cc) {
          ptx::tmem_ld32(T_S + cq * 64 + cc * 32, vs[cc]);
          ptx::tmem_ld32(T_DP + cq * 64 + cc * 32, vd[cc]);
        }
        ptx::tmem_ld_wait();
        ptx::tc_fence_before();
        __syncwarp();
        if (lane == 0) ptx::mbar_arrive(st_empty);  // S^T / dP^T TMEM may be overwritten
        if (gg >= 1) BPROF(1, ptx::mbar_wait(pt_free, (gg - 1) & 1));  // dV(gg-1) read P^T
        ptx::tc_fence_after();
        uint32_t dpk[2][16];
#ifdef MOBIUS_BWD_PROF
        long long tm0 = clock64();
#endif
#pragma unroll
          for (int cc = 0; cc < 2; ++cc) {
            const int c = cq * 2 + cc;  // 32-query slab
            uint32_t ppk[16];
            const uint32_t aL = ptx::smem_u32(sLD + st * 256 + c * 32);
#if MOBIUS_BWD_MATH
            if (it == 0)
              bwd_slab_math_pl<true>(vs[cc], vd[cc], aL, c * 32, r, p.scale_log2, ppk, dpk[cc]);
            else
              bwd_slab_math_pl<false>(vs[cc], vd[cc], aL, c * 32, r, p.scale_log2, ppk, dpk[cc]);
#else
            if (it == 0)
              bwd_slab_math<true>(vs[cc], vd[cc], aL, c * 32, r, p.scale_log2, ppk, dpk[cc]);
            else
              bwd_slab_math<false>(vs[cc], vd[cc], aL, c * 32, r, p.scale_log2, ppk, dpk[cc]);
#endif
            ptx::tmem_st16(T_PT + c * 16, ppk);  // P^T row r, queries c*32.. (2 bf16 per column)
          }
          ptx::tmem_st_wait();
#ifdef MOBIUS_BWD_PROF
        bprof[2] += clock64() - tm0;
#endif
        ptx::tc_fence_before();
        __syncwarp();
        if (lane == 0) ptx::mbar_arrive(pt_full);
        // the single dS^T tile is free once dK / dQ of the previous tile completed
        if (gg >= 1) BPROF(3, mm_wait(gg - 1));
        ptx::tc_fence_after();
#pragma unroll
        for (int cc = 0; cc < 2; ++cc)
#pragma unroll
          for (int k = 0; k < 4; ++k)
            st_shared_v4(sds + sw128_off(r, (cq * 2 + cc) * 4 + k), dpk[cc][4 * k], dpk[cc][4 * k + 1], dpk[cc][4 * k + 2],
                         dpk[cc][4 * k + 3]);
        ptx::fence_proxy_async();
        __syncwarp();
        if (lane == 0) ptx::mbar_arrive(ds_full);
      }
      g += nq;
    }
    BPROF_DUMP("bsmx")
  } else {
    asm volatile("setmaxnreg.dec.sync.aligned.u32 104;");
    // ---------------------------------------- drain warpgroup
    // thread = TMEM lane r: dQ row r of each query tile as soon as its MMAs
    // complete -> four fp32 16-column slabs [128 rows][64 B], 16-byte chunks
    // XOR-swizzled (TMA SWIZZLE_64B) -> TMA reduce-add into the dQ
    // accumulator; at an item's last tile, before its dQ, dV / dK (rows =
    // keys) -> bf16 -> 64-row halves (SWIZZLE_128B) -> TMA stores.  Every
    // slab goes through a ring of NSTG 8 KB staging slots, one bulk group
    // each: a slot is rewritten once at most NSTG - 1 later groups are
    // still reading (the TMA engine reads a 16 KB reduce slab in ~700
    // cycles, so waiting for the previous one serialised the drain).
    const int q4 = warp & 3;
    const int r = q4 * 32 + lane;
    const uint32_t lane_base = (uint32_t)(q4 * 32) << 16;
    const uint32_t T_DV = tmem + lane_base + 256, T_DQ = tmem + lane_base + 384;
    const bool leader = warp == 12 && lane == 0;
    const uint32_t stg0 = ptx::smem_u32(sSTG);
    int ks = 0;  // staged slabs so far
    auto slot_acquire = [&]() -> uint32_t {
      if (leader) asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(C::NSTG - 1) : "memory");
      named_bar(1, 128);
      return stg0 + (ks % C::NSTG) * C::SLOT;
    };
    auto slot_done = [&]() {  // staging written: hand it to the async proxy
      ptx::fence_proxy_async();
      named_bar(1, 128);
      ++ks;
    };
    int g = 0;
    BPROF_DECL
    for (int pass = 0; pass * ncta < n_items; ++pass) {
      const int item = snake_item(pass, ncta, cta);
      if (item >= n_items) continue;
      int kt, hd, b;
      decode(item, kt, hd, b);
      const int nq = n_t - kt;
      for (int it = 0; it < nq; ++it) {
        const int gg = g + it;
        BPROF(0, mm_wait(gg));
        ptx::tc_fence_after();
        if (it == nq - 1) {
          // the item's dV / dK accumulators are final: read them out of TMEM
          // first (the next item's first dV MMA waits for acc_empty), keep
          // them packed bf16 (64 registers), then stage and TMA-store them
          uint32_t pk[2][32];
#pragma unroll
          for (int tv = 0; tv < 2; ++tv) {
            const float f = tv == 0 ? 1.f : p.scale;  // dK = scale * sum dS^T Q (dS^T was stored unscaled)
#pragma unroll
            for (int c = 0; c < 2; ++c) {
              uint32_t v[32];
              __syncwarp();
              ptx::tmem_ld32(T_DV + tv * DH + c * 32, v);
              ptx::tmem_ld_wait();
#pragma unroll
              for (int e = 0; e < 32; e += 2)
                pk[tv][c * 16 + e / 2] = pack_bf16x2(
                    __fmul2_rn(make_float2(__uint_as_float(v[e]), __uint_as_float(v[e + 1])), make_float2(f, f)));
            }
          }
          ptx::tc_fence_before();
          __syncwarp();
          if (lane == 0) ptx::mbar_arrive(acc_empty);
#pragma unroll
          for (int tv = 0; tv < 2; ++tv) {
#pragma unroll
            for (int hf = 0; hf < 2; ++hf) {  // rows [64 hf, 64 hf + 64): lane quadrants 2 hf, 2 hf + 1
              uint32_t stg;
              BPROF(2, stg = slot_acquire());
              if ((q4 >> 1) == hf) {
#pragma unroll
                for (int k = 0; k < 8; ++k)
                  st_shared_v4(stg + sw128_off(r - 64 * hf, k), pk[tv][4 * k], pk[tv][4 * k + 1], pk[tv][4 * k + 2],
                               pk[tv][4 * k + 3]);
              }
              slot_done();
              if (leader) {
                asm volatile("cp.async.bulk.tensor.4d.global.shared::cta.bulk_group [%0, {%2, %3, %4, %5}], [%1];" ::"l"(
                                 reinterpret_cast<uint64_t>(&tdkv)),
                             "r"(stg), "r"(0), "r"(kt * 128 + 64 * hf), "r"((tv == 0 ? 2 * p.nh : p.nh) + hd), "r"(b)
                             : "memory");
                asm volatile("cp.async.bulk.commit_group;" ::: "memory");
              }
            }
          }
        }
        uint32_t v[2][32];
        __syncwarp();
        ptx::tmem_ld32(T_DQ, v[0]);
        ptx::tmem_ld32(T_DQ + 32, v[1]);
        ptx::tmem_ld_wait();
        ptx::tc_fence_before();
        __syncwarp();
        if (lane == 0) ptx::mbar_arrive(dq_empty);  // dQ TMEM may be overwritten
        constexpr int NSL = MOBIUS_BWD_SLAB32 ? 2 : 4, SW = 64 / NSL;  // slabs of SW columns
#pragma unroll
        for (int c = 0; c < NSL; ++c) {
          uint32_t stg;
          BPROF(1, stg = slot_acquire());
          if (MOBIUS_BWD_SLAB32) {  // 128-byte rows, SWIZZLE_128B
#pragma unroll
            for (int k = 0; k < 8; ++k)
              st_shared_v4(stg + r * 128 + ((k ^ (r & 7)) << 4), v[c & 1][4 * k], v[c & 1][4 * k + 1],
                           v[c & 1][4 * k + 2], v[c & 1][4 * k + 3]);
          } else {  // 64-byte rows, SWIZZLE_64B
#pragma unroll
            for (int k = 0; k < 4; ++k)
              st_shared_v4(stg + r * 64 + ((k ^ ((r >> 1) & 3)) << 4), v[c >> 1][(c & 1) * 16 + 4 * k],
                           v[c >> 1][(c & 1) * 16 + 4 * k + 1], v[c >> 1][(c & 1) * 16 + 4 * k + 2],
                           v[c >> 1][(c & 1) * 16 + 4 * k + 3]);
          }
          slot_done();
          if (leader) {
            asm volatile(
                "cp.reduce.async.bulk.tensor.4d.global.shared::cta.add.tile.bulk_group [%0, {%2, %3, %4, %5}], [%1];" ::"l"(
                    reinterpret_cast<uint64_t>(&tdq)),
                "r"(stg), "r"(c * SW), "r"((kt + it) * 128), "r"(hd), "r"(b)
                : "memory");
            asm volatile("cp.async.bulk.commit_group;" ::: "memory");
          }
        }
      }
      g += nq;
    }
    BPROF_DUMP("bdrn")
    if (leader) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");  // last stores / reduces complete
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc<512>(tmem);
  }
}

// Pre-pass of the flash backward, one warp per token row: negD[b, head, q] =
// -sum_d dO[q, d] O[q, d] (stored negated so the softmax-gradient loop adds
// it with FADD2), and the row's fp32 dQ accumulator zeroed (the kernel
// reduce-adds into it).  16-byte loads; DH/8 lanes per head.
template <int DH>
__global__ void __launch_bounds__(256) flash_dsum_kernel(const __nv_bfloat16* __restrict__ dO,
                                                         const __nv_bfloat16* __restrict__ O, float* __restrict__ negD,
                                                         float* __restrict__ dQacc, int rows, int nh, int s) {
  constexpr int LPH = DH / 8;  // lanes per head
  const int lane = threadIdx.x % 32;
  const int row = blockIdx.x * 8 + threadIdx.x / 32;
  if (row >= rows) return;
  const int h = nh * DH, nvec = h / 8;
  const int b = row / s, q = row % s;
  const __nv_bfloat16* dr = dO + (int64_t)row * h;
  const __nv_bfloat16* orow = O + (int64_t)row * h;
  float4* zr = reinterpret_cast<float4*>(dQacc + (int64_t)row * h);
  for (int v0 = 0; v0 < nvec; v0 += 32) {  // nvec is a multiple of LPH; a head never straddles iterations
    const int v = v0 + lane;
    float acc = 0.f;
    if (v < nvec) {
      const uint4 a = *reinterpret_cast<const uint4*>(dr + v * 8);
      const uint4 o = *reinterpret_cast<const uint4*>(orow + v * 8);
      const __nv_bfloat162* a2 = reinterpret_cast<const __nv_bfloat162*>(&a);
      const __nv_bfloat162* o2 = reinterpret_cast<const __nv_bfloat162*>(&o);
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const float2 x = __bfloat1622float2(a2[k]), y = __bfloat1622float2(o2[k]);
        acc += x.x * y.x + x.y * y.y;
      }
      zr[2 * v] = make_float4(0.f, 0.f, 0.f, 0.f);
      zr[2 * v + 1] = make_float4(0.f, 0.f, 0.f, 0.f);
    }
#pragma unroll
    for (int k = LPH / 2; k; k >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, k);
    if (v < nvec && (v % LPH) == 0) negD[((int64_t)b * nh + v / LPH) * s + q] = -acc;
  }
}

// dqkv q-part (bf16, row stride 3h) = scale * dQacc (fp32, row stride h)
// 8 elements per thread: two streaming 16-byte loads (the accumulator is not
// read again before the next call zeroes it), one 16-byte store (h % 8 == 0)
__global__ void flash_dq_cast_kernel(const float* dQacc, __nv_bfloat16* dq, int64_t rows, int h, int64_t ldd,
                                     float scale) {
  const int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) * 8;
  if (i >= rows * h) return;
  const int64_t r = i / h, c = i % h;
  const float4 v0 = __ldcs(reinterpret_cast<const float4*>(dQacc + i));
  const float4 v1 = __ldcs(reinterpret_cast<const float4*>(dQacc + i) + 1);
  uint4 o;
  o.x = pack_bf16(v0.x * scale, v0.y * scale);
  o.y = pack_bf16(v0.z * scale, v0.w * scale);
  o.z = pack_bf16(v1.x * scale, v1.y * scale);
  o.w = pack_bf16(v1.z * scale, v1.w * scale);
  *reinterpret_cast<uint4*>(dq + r * ldd + c) = o;
}

// (batch, head) pairs per item chunk of the backward: MOBIUS_FLASH_GROUP
// (0 or >= the pair count = one chunk, the global heaviest-first order).
// Default 64 at dh 64 (1.5B, mbs 32: bwd 701 -> 663 us; 16 / 32 / 128:
// 667 / 686 / 672 us) and one chunk at dh 128, where a chunk that keeps the
// fp32 dQ of its pairs in L2 (<= ~40 pairs of 1 MB) has too few items to
// balance 148 CTAs (13B shape, mbs 2: 402 us ungrouped, 419-488 grouped).
// The forward stays ungrouped (K / V re-reads measured cheaper than the lost
// balance: 261 us ungrouped, 266-274 grouped).
static int flash_group(int nbh, int dh) {
  static int g = -2;
  if (g == -2) {
    const char* e = getenv("MOBIUS_FLASH_GROUP");
    g = e ? atoi(e) : -1;
  }
  const int v = g == -1 ? (dh == 64 ? 64 : 0) : g;
  return (v <= 0 || v > nbh) ? nbh : v;
}

typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

EncodeTiledFn encode_fn() {
  static EncodeTiledFn fn = nullptr;
  if (!fn) {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<EncodeTiledFn>(p);
  }
  return fn;
}

// {d, token, head-slot, batch} map over a [mbs*s, ld] bf16 buffer whose head
// slots are dh apart; box {64, 128, 1, 1}
int head_map(CUtensorMap* m, const void* base, int64_t ld, int dh, int s, int n_slots, int mbs, int box_rows = 128) {
  EncodeTiledFn enc = encode_fn();
  if (!enc) MOBIUS_FAIL(MOBIUS_ECUDA, "cuTensorMapEncodeTiled unavailable");
  cuuint64_t dims[4] = {(cuuint64_t)dh, (cuuint64_t)s, (cuuint64_t)n_slots, (cuuint64_t)mbs};
  cuuint64_t strides[3] = {(cuuint64_t)(ld * 2), (cuuint64_t)(dh * 2), (cuuint64_t)(s * ld * 2)};
  cuuint32_t box[4] = {64, (cuuint32_t)box_rows, 1, 1};
  cuuint32_t es[4] = {1, 1, 1, 1};
  CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, const_cast<void*>(base), dims, strides, box, es,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) MOBIUS_FAIL(MOBIUS_ECUDA, "flash tensor map (%d)", (int)r);
  return MOBIUS_OK;
}

// fp32 {d, token, head, batch} map over the dQ accumulator [mbs*s, h]; box
// {32, 128, 1, 1} with 128B swizzle, or (cols 16) {16, 128, 1, 1} with 64B swizzle
int dq_map(CUtensorMap* m, const float* base, int h, int dh, int s, int nh, int mbs, int cols = 32) {
  EncodeTiledFn enc = encode_fn();
  if (!enc) MOBIUS_FAIL(MOBIUS_ECUDA, "cuTensorMapEncodeTiled unavailable");
  cuuint64_t dims[4] = {(cuuint64_t)dh, (cuuint64_t)s, (cuuint64_t)nh, (cuuint64_t)mbs};
  cuuint64_t strides[3] = {(cuuint64_t)h * 4, (cuuint64_t)dh * 4, (cuuint64_t)s * h * 4};
  cuuint32_t box[4] = {(cuuint32_t)cols, 128, 1, 1};
  cuuint32_t es[4] = {1, 1, 1, 1};
  CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, const_cast<float*>(base), dims, strides, box, es,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, cols == 16 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) MOBIUS_FAIL(MOBIUS_ECUDA, "flash dQ tensor map (%d)", (int)r);
  return MOBIUS_OK;
}

template <typename K>
int set_smem(K k, int bytes) {
  if (cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes) != cudaSuccess)
    MOBIUS_FAIL(MOBIUS_ECUDA, "flash smem attribute");
  return MOBIUS_OK;
}

}  // namespace

int flash_supported(int dh, int s) { return (dh == 64 || dh == 128) && s % 128 == 0; }

// MOBIUS_FLASH_FWD_V1=1: the round-2 10-warp forward (one query tile at a time) at dh 64
static bool flash_fwd_v1() {
  static int v1 = -1;
  if (v1 < 0) {
    const char* e = getenv("MOBIUS_FLASH_FWD_V1");
    v1 = (e && atoi(e) == 1) ? 1 : 0;
  }
  return v1 == 1;
}

int flash_attn_fwd(const __nv_bfloat16* qkv, __nv_bfloat16* o, float* lse, int mbs, int s, int nh, int dh,
                   cudaStream_t st) {
  MOBIUS_CHECK_ARG(flash_supported(dh, s), "flash: dh %d / s %d unsupported", dh, s);
  const int h = nh * dh;
  CUtensorMap tm;
  int rc = head_map(&tm, qkv, 3 * h, dh, s, 3 * nh, mbs);
  if (rc) return rc;
  CUtensorMap tmo;  // TMA-store view of O, 32-row boxes (one per softmax lane quadrant)
  rc = head_map(&tmo, o, h, dh, s, nh, mbs, 32);
  if (rc) return rc;
  FwdParams p;
  p.O = o;
  p.lse = lse;
  p.s = s;
  p.nh = nh;
  p.h = h;
  p.mbs = mbs;
  p.scale_log2 = 1.4426950408889634f / sqrtf((float)dh);
  p.group = nh * mbs;  // one chunk: global heaviest-first order
  {  // (batch, head) pairs per item chunk: MOBIUS_FLASH_FWD_GROUP, default 128
     // for the dh-64 ping-pong kernel (mbs 32: one chunk 212 us, 32 / 64 / 128 /
     // 256 pairs 212 / 206 / 206 / 211 us - a chunk's K / V stay in L2), one
     // chunk for the generic kernel (grouping cost it balance: 261 vs 266-274 us)
    static int fg = -2;
    if (fg == -2) {
      const char* e = getenv("MOBIUS_FLASH_FWD_GROUP");
      fg = e ? atoi(e) : -1;
    }
    const int want = fg >= 0 ? fg : (dh == 64 && !flash_fwd_v1() ? 128 : 0);
    if (want > 0 && want < p.group) p.group = want;
  }
  int n_items = (s / BQ) * nh * mbs;
  int sms = 148;
  {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  }
  dim3 grid(n_items < sms ? n_items : sms);
  if (dh == 64) {
    static bool once = false;
    // MOBIUS_FLASH_FWD_CP: softmax warps per S row (2: 8 warps of half rows, 4: 16 warps of quarter rows)
    static int cp = -1;
    if (cp < 0) {
      const char* e = getenv("MOBIUS_FLASH_FWD_CP");
      cp = (e && atoi(e) == 4) ? 4 : 2;
    }
    if (!flash_fwd_v1()) {
      static bool once64 = false;
      if (!once64) { rc = set_smem(flash_fwd64_kernel, Fwd64Cfg::SMEM); if (rc) return rc; once64 = true; }
      flash_fwd64_kernel<<<grid, 512, Fwd64Cfg::SMEM, st>>>(tm, tmo, p);
    } else if (cp == 4) {
      static bool once4 = false;
      if (!once4) { rc = set_smem(flash_fwd_kernel<64, 4>, FwdCfg<64>::SMEM); if (rc) return rc; once4 = true; }
      flash_fwd_kernel<64, 4><<<grid, (2 + 16) * 32, FwdCfg<64>::SMEM, st>>>(tm, tmo, p);
    } else {
      if (!once) { rc = set_smem(flash_fwd_kernel<64, 2>, FwdCfg<64>::SMEM); if (rc) return rc; once = true; }
      flash_fwd_kernel<64, 2><<<grid, NT_FWD, FwdCfg<64>::SMEM, st>>>(tm, tmo, p);
    }
  } else {
    static bool once = false;
    if (!once) { rc = set_smem(flash_fwd_kernel<128, 2>, FwdCfg<128>::SMEM); if (rc) return rc; once = true; }
    flash_fwd_kernel<128, 2><<<grid, NT_FWD, FwdCfg<128>::SMEM, st>>>(tm, tm, p);
  }
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) MOBIUS_FAIL(MOBIUS_ECUDA, "flash_fwd launch: %s", cudaGetErrorString(e));
  return MOBIUS_OK;
}

int flash_attn_bwd(const __nv_bfloat16* qkv, const __nv_bfloat16* o, const __nv_bfloat16* dout, const float* lse,
                   float* dsum_ws, float* dq_ws, __nv_bfloat16* dqkv, int mbs, int s, int nh, int dh,
                   cudaStream_t st) {
  MOBIUS_CHECK_ARG(flash_supported(dh, s), "flash: dh %d / s %d unsupported", dh, s);
  const int h = nh * dh;
  const int64_t rows = (int64_t)mbs * s;
  // MOBIUS_FLASH_BWD_V1=1: the round-2 10-warp kernel at dh 64 (softmax-gradient warps drain dQ themselves)
  static int v1 = -1;
  if (v1 < 0) {
    const char* e = getenv("MOBIUS_FLASH_BWD_V1");
    v1 = (e && atoi(e) == 1) ? 1 : 0;
  }
  const bool k64 = dh == 64 && !v1;  // flash_bwd64_kernel
  CUtensorMap tm, tdo, tdq;
  int rc = head_map(&tm, qkv, 3 * h, dh, s, 3 * nh, mbs);
  if (rc) return rc;
  rc = head_map(&tdo, dout, h, dh, s, nh, mbs);
  if (rc) return rc;
  // dh 64 kernel: 16-column dQ slabs and 64-row dV / dK halves (8 KB staging slots)
  rc = dq_map(&tdq, dq_ws, h, dh, s, nh, mbs, (k64 && !MOBIUS_BWD_SLAB32) ? 16 : 32);
  if (rc) return rc;
  CUtensorMap tdkv;  // TMA-store view of dqkv (dK / dV head slots)
  rc = head_map(&tdkv, dqkv, 3 * h, dh, s, 3 * nh, mbs, k64 ? 64 : 128);
  if (rc) return rc;
  if (dh == 64)
    flash_dsum_kernel<64><<<(unsigned)((rows + 7) / 8), 256, 0, st>>>(dout, o, dsum_ws, dq_ws, (int)rows, nh, s);
  else
    flash_dsum_kernel<128><<<(unsigned)((rows + 7) / 8), 256, 0, st>>>(dout, o, dsum_ws, dq_ws, (int)rows, nh, s);
  cudaError_t e;
  BwdParams p;
  p.lse = lse;
  p.Dsum = dsum_ws;
  p.dQacc = dq_ws;
  p.dqkv = dqkv;
  p.s = s;
  p.nh = nh;
  p.h = h;
  p.scale_log2 = 1.4426950408889634f / sqrtf((float)dh);
  p.scale = 1.0f / sqrtf((float)dh);
  p.mbs = mbs;
  p.group = flash_group(nh * mbs, dh);
  const int n_items = (s / 128) * nh * mbs;
  int sms = 148;
  {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  }
  dim3 grid(n_items < sms ? n_items : sms);  // persistent
  if (dh == 64) {
    static bool once = false;
    if (v1) {
      if (!once) { rc = set_smem(flash_bwd_kernel<64, 2>, BwdCfg<64>::SMEM); if (rc) return rc; once = true; }
      flash_bwd_kernel<64, 2><<<grid, NT_FWD, BwdCfg<64>::SMEM, st>>>(tm, tdo, tdq, tdkv, p);
    } else {
      static bool once64 = false;
      if (!once64) { rc = set_smem(flash_bwd64_kernel, Bwd64Cfg::SMEM); if (rc) return rc; once64 = true; }
      flash_bwd64_kernel<<<grid, 512, Bwd64Cfg::SMEM, st>>>(tm, tdo, tdq, tdkv, p);
    }
  } else {
    static bool once = false;
    if (!once) { rc = set_smem(flash_bwd_kernel<128, 2>, BwdCfg<128>::SMEM); if (rc) return rc; once = true; }
    flash_bwd_kernel<128, 2><<<grid, NT_FWD, BwdCfg<128>::SMEM, st>>>(tm, tdo, tdq, tdkv, p);
  }
  {
    const int64_t n = rows * h / 8;
    flash_dq_cast_kernel<<<(unsigned)((n + 255) / 256), 256, 0, st>>>(dq_ws, dqkv, rows, h, 3 * h, p.scale);
  }
  e = cudaGetLastError();
  if (e != cudaSuccess) MOBIUS_FAIL(MOBIUS_ECUDA, "flash_bwd launch: %s", cudaGetErrorString(e));
  return MOBIUS_OK;
}

}  // namespace mobius
