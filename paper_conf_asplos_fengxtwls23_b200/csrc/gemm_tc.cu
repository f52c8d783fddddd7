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
#include "gemm_common.cuh"

namespace mobius {
namespace gemm_detail {

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


// ------------------------------------------------------------ host side
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static EncodeTiledFn get_encode() {
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

int make_map_2d(CUtensorMap* map, const void* ptr, bool f32, int64_t ld, int64_t inner, int64_t outer, int box_inner,
                int box_outer) {
  EncodeTiledFn enc = get_encode();
  if (!enc) MOBIUS_FAIL(MOBIUS_ECUDA, "cuTensorMapEncodeTiled unavailable");
  const int64_t es = f32 ? 4 : 2;
  if ((reinterpret_cast<uintptr_t>(ptr) & 15) != 0 || (ld * es) % 16 != 0)
    MOBIUS_FAIL(MOBIUS_EINVAL, "TMA epilogue map: base and row stride must be 16-byte aligned");
  cuuint64_t dims[4] = {(cuuint64_t)inner, (cuuint64_t)outer, 1, 1};
  cuuint64_t strides[3] = {(cuuint64_t)(ld * es), (cuuint64_t)(ld * es * outer), (cuuint64_t)(ld * es * outer)};
  cuuint32_t box[4] = {(cuuint32_t)box_inner, (cuuint32_t)box_outer, 1, 1};
  cuuint32_t estr[4] = {1, 1, 1, 1};
  CUresult r = enc(map, f32 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32 : CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, const_cast<void*>(ptr),
                   dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                   CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) MOBIUS_FAIL(MOBIUS_ECUDA, "cuTensorMapEncodeTiled (epilogue) failed (%d)", (int)r);
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

}  // namespace gemm_detail

using namespace gemm_detail;

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

// 2-CTA kernel entry and knobs (gemm_tc2.cu)
int gemm_bf16_2cta(const GemmDesc& d, cudaStream_t s);
void gemm_2cta_set_stream_k(int stream_k);

static int g_gemm_mode = -1;  // -1 auto (env MOBIUS_GEMM_2CTA, default on), 0 off, 1 on

void gemm_set_config(int two_cta, int stream_k) {
  g_gemm_mode = two_cta;
  gemm_2cta_set_stream_k(stream_k);
}

static bool use_2cta(const GemmDesc& d) {
  if (g_gemm_mode < 0) {
    const char* e = getenv("MOBIUS_GEMM_2CTA");
    g_gemm_mode = (e && e[0] == '0') ? 0 : 1;
  }
  return g_gemm_mode == 1 && d.causal == CAUSAL_NONE && d.nb1 == 1 && d.nb2 == 1 && d.N >= 256 && d.M >= 256 &&
         d.K >= 64;
}

bool gemm_ones_row_supported(const GemmDesc& d, bool f32) {
  if (f32) return true;  // the SIMT kernel synthesises the row
  const int r = d.M - 1;
  return use_2cta(d) && d.a_mn && d.epi == EPI_ACCUM && r % 64 == 0 && r % 256 != 0;
}

int gemm_bf16(const GemmDesc& d, cudaStream_t s) {
  if (use_2cta(d)) return gemm_bf16_2cta(d, s);
  MOBIUS_CHECK_ARG(!d.ones_row, "gemm: the ones row needs the 2-CTA kernel");
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
