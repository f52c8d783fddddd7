// Microbenchmark: cycles per tcgen05.mma (cta_group::1, kind::f16, bf16)
// issued back to back into one TMEM accumulator, for the instruction shapes
// the flash kernels use (M = 128, N = 64 / 128 / 256, K = 16; SS with K-major
// or MN-major B, and TS with A from TMEM).  One CTA per SM; operands are
// zero-filled smem (data-independent timing).  Research tool for DESIGN §8
// next step 1, not part of the product.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 \
//          -I paper_conf_asplos_fengxtwls23_b200/csrc tools/probe/mma_probe.cu -o /tmp/mma_probe
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#include "ptx.cuh"

using namespace mobius;

// issued by a converged warp: elect.sync picks one lane inside the asm, so
// the surrounding control flow stays warp-uniform and the compiler can keep
// descriptors in uniform registers (no per-MMA waterfall loop)
__device__ __forceinline__ void mma_ss_elect(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc) {
  asm volatile(
      "{\n\t.reg .pred e;\n\t"
      "elect.sync _|e, 0xffffffff;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, 1;\n\t}\n" ::"r"(d),
      "l"(a), "l"(b), "r"(idesc));
}
__device__ __forceinline__ void mma_ts_elect(uint32_t d, uint32_t a, uint64_t b, uint32_t idesc) {
  asm volatile(
      "{\n\t.reg .pred e;\n\t"
      "elect.sync _|e, 0xffffffff;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, 1;\n\t}\n" ::"r"(d),
      "r"(a), "l"(b), "r"(idesc));
}

template <int TS, int ELECT>
__global__ void __launch_bounds__(128, 1) probe(int n_iter, uint32_t idesc, int b_mn, int n_acc, int acc_stride,
                                               long long* out) {
  constexpr int ts = TS, elect_mode = ELECT;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t bar;
  __shared__ uint32_t tslot;
  for (int i = threadIdx.x; i < 96 * 1024 / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(smem)[i] = 0;
  if (threadIdx.x == 0) {
    ptx::mbar_init(&bar, 1);
    ptx::fence_mbar_init();
  }
  if (threadIdx.x / 32 == 0) ptx::tmem_alloc<512>(&tslot);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = tslot;
  if (threadIdx.x < 32 && (elect_mode || threadIdx.x == 0)) {
    const uint32_t a = ptx::smem_u32(smem), b = ptx::smem_u32(smem + 32768);
    // descriptors and accumulator addresses precomputed: the timed loop is
    // only the MMA issue (mode 2 rebuilds them per MMA, like the kernels)
    uint64_t bds[8], ads[8];
    uint32_t dd[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      bds[k] = b_mn ? ptx::sdesc_sw128(b + k * 2048, 16384, 1024)
                    : ptx::sdesc_sw128(b + (k >> 2) * 16384 + (k & 3) * 32, 16, 1024);
      ads[k] = ptx::sdesc_sw128(a + (k >> 2) * 16384 + (k & 3) * 32, 16, 1024);
      dd[k] = tmem + (uint32_t)((k % n_acc) * acc_stride);
    }
    long long t0 = clock64();
    for (int it = 0; it < n_iter; ++it) {
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        if constexpr (ELECT) {
          if constexpr (TS)
            mma_ts_elect(dd[k], tmem + 384 + 8 * k, bds[k], idesc);
          else
            mma_ss_elect(dd[k], ads[k], bds[k], idesc);
        } else if constexpr (TS) {
          ptx::mma_bf16_ts(dd[k], tmem + 384 + 8 * k, bds[k], idesc, 1u);
        } else {
          ptx::mma_bf16(dd[k], ads[k], bds[k], idesc, 1u);
        }
      }
    }
    if (threadIdx.x == 0) {
      ptx::mma_commit(&bar);
      ptx::mbar_wait(&bar, 0);
      long long t1 = clock64();
      out[blockIdx.x] = t1 - t0;
    }
  }
  __syncthreads();
  if (threadIdx.x / 32 == 0) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc<512>(tmem);
  }
}

int main() {
  long long* d;
  cudaMalloc(&d, 148 * sizeof(long long));
  cudaFuncSetAttribute(probe<0, 0>, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
  cudaFuncSetAttribute(probe<0, 1>, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
  cudaFuncSetAttribute(probe<1, 0>, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
  cudaFuncSetAttribute(probe<1, 1>, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
  struct Case { const char* name; int N, b_mn, ts, n_acc, elect; } cases[] = {
      {"SS N=64  lane0", 64, 1, 0, 1, 0},  {"SS N=64  elect", 64, 1, 0, 1, 1},
      {"SS N=128 lane0", 128, 0, 0, 1, 0}, {"SS N=128 elect", 128, 0, 0, 1, 1},
      {"TS N=64  lane0", 64, 1, 1, 1, 0},  {"TS N=64  elect", 64, 1, 1, 1, 1},
      {"SS N=256 lane0", 256, 0, 0, 1, 0}, {"SS N=256 elect", 256, 0, 0, 1, 1}};
  const int n_iter = 2000;
  for (auto& c : cases) {
    const uint32_t idesc = ptx::idesc_bf16(128, c.N, 0, c.b_mn);
    if (c.ts && c.elect) probe<1, 1><<<148, 128, 100 * 1024>>>(n_iter, idesc, c.b_mn, c.n_acc, c.N, d);
    else if (c.ts) probe<1, 0><<<148, 128, 100 * 1024>>>(n_iter, idesc, c.b_mn, c.n_acc, c.N, d);
    else if (c.elect) probe<0, 1><<<148, 128, 100 * 1024>>>(n_iter, idesc, c.b_mn, c.n_acc, c.N, d);
    else probe<0, 0><<<148, 128, 100 * 1024>>>(n_iter, idesc, c.b_mn, c.n_acc, c.N, d);
    cudaError_t e = cudaDeviceSynchronize();
    long long h[148];
    cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    double avg = 0;
    for (int i = 0; i < 148; ++i) avg += h[i];
    avg /= 148.0;
    const double per = avg / (n_iter * 8.0), ideal = 128.0 * c.N * 16 * 2 / 8192.0;
    printf("%-22s %s  %7.1f cycles/MMA  (math %5.1f)  -> %4.0f%% of the per-SM bf16 rate\n", c.name,
           e == cudaSuccess ? "ok " : cudaGetErrorString(e), per, ideal, 100.0 * ideal / per);
  }
  return 0;
}
