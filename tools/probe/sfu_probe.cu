// Microbenchmark for the flash softmax budget (research tool, not product):
//  (1) MUFU ex2.approx throughput per SM with W warps of independent chains
//  (2) tcgen05.ld 32x32b.x32 (+ wait) throughput per SM with W warps
//  (3) tcgen05.st 32x32b.x16 (+ wait) throughput per SM with W warps
//  (4) FFMA2 throughput per SM with W warps (packed f32x2 FMA pipe rate)
// One CTA per SM; cycles from clock64 of warp 0 around the timed loop.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 \
//          -I paper_conf_asplos_fengxtwls23_b200/csrc tools/probe/sfu_probe.cu -o /tmp/sfu_probe
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#include "ptx.cuh"

using namespace mobius;

__device__ __forceinline__ float ex2(float x) {
  float y;
  asm volatile("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}

template <int MODE>
__global__ void __launch_bounds__(512, 1) probe(int n_iter, long long* out, float* sink) {
  __shared__ uint32_t tslot;
  const int warp = threadIdx.x / 32;
  if (warp == 0) ptx::tmem_alloc<512>(&tslot);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = tslot;
  const uint32_t lb = (uint32_t)((warp & 3) * 32) << 16;
  float acc[8];
  for (int i = 0; i < 8; ++i) acc[i] = threadIdx.x * 1e-3f + i;
  uint32_t r[32];
  for (int i = 0; i < 32; ++i) r[i] = i;
  __syncthreads();
  long long t0 = clock64();
  for (int it = 0; it < n_iter; ++it) {
    if (MODE == 0) {
#pragma unroll
      for (int k = 0; k < 8; ++k) {
#pragma unroll
        for (int i = 0; i < 8; ++i) acc[i] = ex2(acc[i]) * -0.5f;
      }
    } else if (MODE == 1) {
      ptx::tmem_ld32(tmem + lb + ((warp >> 2) & 3) * 64, r);
      ptx::tmem_ld_wait();
      acc[0] += __uint_as_float(r[0] ^ r[31]);
    } else if (MODE == 2) {
      uint32_t s16[16];
#pragma unroll
      for (int i = 0; i < 16; ++i) s16[i] = r[i] + it;
      ptx::tmem_st16(tmem + lb + ((warp >> 2) & 3) * 64, s16);
      ptx::tmem_st_wait();
    } else if (MODE == 3) {
#pragma unroll
      for (int k = 0; k < 8; ++k) {
#pragma unroll
        for (int i = 0; i < 8; i += 2) {
          float2 v = __ffma2_rn(make_float2(acc[i], acc[i + 1]), make_float2(0.999f, 0.999f), make_float2(1e-3f, 1e-3f));
          acc[i] = v.x;
          acc[i + 1] = v.y;
        }
      }
    } else if (MODE == 5) {  // ex2.approx.f16x2: two exponentials per lane per instruction
#pragma unroll
      for (int k = 0; k < 8; ++k) {
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          uint32_t h = __float_as_uint(acc[i]), o;
          asm volatile("ex2.approx.f16x2 %0, %1;" : "=r"(o) : "r"(h));
          acc[i] = __uint_as_float(o ^ 0x80008000u);
        }
      }
    } else if (MODE == 6) {  // ex2.approx.ftz.bf16x2
#pragma unroll
      for (int k = 0; k < 8; ++k) {
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          uint32_t h = __float_as_uint(acc[i]), o;
          asm volatile("ex2.approx.ftz.bf16x2 %0, %1;" : "=r"(o) : "r"(h));
          acc[i] = __uint_as_float(o ^ 0x80008000u);
        }
      }
    } else if (MODE == 7) {  // tanh.approx.f32
#pragma unroll
      for (int k = 0; k < 8; ++k) {
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          float y;
          asm volatile("tanh.approx.f32 %0, %1;" : "=f"(y) : "f"(acc[i]));
          acc[i] = y * 1.5f;
        }
      }
    } else if (MODE == 8) {  // rcp.approx.ftz.f32
#pragma unroll
      for (int k = 0; k < 8; ++k) {
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          float y;
          asm volatile("rcp.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(acc[i]));
          acc[i] = y + 0.5f;
        }
      }
    } else if (MODE == 4) {  // four tcgen05.ld x32 in flight, one wait (a 128-column row chunk)
      uint32_t r2[32], r3[32], r4[32];
      ptx::tmem_ld32(tmem + lb + 0, r);
      ptx::tmem_ld32(tmem + lb + 32, r2);
      ptx::tmem_ld32(tmem + lb + 64, r3);
      ptx::tmem_ld32(tmem + lb + 96, r4);
      ptx::tmem_ld_wait();
      acc[0] += __uint_as_float(r[0] ^ r2[31] ^ r3[7] ^ r4[9]);
    }
  }
  long long t1 = clock64();
  float s = 0;
  for (int i = 0; i < 8; ++i) s += acc[i];
  sink[blockIdx.x * blockDim.x + threadIdx.x] = s;
  if (threadIdx.x == 0) out[blockIdx.x] = t1 - t0;
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 0) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc<512>(tmem);
  }
}

template <int MODE>
void run(const char* name, int warps, double units_per_iter_per_warp, const char* unit) {
  long long* d;
  float* sink;
  cudaMalloc(&d, 148 * sizeof(long long));
  cudaMalloc(&sink, 148 * 512 * sizeof(float));
  const int n_iter = 4000;
  probe<MODE><<<148, warps * 32>>>(n_iter, d, sink);
  cudaError_t e = cudaDeviceSynchronize();
  long long h[148];
  cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
  double avg = 0;
  for (int i = 0; i < 148; ++i) avg += h[i];
  avg /= 148.0;
  const double units = units_per_iter_per_warp * warps * n_iter;
  printf("%-28s warps %2d %s  %8.3f %s per cycle per SM (%.2f cycles per warp-op)\n", name, warps,
         e == cudaSuccess ? "ok " : cudaGetErrorString(e), units / avg, unit, avg / (n_iter * (units_per_iter_per_warp / 32.0) * warps) );
  cudaFree(d);
  cudaFree(sink);
}

int main() {
  for (int w : {4, 8, 16}) run<0>("MUFU ex2", w, 64 * 32, "ex2");
  for (int w : {4, 8, 16}) run<7>("MUFU tanh", w, 64 * 32, "tanh");
  for (int w : {4, 8, 16}) run<8>("MUFU rcp", w, 64 * 32, "rcp");
  for (int w : {4, 8, 16}) run<5>("MUFU ex2 f16x2", w, 64 * 32 * 2, "ex2");
  for (int w : {4, 8, 16}) run<6>("MUFU ex2 bf16x2", w, 64 * 32 * 2, "ex2");
  for (int w : {4, 8, 16}) run<3>("FFMA2", w, 32 * 32 * 2, "flop-lanes");
  for (int w : {4, 8, 16}) run<1>("tcgen05.ld 32x32b.x32", w, 32 * 32 * 4, "bytes");
  for (int w : {4, 8, 16}) run<4>("tcgen05.ld 4 x x32 in flight", w, 4 * 32 * 32 * 4, "bytes");
  for (int w : {4, 8, 16}) run<2>("tcgen05.st 32x32b.x16", w, 16 * 32 * 4, "bytes");
  return 0;
}
