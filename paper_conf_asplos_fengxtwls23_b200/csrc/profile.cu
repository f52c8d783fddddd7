// mobius_profile: layer-similarity profiling.  "Mobius
// merges a group of equal layers into one based on the model layer
// similarity": one transformer block, the embedding and the head are timed
// once each at the config's micro-batch size (prefetch disabled: weights
// resident, no transfers) and the block time is replicated over all L
// blocks.  t_bwd includes the forward recompute the runtime performs.
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <vector>

#include "common.h"
#include "elem.h"
#include "flash.h"
#include "ops.h"

using namespace mobius;

namespace {

template <typename T>
int profile_impl(const mobius_model_cfg& c, mobius_layer_profile* out, int Lp) {
  Shape sh{c.hidden, c.n_heads, c.seq_len, c.micro_batch, c.vocab};
  const int64_t e = sizeof(T), Tn = sh.T(), h = sh.h;
  BlockLayout BL(h);
  EmbedLayout EL(h, c.vocab, c.seq_len);
  HeadLayout HL(h, c.vocab);
  int64_t wmax = std::max(BL.total, std::max(EL.total, HL.total));
  const bool fl = use_flash<T>(sh);
  int64_t ab = block_acts_bytes(sh, (int)e, fl), sb = scratch_bytes(sh, (int)e, true, fl);
  int64_t xb = (Tn * h * e + 255) & ~int64_t(255);
  int64_t tokb = ((int64_t)sh.mbs * (sh.s + 1) * 4 + 255) & ~int64_t(255);
  int64_t total = wmax * e + wmax * 4 + ab + sb + 4 * xb + tokb + 256 + 4096;
  uint8_t* buf = nullptr;
  if (cudaMalloc(&buf, total) != cudaSuccess) MOBIUS_FAIL(MOBIUS_ENOMEM, "profile arena (%lld bytes)", (long long)total);
  cudaMemset(buf, 0, total);
  uint8_t* p = buf;
  auto take = [&](int64_t b) { uint8_t* r = p; p += (b + 255) & ~int64_t(255); return r; };
  T* w = (T*)take(wmax * e);
  float* g = (float*)take(wmax * 4);
  uint8_t* actb = take(ab);
  uint8_t* scb = take(sb);
  T* x0 = (T*)take(xb);
  T* x1 = (T*)take(xb);
  T* d0 = (T*)take(xb);
  T* d1 = (T*)take(xb);
  int32_t* tok = (int32_t*)take(tokb);
  double* loss = (double*)take(8);
  BlockActs<T> acts;
  Scratch<T> sc;
  carve_block_acts<T>(sh, actb, acts);
  carve_scratch<T>(sh, scb, true, sc);
  scratch_zero<T>(sc, 0);
  {  // token ids spread over the vocabulary (a multiplicative hash of the position)
    std::vector<int32_t> ht((size_t)sh.mbs * (sh.s + 1));
    for (size_t i = 0; i < ht.size(); ++i) ht[i] = (int32_t)((i * 2654435761ull) % (uint64_t)sh.V);
    cudaMemcpy(tok, ht.data(), ht.size() * 4, cudaMemcpyHostToDevice);
  }
  acts.x = x0;
  cudaStream_t st;
  cudaStreamCreate(&st);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  auto time = [&](auto&& fn) -> int64_t {
    for (int i = 0; i < 2; ++i) fn();
    cudaEventRecord(a, st);
    const int it = 5;
    for (int i = 0; i < it; ++i) fn();
    cudaEventRecord(b, st);
    cudaEventSynchronize(b);
    float ms = 0.f;
    cudaEventElapsedTime(&ms, a, b);
    return (int64_t)(ms * 1e6 / it);
  };
  int rc = MOBIUS_OK;
  int64_t tbf = time([&] { rc |= block_fwd<T>(sh, w, acts, x1, sc, st); });
  int64_t tbb = time([&] {
    rc |= block_fwd<T>(sh, w, acts, x1, sc, st);
    rc |= block_bwd<T>(sh, w, acts, d0, d1, g, sc, st);
  });
  int64_t tef = time([&] { rc |= embed_layer_fwd<T>(sh, w, tok, x0, st); });
  int64_t teb = time([&] {
    rc |= embed_layer_fwd<T>(sh, w, tok, x0, st);
    rc |= embed_layer_bwd<T>(sh, w, tok, d0, g, st);
  });
  int64_t th = time([&] { rc |= head_layer_fwd_bwd<T>(sh, w, x0, tok, 1e-3f, d0, g, loss, sc, st); });
  cudaError_t err = cudaStreamSynchronize(st);
  cudaEventDestroy(a);
  cudaEventDestroy(b);
  cudaStreamDestroy(st);
  cudaFree(buf);
  if (rc) return rc;
  if (err != cudaSuccess) MOBIUS_FAIL(MOBIUS_ECUDA, "profile: %s", cudaGetErrorString(err));
  for (int i = 0; i < Lp; ++i) {
    if (i == 0) {
      out[i].t_fwd_ns = tef;
      out[i].t_bwd_ns = teb;
    } else if (i == Lp - 1) {
      out[i].t_fwd_ns = 0;   // the head's fwd+bwd runs inside B of the last stage
      out[i].t_bwd_ns = th;
    } else {
      out[i].t_fwd_ns = tbf;
      out[i].t_bwd_ns = tbb;
    }
  }
  return MOBIUS_OK;
}

}  // namespace

extern "C" int mobius_profile(const mobius_model_cfg* cfg, int device, mobius_layer_profile* out, int* n_out) {
  int rc = mobius_layer_sizes(cfg, out, n_out);
  if (rc) return rc;
  if (cudaSetDevice(device) != cudaSuccess) MOBIUS_FAIL(MOBIUS_ECUDA, "cudaSetDevice(%d)", device);
  if (cfg->dtype == MOBIUS_F32) return profile_impl<float>(*cfg, out, *n_out);
  return profile_impl<__nv_bfloat16>(*cfg, out, *n_out);
}
