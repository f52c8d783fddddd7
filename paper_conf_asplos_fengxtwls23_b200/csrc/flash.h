// Fused causal attention on tcgen05 (bf16 path), see flash.cu.
#pragma once

#include <cuda_bf16.h>
#include <cuda_runtime.h>

namespace mobius {

int flash_supported(int dh, int s);
// qkv [mbs*s, 3h] (q|k|v, heads of dh contiguous columns) -> o [mbs*s, h],
// lse [mbs, nh, s] (log2 domain)
int flash_attn_fwd(const __nv_bfloat16* qkv, __nv_bfloat16* o, float* lse, int mbs, int s, int nh, int dh,
                   cudaStream_t st);
// dout [mbs*s, h] -> dqkv [mbs*s, 3h]; workspaces: dsum [mbs*nh*s] fp32,
// dq [mbs*s, h] fp32
int flash_attn_bwd(const __nv_bfloat16* qkv, const __nv_bfloat16* o, const __nv_bfloat16* dout, const float* lse,
                   float* dsum_ws, float* dq_ws, __nv_bfloat16* dqkv, int mbs, int s, int nh, int dh, cudaStream_t st);

}  // namespace mobius
