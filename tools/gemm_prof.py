"""One launch each of the 1.5B-block GEMM shapes (for ncu --set full)."""
import os
import sys

# T = mbs * s tokens per microbatch: 16384 for the bench's 1.5b default
# (mbs 16); GEMM_T=8192 gives the v3 (mbs 8) shapes
T, h = int(os.environ.get("GEMM_T", "16384")), 1600
# name, M, N, K, a_mn, b_mn, epi, c_f32 - the 12 GEMMs of one block fwd + bwd
SHAPES = [("qkv_fwd_bias", T, 3 * h, h, 0, 1, 1, 0), ("o_fwd_res", T, h, h, 0, 1, 3, 0),
          ("fc1_fwd_gelu", T, 4 * h, h, 0, 1, 2, 0), ("fc2_fwd_res", T, h, 4 * h, 0, 1, 3, 0),
          ("fc2_dX_geluprime", T, 4 * h, h, 0, 0, 4, 0), ("fc1_dX", T, h, 4 * h, 0, 0, 0, 0),
          ("fc1_dW", h, 4 * h, T, 1, 1, 5, 1), ("qkv_dW", h, 3 * h, T, 1, 1, 5, 1),
          ("fc2_dW", 4 * h, h, T, 1, 1, 5, 1), ("o_dX", T, h, h, 0, 0, 0, 0), ("o_dW", h, h, T, 1, 1, 5, 1),
          ("qkv_dX", T, h, 3 * h, 0, 0, 0, 0)]

if __name__ == "__main__":
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import torch
    from paper_conf_asplos_fengxtwls23_b200 import BF16, kt

    def mk(*s):
        return (torch.randn(*s, device="cuda") * 0.1).to(torch.bfloat16)

    for name, M, N, K, amn, bmn, epi, cf in SHAPES:
        A = mk(K, M) if amn else mk(M, K)
        B = mk(K, N) if bmn else mk(N, K)
        C = torch.zeros(M, N, device="cuda", dtype=torch.float32 if cf else torch.bfloat16)
        bias, R, AUX = mk(N), mk(M, N), mk(M, N)
        kt.gemm(BF16, M, N, K, A, M if amn else K, amn, B, N if bmn else K, bmn, C, N, c_f32=bool(cf), epi=epi,
                bias=bias if epi in (1, 2, 3) else None, R=R if epi in (3, 4) else None, ldr=N,
                AUX=AUX if epi == 2 else None, ldx=N, accumulate=(epi == 5))
    torch.cuda.synchronize()
