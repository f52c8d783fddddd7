"""Run one bf16 GEMM shape a few times (for ncu / A-B of kernel knobs).
usage: python tools/gemm_one.py M N K a_mn b_mn epi c_f32 [two_cta stream_k] [iters]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
from paper_conf_asplos_fengxtwls23_b200 import BF16, kt  # noqa: E402

M, N, K, amn, bmn, epi, cf = map(int, sys.argv[1:8])
two, sk = (int(sys.argv[8]), int(sys.argv[9])) if len(sys.argv) > 9 else (-1, -1)
it = int(sys.argv[10]) if len(sys.argv) > 10 else 5
kt.gemm_config(two, sk)
dev = "cuda"


def mk(*s):
    return (torch.randn(*s, device=dev) * 0.1).to(torch.bfloat16)


A = mk(K, M) if amn else mk(M, K)
B = mk(K, N) if bmn else mk(N, K)
C = torch.zeros(M, N, device=dev, dtype=torch.float32 if cf else torch.bfloat16)
bias, R, AUX = mk(N), mk(M, N), mk(M, N)
f = lambda: kt.gemm(BF16, M, N, K, A, M if amn else K, amn, B, N if bmn else K, bmn, C, N, c_f32=bool(cf), epi=epi,  # noqa
                    bias=bias if epi in (1, 2, 3) else None, R=R if epi in (3, 4) else None, ldr=N,
                    AUX=AUX if epi == 2 else None, ldx=N, accumulate=(epi == 5))
for _ in range(it):
    f()
torch.cuda.synchronize()
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
a.record()
for _ in range(20):
    f()
b.record()
torch.cuda.synchronize()
ms = a.elapsed_time(b) / 20
print(f"{M}x{N}x{K} two_cta={two} sk={sk}: {ms*1e3:.1f} us {2.0*M*N*K/ms/1e9:.1f} TF/s")
