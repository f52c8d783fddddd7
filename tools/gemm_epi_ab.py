"""Time one GEMM shape under each epilogue (CUDA events, warm) to isolate
the epilogue's cost: usage python tools/gemm_epi_ab.py M N K [epis...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
from paper_conf_asplos_fengxtwls23_b200 import BF16, kt  # noqa: E402

M, N, K = map(int, sys.argv[1:4])
epis = [int(e) for e in sys.argv[4:]] or [0, 1, 2, 3, 4]


def mk(*s):
    return (torch.randn(*s, device="cuda") * 0.1).to(torch.bfloat16)


A, B = mk(M, K), mk(K, N)
C = torch.zeros(M, N, device="cuda", dtype=torch.bfloat16)
bias, R, AUX = mk(N), mk(M, N), mk(M, N)
for epi in epis:
    f = lambda: kt.gemm(BF16, M, N, K, A, K, 0, B, N, 1, C, N, epi=epi,  # noqa
                        bias=bias if epi in (1, 2, 3) else None, R=R if epi in (3, 4) else None, ldr=N,
                        AUX=AUX if epi == 2 else None, ldx=N)
    for _ in range(5):
        f()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(20):
        f()
    b.record()
    torch.cuda.synchronize()
    us = a.elapsed_time(b) / 20 * 1e3
    print(f"M={M} N={N} K={K} epi={epi}: {us:8.1f} us {2 * M * N * K / us / 1e6:7.0f} TF/s")
