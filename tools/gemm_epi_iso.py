"""fc1-forward shape (T x 4h x h) with each epilogue: isolates the cost of the
fused bias+GeLU epilogue (two outputs) from the mainloop.  Research tool."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ.setdefault("MOBIUS_KT_NOSYNC", "1")
import torch  # noqa: E402
from paper_conf_asplos_fengxtwls23_b200 import BF16, kt  # noqa: E402


def t(fn, it=20):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(it):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / it * 1e3


def mk(*s):
    return (torch.randn(*s, device="cuda") * 0.1).to(torch.bfloat16)


T, h = int(os.environ.get("GEMM_T", "32768")), 1600
for (M, N, K) in ((T, 4 * h, h), (T, 3 * h, h)):
    A, B = mk(M, K), mk(K, N)
    C, X = torch.zeros(M, N, device="cuda", dtype=torch.bfloat16), torch.zeros(M, N, device="cuda", dtype=torch.bfloat16)
    bias = mk(N)
    for epi, name in ((0, "store"), (1, "bias"), (2, "bias+gelu (2 outputs)")):
        us = t(lambda: kt.gemm(BF16, M, N, K, A, K, False, B, N, True, C, N, epi=epi, bias=bias if epi else None,
                               AUX=X if epi == 2 else None, ldx=N))
        print(f"{M}x{N}x{K} {name:24s} {us:7.1f} us {2.0 * M * N * K / us / 1e6:6.0f} TF/s")
