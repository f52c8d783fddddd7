"""Time the dWte scatter (embed_bwd) at the bench shape: T = mbs*s tokens,
h = 1600, V = 50304, uniform / zipf / single-id token streams."""
import os
import sys
os.environ.setdefault('MOBIUS_KT_NOSYNC', '1')
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
from paper_conf_asplos_fengxtwls23_b200 import BF16, kt  # noqa: E402

mbs, s, h, V = int(os.environ.get("MBS", "32")), 1024, 1600, 50304


def t(fn, it=10):
    for _ in range(2):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(it):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / it * 1e3


dx = torch.randn(mbs * s, h, device="cuda").to(torch.bfloat16)
dwte = torch.zeros(V, h, device="cuda")
dwpe = torch.zeros(s, h, device="cuda")
for name in ("uniform", "zipf", "single"):
    if name == "uniform":
        tok = torch.randint(0, V, (mbs, s + 1), device="cuda", dtype=torch.int32)
    elif name == "zipf":
        import numpy as np
        tok = torch.from_numpy(np.minimum(np.random.default_rng(0).zipf(1.2, size=(mbs, s + 1)) - 1, V - 1)
                               .astype(np.int32)).cuda()
    else:
        tok = torch.full((mbs, s + 1), V - 1, device="cuda", dtype=torch.int32)
    us = t(lambda: kt.embed_bwd(BF16, tok, dx, dwte, dwpe, mbs, s, h, V))
    print(f"embed_bwd {name:8s} T={mbs * s}: {us:9.1f} us  ({mbs * s * h * 2 / us / 1e3:7.1f} GB/s of dx)")
