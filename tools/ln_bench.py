"""Time LayerNorm forward and backward (dx + gamma/beta grads) at the bench
shape (T = mbs*s rows, h = 1600).  MOBIUS_LN_FLOATROW=1 selects the generic
kernels for an A/B in a second process."""
import os
import sys
os.environ.setdefault('MOBIUS_KT_NOSYNC', '1')
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
from paper_conf_asplos_fengxtwls23_b200 import BF16, kt  # noqa: E402

mbs, s, h = int(os.environ.get("MBS", "32")), 1024, 1600
T = mbs * s


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


g = torch.Generator(device="cuda").manual_seed(0)
x = torch.randn(T, h, device="cuda", generator=g).to(torch.bfloat16)
dy = torch.randn(T, h, device="cuda", generator=g).to(torch.bfloat16)
dres = torch.randn(T, h, device="cuda", generator=g).to(torch.bfloat16)
gam = (1 + 0.1 * torch.randn(h, device="cuda", generator=g)).to(torch.bfloat16)
bet = (0.1 * torch.randn(h, device="cuda", generator=g)).to(torch.bfloat16)
y = torch.empty_like(x)
dx = torch.empty_like(x)
mu = torch.empty(T, device="cuda")
rs = torch.empty(T, device="cuda")
dg = torch.zeros(h, device="cuda")
db = torch.zeros(h, device="cuda")
tag = "generic" if os.environ.get("MOBIUS_LN_FLOATROW") == "1" else "packed"
us = t(lambda: kt.layernorm_fwd(BF16, x, gam, bet, y, mu, rs, T, h))
print(f"ln_fwd {tag:8s} T={T}: {us:8.1f} us ({4 * T * h / us / 1e3:7.1f} GB/s)")
us = t(lambda: kt.layernorm_bwd(BF16, dy, x, gam, mu, rs, dres, dx, dg, db, T, h))
print(f"ln_bwd {tag:8s} T={T}: {us:8.1f} us ({(8 + 4) * T * h / us / 1e3:7.1f} GB/s, dx 3 reads + 1 write, grads 2 reads)")
print("checksum", float(dx.float().abs().sum()), float(dg.abs().sum()))
