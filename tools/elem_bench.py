"""Time the HBM-bound kernels at the 1.5B block shapes (T=8192, h=1600)."""
import sys, os
os.environ.setdefault('MOBIUS_KT_NOSYNC', '1')
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_asplos_fengxtwls23_b200 import BF16, kt
T, h = int(os.environ.get("ELEM_T", "16384")), 1600
def t(fn, it=20):
    for _ in range(3): fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(it): fn()
    b.record(); torch.cuda.synchronize()
    return a.elapsed_time(b) / it * 1e3
mk = lambda *s: torch.randn(*s, device="cuda").to(torch.bfloat16)
x, dy, dres, g, bb = mk(T, h), mk(T, h), mk(T, h), mk(h), mk(h)
y = torch.empty_like(x); dx = torch.empty_like(x)
mu = torch.empty(T, device="cuda"); rs = torch.empty(T, device="cuda")
dg = torch.zeros(h, device="cuda"); db = torch.zeros(h, device="cuda")
us = t(lambda: kt.layernorm_fwd(BF16, x, g, bb, y, mu, rs, T, h)); print(f"ln_fwd   {us:7.1f} us  {2*T*h*2/us/1e3:7.1f} GB/s")
us = t(lambda: kt.layernorm_bwd(BF16, dy, x, g, mu, rs, dres, dx, dg, db, T, h)); print(f"ln_bwd   {us:7.1f} us  {4*T*h*2/us/1e3:7.1f} GB/s (dx + param grads)")
for n in (h, 4 * h, 3 * h):
    X = mk(T, n); o = torch.zeros(n, device="cuda")
    us = t(lambda: kt.colsum(BF16, X, n, T, n, o)); print(f"colsum n={n:5d} {us:7.1f} us  {T*n*2/us/1e3:7.1f} GB/s")
# cold inputs: a fresh buffer set per call (larger than L2 in total), the in-step situation
NB = 6
xs = [mk(T, h) for _ in range(NB)]
ys = [torch.empty_like(x) for x in xs]
dys = [mk(T, h) for _ in range(NB)]
dxs = [torch.empty_like(x) for x in xs]
k = [0]
def nxt():
    k[0] = (k[0] + 1) % NB
    return k[0]
us = t(lambda: (lambda i: kt.layernorm_fwd(BF16, xs[i], g, bb, ys[i], mu, rs, T, h))(nxt()))
print(f"ln_fwd   cold {us:7.1f} us  {2*T*h*2/us/1e3:7.1f} GB/s")
us = t(lambda: (lambda i: kt.layernorm_bwd(BF16, dys[i], xs[i], g, mu, rs, dres, dxs[i], dg, db, T, h))(nxt()))
print(f"ln_bwd   cold {us:7.1f} us  {4*T*h*2/us/1e3:7.1f} GB/s (dx + param grads)")
# cross entropy over the LM-head logits of one microbatch (in place)
Vv, s_ = 50304, 1024
rows_ce = T
z = mk(rows_ce, Vv)
tok = torch.randint(0, Vv, (rows_ce // s_, s_ + 1), device="cuda", dtype=torch.int32)
lr_ = torch.empty(rows_ce, device="cuda")
us = t(lambda: kt.cross_entropy(BF16, z, tok, lr_, rows_ce, Vv, s_, 1.0 / rows_ce), it=5)
print(f"cross_entropy {us:7.1f} us  {2*rows_ce*Vv*2/us/1e3:7.1f} GB/s (1 read + 1 write of the logits)")
