"""Time the tcgen05 GEMM / flash kernels at the 1.5B block shapes (kernel-level
perf loop; not part of the bench contract)."""
import sys, os
os.environ.setdefault('MOBIUS_KT_NOSYNC', '1')
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_asplos_fengxtwls23_b200 import BF16, kt

T, h, V = 8192, int(sys.argv[1]) if len(sys.argv) > 1 else 1600, 50304
dev = "cuda"
def t(fn, it=10):
    for _ in range(3): fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(it): fn()
    b.record(); torch.cuda.synchronize()
    return a.elapsed_time(b) / it

def mk(*s): return (torch.randn(*s, device=dev) * 0.1).to(torch.bfloat16)
shapes = [  # name, M, N, K, a_mn, b_mn, epi, c_f32
    ("qkv fwd", T, 3*h, h, 0, 1, 1, 0), ("o fwd +res", T, h, h, 0, 1, 3, 0), ("fc1 fwd +gelu", T, 4*h, h, 0, 1, 2, 0),
    ("fc2 fwd +res", T, h, 4*h, 0, 1, 3, 0), ("fc2 dX gelu'", T, 4*h, h, 0, 0, 4, 0), ("fc1 dX", T, h, 4*h, 0, 0, 0, 0),
    ("qkv dX", T, h, 3*h, 0, 0, 0, 0), ("fc1 dW", h, 4*h, T, 1, 1, 5, 1), ("fc2 dW", 4*h, h, T, 1, 1, 5, 1),
    ("qkv dW", h, 3*h, T, 1, 1, 5, 1), ("head fwd", T, V, h, 0, 1, 0, 0), ("head dX", T, h, V, 0, 0, 0, 0),
    ("head dW", h, V, T, 1, 1, 5, 1)]
tot_ms = 0; tot_fl = 0
for name, M, N, K, amn, bmn, epi, cf in shapes:
    A = mk(K, M) if amn else mk(M, K)
    B = mk(K, N) if bmn else mk(N, K)
    C = torch.zeros(M, N, device=dev, dtype=torch.float32 if cf else torch.bfloat16)
    bias = mk(N); R = mk(M, N); AUX = mk(M, N)
    f = lambda: kt.gemm(BF16, M, N, K, A, M if amn else K, amn, B, N if bmn else K, bmn, C, N, c_f32=bool(cf), epi=epi,
                        bias=bias if epi in (1, 2, 3) else None, R=R if epi in (3, 4) else None, ldr=N,
                        AUX=AUX if epi == 2 else None, ldx=N, accumulate=(epi == 5))
    ms = t(f)
    fl = 2.0 * M * N * K
    tot_ms += ms; tot_fl += fl
    print(f"{name:16s} {M:6d}x{N:6d}x{K:6d}  {ms*1e3:8.1f} us  {fl/ms/1e9:7.1f} TF/s")
print(f"total {tot_ms:.3f} ms  {tot_fl/tot_ms/1e9:.1f} TF/s")
for mbs, s, nh, dh in ((8, 1024, h // 64, 64),):
    qkv = mk(mbs * s, 3 * nh * dh); o = mk(mbs * s, nh * dh); do = mk(mbs * s, nh * dh); dq = mk(mbs * s, 3 * nh * dh)
    ms_f = t(lambda: kt.attention(BF16, mbs, s, nh, dh, qkv, o))
    ms_fb = t(lambda: kt.attention(BF16, mbs, s, nh, dh, qkv, o, do, dq))
    fl = 2.0 * mbs * nh * s * s * dh  # causal fwd algorithmic
    print(f"flash fwd mbs={mbs} s={s} nh={nh} dh={dh}: {ms_f*1e3:.1f} us ({fl/ms_f/1e9:.1f} TF/s); fwd+bwd {ms_fb*1e3:.1f} us (bwd {(ms_fb-ms_f)*1e3:.1f} us, {2*fl/(ms_fb-ms_f)/1e9:.1f} TF/s)")
