"""Time the flash attention fwd / bwd kernels (CUDA events, back to back).
usage: python tools/flash_time.py [dh] [mbs] [s] [nh]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ.setdefault("MOBIUS_KT_NOSYNC", "1")
import torch  # noqa: E402
from paper_conf_asplos_fengxtwls23_b200 import BF16, kt  # noqa: E402

dh = int(sys.argv[1]) if len(sys.argv) > 1 else 64
mbs = int(sys.argv[2]) if len(sys.argv) > 2 else 8
s = int(sys.argv[3]) if len(sys.argv) > 3 else 1024
nh = int(sys.argv[4]) if len(sys.argv) > 4 else 1600 // dh


def mk(*sh):
    return (torch.randn(*sh, device="cuda") * 0.5).to(torch.bfloat16)


qkv, o, do, dq = mk(mbs * s, 3 * nh * dh), mk(mbs * s, nh * dh), mk(mbs * s, nh * dh), mk(mbs * s, 3 * nh * dh)


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
    return a.elapsed_time(b) / it


f = t(lambda: kt.attention(BF16, mbs, s, nh, dh, qkv, o))
fb = t(lambda: kt.attention(BF16, mbs, s, nh, dh, qkv, o, do, dq))
fl = 2.0 * mbs * nh * s * s * dh  # causal fwd algorithmic (2 GEMMs x half)
print(f"dh={dh} mbs={mbs} s={s} nh={nh}: fwd {f*1e3:.1f} us ({fl/f/1e9:.0f} TF/s), "
      f"bwd {(fb-f)*1e3:.1f} us ({2.5*fl/(fb-f)/1e9:.0f} TF/s)")
