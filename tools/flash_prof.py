import sys, os
os.environ.setdefault('MOBIUS_KT_NOSYNC', '1')
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_asplos_fengxtwls23_b200 import BF16, kt
mbs, s, nh, dh = 8, 1024, 25, 64
mk = lambda *sh: (torch.randn(*sh, device="cuda") * 0.5).to(torch.bfloat16)
qkv = mk(mbs * s, 3 * nh * dh); o = mk(mbs * s, nh * dh); do = mk(mbs * s, nh * dh); dq = mk(mbs * s, 3 * nh * dh)
for _ in range(int(sys.argv[1]) if len(sys.argv) > 1 else 2):
    kt.attention(BF16, mbs, s, nh, dh, qkv, o, do, dq)
torch.cuda.synchronize()
