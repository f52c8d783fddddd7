MOBIUS_LIB_PATH=tools/gpu/var/libmobius_MOBIUS_BWD_PROF1.so python - <<'PY' 2>&1 | grep "blk 0 " | sort
import os, sys
sys.path.insert(0, '.')
import torch
from paper_conf_asplos_fengxtwls23_b200 import BF16, kt
mbs, s, nh, dh = 32, 1024, 25, 64
def mk(*sh): return (torch.randn(*sh, device="cuda") * 0.5).to(torch.bfloat16)
qkv, o, do, dq = mk(mbs*s, 3*nh*dh), mk(mbs*s, nh*dh), mk(mbs*s, nh*dh), mk(mbs*s, 3*nh*dh)
kt.attention(BF16, mbs, s, nh, dh, qkv, o, do, dq); torch.cuda.synchronize()
PY
