MOBIUS_LIB_PATH=tools/gpu/var/libmobius_MOBIUS_BWD_PROF1.so python - <<'PY' 2>&1 | grep "blk 0 " | grep "fmma\|fsmx" | sort
import os, sys
sys.path.insert(0, '.')
import torch
from paper_conf_asplos_fengxtwls23_b200 import BF16, kt
mbs, s, nh, dh = 32, 1024, 25, 64
def mk(*sh): return (torch.randn(*sh, device="cuda") * 0.5).to(torch.bfloat16)
qkv, o = mk(mbs*s, 3*nh*dh), mk(mbs*s, nh*dh)
kt.attention(BF16, mbs, s, nh, dh, qkv, o); torch.cuda.synchronize()
PY
