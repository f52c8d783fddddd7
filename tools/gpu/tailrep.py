import sys, os
sys.path.insert(0, os.getcwd())
import numpy as np
import synth
from paper_conf_asplos_fengxtwls23_b200 import BF16, MobiusContext, plan_from_sizes, FLAG_DEVICE_TAIL_UPDATE
sys.path.insert(0, os.path.join(os.getcwd(), "tests"))
from test_gpu_step import mk_cfg
c = synth.TINY; M = 2
w = synth.round_bf16(synth.perturb_norm_params(c, synth.gen_params(c), scale=0.1))
toks = [synth.gen_tokens(c, M, seed=20 + i) for i in range(3)]
plan = plan_from_sizes((3, 3), 1, M, hbm_cap_bytes=4 << 20)
def run(flags):
    ctx = MobiusContext(mk_cfg(c, BF16), plan, init_params=w, flags=flags)
    for t in toks: ctx.step(t)
    p = ctx.read_params(c.n_params); ctx.close(); return p
rel = lambda a, b: float(np.linalg.norm(a - b) / np.linalg.norm(b))
ps = [run(0) for _ in range(3)] + [run(FLAG_DEVICE_TAIL_UPDATE) for _ in range(3)]
for i in range(6):
    print(i, [round(rel(ps[i] - w, ps[j] - w), 4) for j in range(6)])
