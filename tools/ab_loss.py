import os, sys, math
sys.path.insert(0, os.getcwd())
import numpy as np, synth
from paper_conf_asplos_fengxtwls23_b200 import BF16, MobiusContext, make_topology, mobius_plan, mobius_profile, model_cfg
c = synth.GPT_1_5B; M = 4
cfg = model_cfg(c.n_layers, c.hidden, c.n_heads, c.seq_len, c.vocab, c.micro_batch, dtype=BF16)
prof = mobius_profile(cfg, 0)
plan = mobius_plan(prof, 1, 1 << 30, M, make_topology([0], 55 * 10 ** 9, 0))
ctx = MobiusContext(cfg, plan, seed=1234)
tok = synth.gen_tokens(c, M)
print(os.environ.get("TAG"), [round(ctx.step(tok), 4) for _ in range(5)], flush=True)
ctx.close()
