import sys, os
sys.path.insert(0, os.getcwd())
import numpy as np
import synth
from oracle import model as om
from paper_conf_asplos_fengxtwls23_b200 import *
from tests.test_gpu_step import _arena_plan, tensor_errs, mk_cfg
c = synth.TINY; M = 2
for offload in (False, True):
  for sizes in [(1, 2, 1, 2), (2, 1, 2, 1)]:
    flags = FLAG_ARENA_CAP | (FLAG_CKPT_OFFLOAD if offload else 0)
    w = synth.round_bf16(synth.perturb_norm_params(c, synth.gen_params(c), scale=0.1))
    cfg, plan, cap = _arena_plan(c, BF16, sizes, M, ring_extra=64 << 10, flags=flags)
    tok1 = synth.gen_tokens(c, M, seed=31)
    ctx = MobiusContext(cfg, plan, init_params=w, flags=flags)
    l1 = ctx.step(tok1)
    g1 = ctx.read_grads(c.n_params)
    ctx.close()
    ref_l1, ref_g1 = om.reference_loss_and_grads(c, w, tok1)
    e = tensor_errs(c, g1, ref_g1)
    print(offload, sizes, abs(l1-ref_l1)/ref_l1, {k: round(v, 4) for k, v in e.items() if v > 0.02})
