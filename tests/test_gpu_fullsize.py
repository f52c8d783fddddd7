"""Full-size checks (BASELINE configs[1] GPT-1.5B and configs[2] GPT-13B
shapes) in the launch configuration bench.py uses.

* one transformer block fwd+bwd at the full hidden size / sequence length
  against the oracle (numpy fp32 on the host, tens of seconds), rel 2e-2;
* the LM head + CE at V = 50304 against the oracle;
* the whole 48-layer 1.5B step with the planner's partition under the 1 GiB
  stage cap: properties that hold at any size - schedule trace == Fig-4
  queue of the plan, H2D/D2H byte counters == O-10 of the plan, initial
  loss ~ log V + h*0.02^2/2, loss decreasing on a fixed batch.
"""
import math

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a GPU", allow_module_level=True)

import synth  # noqa: E402
from oracle import model as om  # noqa: E402
from oracle import planner as op  # noqa: E402
from oracle import schedule as osch  # noqa: E402
from paper_conf_asplos_fengxtwls23_b200 import (BF16, MobiusContext, kt, make_topology, mobius_layer_sizes,  # noqa: E402
                                                mobius_plan, mobius_profile, model_cfg)

DEV = "cuda:0"


def rel(a, b):
    a = np.asarray(a, np.float64).reshape(-1)
    b = np.asarray(b, np.float64).reshape(-1)
    return float(np.linalg.norm(a - b) / max(np.linalg.norm(b), 1e-30))


def to_dev(x):
    return torch.from_numpy(np.ascontiguousarray(x, dtype=np.float32)).to(DEV).to(torch.bfloat16)


def from_dev(t):
    return t.float().cpu().numpy()


@pytest.mark.parametrize("name", ["1.5b", "13b"])
def test_block_full_size(name):
    base = synth.CONFIGS[name]
    cfg = synth.GPTConfig(n_layers=base.n_layers, hidden=base.hidden, n_heads=base.n_heads, seq_len=base.seq_len,
                          vocab=64, micro_batch=1)
    rng = np.random.default_rng(3)
    p = {}
    for nm, shape, init in cfg.layer_specs(1):
        if init == "normal":
            v = rng.standard_normal(shape) * 0.02
        elif init == "normal_proj":
            v = rng.standard_normal(shape) * 0.02 / math.sqrt(2 * cfg.n_layers)
        elif init == "ones":
            v = 1 + 0.1 * rng.standard_normal(shape)
        else:
            v = 0.1 * rng.standard_normal(shape)
        p[nm] = synth.round_bf16(v.astype(np.float32))
    flat = np.concatenate([p[nm].reshape(-1) for nm, _, _ in cfg.layer_specs(1)])
    T, h = cfg.seq_len, cfg.hidden
    x = synth.round_bf16(rng.standard_normal((T, h)).astype(np.float32))
    dy = synth.round_bf16((rng.standard_normal((T, h)) * 1e-3).astype(np.float32))
    y_ref, cache = om.block_fwd(cfg, p, x, 1)
    dx_ref, g_ref = om.block_bwd(cfg, p, dy, cache, 1)
    tx, tdy = to_dev(x), to_dev(dy)
    ty, tdx = torch.empty_like(tx), torch.empty_like(tx)
    grads = torch.zeros(flat.size, device=DEV)
    kt.block(BF16, h, cfg.n_heads, T, 1, to_dev(flat), tx, ty, tdy, tdx, grads)
    torch.cuda.synchronize()
    errs = {"y": rel(from_dev(ty), y_ref), "dx": rel(from_dev(tdx), dx_ref)}
    G = from_dev(grads)
    pos = 0
    for nm, shape, _ in cfg.layer_specs(1):
        n = int(np.prod(shape))
        errs[nm] = rel(G[pos:pos + n], g_ref[nm])
        pos += n
    assert max(errs.values()) < 2e-2, errs


def test_head_full_vocab():
    """LM head GEMM + fused CE at V = 50304 (K9) vs the oracle."""
    V, h, s = 50304, 1600, 256
    rng = np.random.default_rng(5)
    a = synth.round_bf16(rng.standard_normal((s, h)).astype(np.float32))
    W = synth.round_bf16((rng.standard_normal((h, V)) * 0.02).astype(np.float32))
    tok = rng.integers(0, V, size=(1, s + 1)).astype(np.int32)
    z = a.astype(np.float64) @ W.astype(np.float64)
    m = z.max(-1, keepdims=True)
    e = np.exp(z - m)
    lse = (m + np.log(e.sum(-1, keepdims=True)))[:, 0]
    loss_ref = lse - z[np.arange(s), tok[0, 1:]]
    tz = torch.empty((s, V), device=DEV, dtype=torch.bfloat16)
    kt.gemm(BF16, s, V, h, to_dev(a), h, False, to_dev(W), V, True, tz, V)
    lr = torch.empty(s, device=DEV)
    kt.cross_entropy(BF16, tz, torch.from_numpy(tok).to(DEV), lr, s, V, s, 1.0 / s)
    torch.cuda.synchronize()
    assert rel(from_dev(lr), loss_ref) < 2e-3


def test_full_1p5b_step_properties():
    c = synth.GPT_1_5B
    M = 4
    cfg = model_cfg(c.n_layers, c.hidden, c.n_heads, c.seq_len, c.vocab, c.micro_batch, dtype=BF16)
    prof = mobius_profile(cfg, 0)
    plan = mobius_plan(prof, 1, 1 << 30, M, make_topology([0], 55 * 10 ** 9, 0))
    K = plan.n_stages
    assert K >= 4  # the 1 GiB cap forces DRAM swaps of a 3.1 GB model
    ctx = MobiusContext(cfg, plan, seed=1234)
    tok = synth.gen_tokens(c, M)
    l1 = ctx.step(tok)
    trace = ctx.read_trace()
    st = ctx.stats()
    l2 = ctx.step(tok)
    l3 = ctx.step(tok)
    l4 = ctx.step(tok)
    ctx.close()
    # at init LN_f(x) has unit-variance entries, so the logits are
    # ~N(0, h * 0.02^2) and E[CE] = log V + sigma^2 / 2 (lognormal mean)
    expect = math.log(c.vocab) + c.hidden * 0.02 ** 2 / 2
    assert abs(l1 - expect) < 0.05, (l1, expect)
    # training signal: Adam's sign-like first updates (every weight moves by
    # ~lr) overshoot on step 3 for this init and lr (measured 11.147, 11.007,
    # 11.18, 10.84 with every GEMM / optimizer variant), so check the trend
    assert l2 < l1 and l4 < l2 and np.isfinite(l3), (l1, l2, l3, l4)
    sizes = [plan.stage_first_layer[j + 1] - plan.stage_first_layer[j] for j in range(K)]
    sg = [0] * K
    assert trace == osch.per_gpu_ops(sg, M)[0]
    sz = mobius_layer_sizes(cfg)
    layers = [op.LayerProfile(0, 0, p.mem_fwd, p.mem_bwd, p.xfer_fwd, p.xfer_bwd, p.act_out) for p in sz]
    ss = op.stage_sums(layers, sizes)
    h2d, d2h, _ = osch.byte_counts(ss, sg, M, [s["Xf"] for s in ss], n_gpus=1)
    assert st.h2d_bytes == h2d[0] == plan.h2d_bytes[0]
    assert st.d2h_bytes == d2h[0]


def test_bench_launch_config_step_properties():
    """The bench's launch configuration (BASELINE configs[1], bench.py
    defaults): GPT-1.5B, mbs 32 x M 4, 1 GiB stage ring, kept activations
    and the device tail update.  Properties that hold at this size: the init
    loss equals its closed form, the loss falls, the schedule trace is Fig 4's,
    and every stage byte the paper's O-10 count moves over the host link
    either still does or (first stage, from step 2) is served device-to-device."""
    import dataclasses
    from paper_conf_asplos_fengxtwls23_b200 import FLAG_DEVICE_TAIL_UPDATE, FLAG_KEEP_ACTS
    c = dataclasses.replace(synth.GPT_1_5B, micro_batch=32)
    M = 4
    cfg = model_cfg(c.n_layers, c.hidden, c.n_heads, c.seq_len, c.vocab, c.micro_batch, dtype=BF16)
    prof = mobius_profile(cfg, 0)
    plan = mobius_plan(prof, 1, 1 << 30, M, make_topology([0], 55 * 10 ** 9, 0))
    K = plan.n_stages
    ctx = MobiusContext(cfg, plan, seed=1234, flags=FLAG_KEEP_ACTS | FLAG_DEVICE_TAIL_UPDATE)
    tok = synth.gen_tokens(c, M)
    l1 = ctx.step(tok)
    trace = ctx.read_trace()
    st1 = ctx.stats()
    l2 = ctx.step(tok)
    st2 = ctx.stats()
    l3 = ctx.step(tok)
    ctx.close()
    expect = math.log(c.vocab) + c.hidden * 0.02 ** 2 / 2
    assert abs(l1 - expect) < 0.05, (l1, expect)
    assert l2 < l1 and np.isfinite(l3), (l1, l2, l3)
    assert trace == osch.per_gpu_ops([0] * K, M)[0]
    sizes = [plan.stage_first_layer[j + 1] - plan.stage_first_layer[j] for j in range(K)]
    sz = mobius_layer_sizes(cfg)
    layers = [op.LayerProfile(0, 0, p.mem_fwd, p.mem_bwd, p.xfer_fwd, p.xfer_bwd, p.act_out) for p in sz]
    ss = op.stage_sums(layers, sizes)
    h2d, d2h, _ = osch.byte_counts(ss, [0] * K, M, [s["Xf"] for s in ss], n_gpus=1)
    assert st1.h2d_bytes == h2d[0] and st1.d2d_bytes == 0
    assert st2.h2d_bytes + st2.d2d_bytes == h2d[0] and st2.d2d_bytes > 0
    assert st1.recompute <= 2  # nearly every block's activations kept (reading #17)
