"""Pins for oracle/model.py (SURVEY §8(c) "What pins each part", block and
model fwd/bwd): finite differences in fp64, an independent torch fp64
autograd implementation of the same equations, closed forms, and
microbatching invariance.  CPU only."""
import math

import numpy as np
import pytest
import torch
import torch.nn.functional as F

import synth
from oracle import model as om

CFG = synth.MICRO


def _params(cfg, seed=1234):
    p = synth.gen_params(cfg, seed).astype(np.float64)
    # non-trivial LN gains/biases and linear biases so that every term of
    # the gradient is exercised (a dropped bias/gain term must fail)
    return synth.perturb_norm_params(cfg, p.astype(np.float32), scale=0.2).astype(np.float64) * 1.0


def _tokens(cfg, M):
    return synth.gen_tokens(cfg, M)


@pytest.mark.parametrize("M", [1, 2])
def test_finite_differences_fp64(M):
    cfg = CFG
    w = _params(cfg)
    # larger weights so the model is far from linear
    w = w * 5.0
    tok = _tokens(cfg, M)
    loss, g = om.reference_loss_and_grads(cfg, w, tok, dtype=np.float64)
    assert abs(loss - om.reference_loss(cfg, w, tok)) < 1e-12
    rng = np.random.default_rng(7)
    eps = 1e-6
    # one random direction restricted to each tensor, plus two global ones
    offs = cfg.layer_offsets()
    dirs = []
    for i in range(cfg.n_profile_layers):
        pos = offs[i]
        for name, shape, _ in cfg.layer_specs(i):
            n = int(np.prod(shape))
            d = np.zeros_like(w)
            d[pos:pos + n] = rng.standard_normal(n)
            dirs.append((f"L{i}.{name}", d))
            pos += n
    for k in range(2):
        dirs.append((f"global{k}", rng.standard_normal(w.shape)))
    for name, d in dirs:
        fd = (om.reference_loss(cfg, w + eps * d, tok) - om.reference_loss(cfg, w - eps * d, tok)) / (2 * eps)
        an = float(g @ d)
        assert abs(an - fd) <= 1e-7 * max(1.0, abs(fd)) + 1e-9, (name, an, fd)


def _torch_model_loss(cfg, flat, tok):
    """Independent torch implementation of the same GPT (library ops:
    F.layer_norm, F.gelu(tanh), F.scaled_dot_product_attention(causal),
    F.cross_entropy)."""
    L, h, nh, s = cfg.n_layers, cfg.hidden, cfg.n_heads, cfg.seq_len
    dh = h // nh
    offs = cfg.layer_offsets()

    def get(i):
        pos = offs[i]
        out = {}
        for name, shape, _ in cfg.layer_specs(i):
            n = int(np.prod(shape))
            out[name] = flat[pos:pos + n].view(*shape)
            pos += n
        return out

    M, mbs, _ = tok.shape
    total = 0.0
    for m in range(M):
        inp = torch.as_tensor(tok[m, :, :-1], dtype=torch.long)
        tgt = torch.as_tensor(tok[m, :, 1:], dtype=torch.long)
        e = get(0)
        x = e["wte"][inp] + e["wpe"][:s][None]
        for i in range(1, L + 1):
            p = get(i)
            a = F.layer_norm(x, (h,), p["ln1_g"], p["ln1_b"], eps=1e-5)
            qkv = a @ p["w_qkv"] + p["b_qkv"]
            q, k, v = qkv.split(h, dim=-1)
            q = q.view(mbs, s, nh, dh).transpose(1, 2)
            k = k.view(mbs, s, nh, dh).transpose(1, 2)
            v = v.view(mbs, s, nh, dh).transpose(1, 2)
            o = F.scaled_dot_product_attention(q, k, v, is_causal=True)
            o = o.transpose(1, 2).reshape(mbs, s, h)
            x = x + o @ p["w_o"] + p["b_o"]
            a2 = F.layer_norm(x, (h,), p["ln2_g"], p["ln2_b"], eps=1e-5)
            x = x + F.gelu(a2 @ p["w_1"] + p["b_1"], approximate="tanh") @ p["w_2"] + p["b_2"]
        hd = get(L + 1)
        a = F.layer_norm(x, (h,), hd["lnf_g"], hd["lnf_b"], eps=1e-5)
        z = a @ hd["w_head"]
        total = total + F.cross_entropy(z.reshape(-1, z.shape[-1]), tgt.reshape(-1), reduction="sum")
    return total / (M * mbs * s)


@pytest.mark.parametrize("cfgname,M", [("micro", 2), ("micro", 3)])
def test_torch_fp64_autograd(cfgname, M):
    cfg = synth.CONFIGS[cfgname]
    w = _params(cfg) * 3.0
    tok = _tokens(cfg, M)
    loss, g = om.reference_loss_and_grads(cfg, w, tok, dtype=np.float64)
    tw = torch.tensor(w, dtype=torch.float64, requires_grad=True)
    tl = _torch_model_loss(cfg, tw, tok)
    tl.backward()
    assert abs(loss - tl.item()) <= 1e-12 * abs(loss)
    tg = tw.grad.numpy()
    assert np.linalg.norm(g - tg) <= 1e-11 * np.linalg.norm(tg)
    # per tensor too (a transposed operand in a small tensor must not hide)
    offs = cfg.layer_offsets()
    for i in range(cfg.n_profile_layers):
        pos = offs[i]
        for name, shape, _ in cfg.layer_specs(i):
            n = int(np.prod(shape))
            a, b = g[pos:pos + n], tg[pos:pos + n]
            assert np.allclose(a, b, rtol=1e-9, atol=1e-14), (i, name)
            pos += n


def test_closed_forms():
    rng = np.random.default_rng(0)
    # LN output has zero mean and unit (biased) variance with g=1, b=0
    x = rng.standard_normal((5, 64)) * 3 + 2
    y, _ = om.layernorm_fwd(x, np.ones(64), np.zeros(64))
    assert np.allclose(y.mean(-1), 0, atol=1e-12)
    assert np.allclose(y.var(-1), 1 / (1 + 1e-5 / x.var(-1)), rtol=1e-12)
    # GeLU: gelu(0) = 0, gelu'(0) = 1/2, large-u asymptotes, matches torch
    assert om.gelu_fwd(np.array([0.0]))[0] == 0.0
    assert om.gelu_grad(np.array([0.0]))[0] == 0.5
    u = np.linspace(-6, 6, 101)
    assert np.allclose(om.gelu_fwd(u), F.gelu(torch.tensor(u), approximate="tanh").numpy(), rtol=1e-14, atol=1e-15)
    assert np.allclose(om.gelu_grad(np.array([30.0, -30.0])), [1.0, 0.0])
    # seq len 1: attention output = v (softmax of one element is 1)
    mbs, s, nh, dh = 3, 1, 2, 4
    qkv = rng.standard_normal((mbs * s, 3 * nh * dh))
    o, _ = om.attention_fwd(qkv, mbs, s, nh)
    assert np.array_equal(o, qkv[:, 2 * nh * dh:])
    # causal: row 0 attends only to itself
    s = 5
    qkv = rng.standard_normal((mbs * s, 3 * nh * dh))
    o, (q, k, v, P) = om.attention_fwd(qkv, mbs, s, nh)
    assert np.allclose(np.triu(P[0, 0], 1), 0)
    assert np.allclose(P.sum(-1), 1)
    assert np.allclose(o.reshape(mbs, s, nh, dh)[:, 0], qkv[:, 2 * nh * dh:].reshape(mbs, s, nh, dh)[:, 0])
    # CE gradient = (softmax - onehot)/N through the head with identity LN and
    # identity-ish projection: check dz directly via a 1-token case
    cfg = synth.GPTConfig(n_layers=1, hidden=4, n_heads=1, seq_len=1, vocab=4, micro_batch=1)
    p = {"lnf_g": np.ones(4), "lnf_b": np.zeros(4), "w_head": np.eye(4)}
    x = np.array([[1.0, -1.0, 2.0, 0.5]])
    ls, dx, g = om.head_fwd_bwd(cfg, p, x, np.array([[2]]), 1)
    a, _ = om.layernorm_fwd(x, p["lnf_g"], p["lnf_b"])
    sm = np.exp(a[0]) / np.exp(a[0]).sum()
    assert abs(ls - (np.log(np.exp(a[0]).sum()) - a[0, 2])) < 1e-14
    onehot = np.eye(4)[2]
    assert np.allclose(g["w_head"], np.outer(a[0], sm - onehot))


def test_microbatch_invariance_fp32():
    """M x mbs vs 1 x (M*mbs): same tokens, same gradient up to fp32
    rounding (microbatching does not change the update)."""
    cfg = synth.GPTConfig(n_layers=2, hidden=32, n_heads=2, seq_len=16, vocab=64, micro_batch=2)
    w = synth.perturb_norm_params(cfg, synth.gen_params(cfg), scale=0.2)
    tok = synth.gen_tokens(cfg, 3)
    l1, g1 = om.reference_loss_and_grads(cfg, w, tok)
    cfg6 = synth.GPTConfig(n_layers=2, hidden=32, n_heads=2, seq_len=16, vocab=64, micro_batch=6)
    l2, g2 = om.reference_loss_and_grads(cfg6, w, tok.reshape(1, 6, -1))
    assert abs(l1 - l2) <= 1e-6 * abs(l2)
    assert np.linalg.norm(g1 - g2) <= 1e-5 * np.linalg.norm(g2)


def test_pack_roundtrip_and_layout():
    cfg = synth.TINY
    w = synth.gen_params(cfg)
    assert w.size == cfg.n_params
    layers = [om.unpack_layer(cfg, w, i) for i in range(cfg.n_profile_layers)]
    assert np.array_equal(om.pack_layers(cfg, layers), w)
    # 12 h^2 + 13 h params per block
    h = cfg.hidden
    assert cfg.layer_numel(1) == 12 * h * h + 13 * h
    # initial LN gains are 1, biases 0 (O-1)
    assert np.all(layers[1]["ln1_g"] == 1) and np.all(layers[1]["b_qkv"] == 0)
    assert abs(layers[1]["w_o"].std() - 0.02 / math.sqrt(2 * cfg.n_layers)) < 2e-3 * 0.02
