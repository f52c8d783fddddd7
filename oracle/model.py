"""GPT forward / backward, plain numpy (TEST INFRASTRUCTURE ONLY, see
oracle/__init__.py).

What it computes has a plain definition: the mean next-token cross-entropy
of a GPT-like model on a batch and its exact gradient.  Mobius only changes
where/when that gradient is computed (synchronous update "in the same way as
GPipe"), so the oracle is that definition written out.

Architecture (reading #1; the paper only says "GPT-like
Transformer based models", Table 3):
  x0 = Wte[tok] + Wpe[0..s-1]
  block: a = LN1(x); qkv = a Wqkv + bqkv; S = q k^T / sqrt(dh) (causal);
         P = softmax(S); o = P v; x1 = x + o Wo + bo;
         a2 = LN2(x1); u = a2 W1 + b1; y = x1 + gelu_tanh(u) W2 + b2
  head:  z = LN_f(x) Whead;  loss = (1/N_tok) sum_t [logsumexp(z_t) - z_t[target]]
LN(x) = g * (x - mu) / sqrt(var + 1e-5) + b, biased variance.
Backward uses the textbook formulas listed in SURVEY §8(c) O-2.

Every function takes a ``dtype`` implicitly from its inputs (fp32 for the
parity reference of the GPU paths, fp64 for the finite-difference pins).
"""
from __future__ import annotations

import math

import numpy as np

LN_EPS = 1e-5
GELU_C = math.sqrt(2.0 / math.pi)
GELU_A = 0.044715


# --------------------------------------------------------------------------
# parameter views
# --------------------------------------------------------------------------
def unpack_layer(cfg, flat: np.ndarray, i: int) -> dict:
    """Views into the flat oracle-layout vector for profile layer i."""
    offs = cfg.layer_offsets()
    pos = offs[i]
    out = {}
    for name, shape, _ in cfg.layer_specs(i):
        n = int(np.prod(shape))
        out[name] = flat[pos:pos + n].reshape(shape)
        pos += n
    assert pos == offs[i + 1]
    return out


def zeros_like_layer(cfg, i: int, dtype) -> dict:
    return {name: np.zeros(shape, dtype=dtype) for name, shape, _ in cfg.layer_specs(i)}


def pack_layers(cfg, layers: list, dtype=np.float32) -> np.ndarray:
    """Inverse of unpack_layer over all profile layers (dict per layer)."""
    parts = []
    for i in range(cfg.n_profile_layers):
        for name, shape, _ in cfg.layer_specs(i):
            parts.append(np.asarray(layers[i][name], dtype=dtype).reshape(-1))
    return np.concatenate(parts)


# --------------------------------------------------------------------------
# elementwise / row ops
# --------------------------------------------------------------------------
def layernorm_fwd(x, g, b):
    mu = x.mean(axis=-1, keepdims=True)
    var = ((x - mu) ** 2).mean(axis=-1, keepdims=True)
    rstd = 1.0 / np.sqrt(var + x.dtype.type(LN_EPS))
    xhat = (x - mu) * rstd
    return xhat * g + b, (xhat, rstd)


def layernorm_bwd(dy, g, cache):
    """dx = rstd (dyhat - mean(dyhat) - xhat mean(dyhat xhat)), dyhat = g dy."""
    xhat, rstd = cache
    dyhat = dy * g
    dx = rstd * (dyhat - dyhat.mean(axis=-1, keepdims=True)
                 - xhat * (dyhat * xhat).mean(axis=-1, keepdims=True))
    dg = (dy * xhat).reshape(-1, dy.shape[-1]).sum(axis=0)
    db = dy.reshape(-1, dy.shape[-1]).sum(axis=0)
    return dx, dg, db


def gelu_fwd(u):
    t = np.tanh(u.dtype.type(GELU_C) * (u + u.dtype.type(GELU_A) * u ** 3))
    return 0.5 * u * (1.0 + t)


def gelu_grad(u):
    """d/du of 0.5 u (1 + tanh(c (u + a u^3)))."""
    c = u.dtype.type(GELU_C)
    a = u.dtype.type(GELU_A)
    t = np.tanh(c * (u + a * u ** 3))
    return 0.5 * (1.0 + t) + 0.5 * u * (1.0 - t * t) * c * (1.0 + 3.0 * a * u * u)


def softmax_rows(s):
    m = s.max(axis=-1, keepdims=True)
    e = np.exp(s - m)
    return e / e.sum(axis=-1, keepdims=True)


# --------------------------------------------------------------------------
# attention core (K3/K4 in SURVEY §2.2)
# --------------------------------------------------------------------------
def split_heads(x, mbs, s, nh, dh):
    return x.reshape(mbs, s, nh, dh).transpose(0, 2, 1, 3)


def merge_heads(x):
    mbs, nh, s, dh = x.shape
    return x.transpose(0, 2, 1, 3).reshape(mbs * s, nh * dh)


def attention_fwd(qkv, mbs, s, nh):
    """qkv [T, 3h] with columns q|k|v, heads of dh contiguous columns (O-2)."""
    h = qkv.shape[1] // 3
    dh = h // nh
    q = split_heads(qkv[:, 0:h], mbs, s, nh, dh)
    k = split_heads(qkv[:, h:2 * h], mbs, s, nh, dh)
    v = split_heads(qkv[:, 2 * h:3 * h], mbs, s, nh, dh)
    scale = qkv.dtype.type(1.0 / math.sqrt(dh))
    S = (q @ k.transpose(0, 1, 3, 2)) * scale
    mask = np.triu(np.ones((s, s), dtype=bool), k=1)       # j > i masked
    S = np.where(mask, -np.inf, S)
    P = softmax_rows(S)
    o = P @ v
    return merge_heads(o), (q, k, v, P)


def attention_bwd(do, cache, mbs, s, nh):
    q, k, v, P = cache
    dh = q.shape[-1]
    scale = q.dtype.type(1.0 / math.sqrt(dh))
    do4 = split_heads(do, mbs, s, nh, dh)
    dP = do4 @ v.transpose(0, 1, 3, 2)
    dv = P.transpose(0, 1, 3, 2) @ do4
    dS = P * (dP - (dP * P).sum(axis=-1, keepdims=True))   # masked P = 0 -> dS = 0
    dq = (dS @ k) * scale
    dk = (dS.transpose(0, 1, 3, 2) @ q) * scale
    return np.concatenate([merge_heads(dq), merge_heads(dk), merge_heads(dv)], axis=1)


# --------------------------------------------------------------------------
# layers
# --------------------------------------------------------------------------
def embed_fwd(cfg, p, tok):
    """tok [mbs, s] int -> x0 [mbs*s, h]."""
    mbs, s = tok.shape
    x = p["wte"][tok.reshape(-1)] + np.tile(p["wpe"][:s], (mbs, 1))
    return x, tok


def embed_bwd(cfg, p, dx, tok):
    mbs, s = tok.shape
    g = {"wte": np.zeros_like(p["wte"]), "wpe": np.zeros_like(p["wpe"])}
    np.add.at(g["wte"], tok.reshape(-1), dx)
    g["wpe"][:s] += dx.reshape(mbs, s, -1).sum(axis=0)
    return g


def block_fwd(cfg, p, x, mbs):
    s, nh = cfg.seq_len, cfg.n_heads
    a, c_ln1 = layernorm_fwd(x, p["ln1_g"], p["ln1_b"])
    qkv = a @ p["w_qkv"] + p["b_qkv"]
    o, c_att = attention_fwd(qkv, mbs, s, nh)
    x1 = x + o @ p["w_o"] + p["b_o"]
    a2, c_ln2 = layernorm_fwd(x1, p["ln2_g"], p["ln2_b"])
    u = a2 @ p["w_1"] + p["b_1"]
    gu = gelu_fwd(u)
    y = x1 + gu @ p["w_2"] + p["b_2"]
    return y, (a, c_ln1, o, c_att, a2, c_ln2, u, gu)


def block_bwd(cfg, p, dy, cache, mbs):
    s, nh = cfg.seq_len, cfg.n_heads
    a, c_ln1, o, c_att, a2, c_ln2, u, gu = cache
    g = {}
    # MLP
    g["w_2"] = gu.T @ dy
    g["b_2"] = dy.sum(axis=0)
    dgu = dy @ p["w_2"].T
    du = dgu * gelu_grad(u)
    g["w_1"] = a2.T @ du
    g["b_1"] = du.sum(axis=0)
    da2 = du @ p["w_1"].T
    dx1_ln, g["ln2_g"], g["ln2_b"] = layernorm_bwd(da2, p["ln2_g"], c_ln2)
    dx1 = dy + dx1_ln
    # attention
    g["w_o"] = o.T @ dx1
    g["b_o"] = dx1.sum(axis=0)
    do = dx1 @ p["w_o"].T
    dqkv = attention_bwd(do, c_att, mbs, s, nh)
    g["w_qkv"] = a.T @ dqkv
    g["b_qkv"] = dqkv.sum(axis=0)
    da = dqkv @ p["w_qkv"].T
    dx_ln, g["ln1_g"], g["ln1_b"] = layernorm_bwd(da, p["ln1_g"], c_ln1)
    dx = dx1 + dx_ln
    return dx, g


def head_fwd_bwd(cfg, p, x, targets, n_tok_total):
    """LN_f + LM head + mean CE (scaled by the GLOBAL token count of the
    step, so that microbatch gradients add up to the full-batch gradient).
    Returns (loss_sum, dx, grads)."""
    a, c_ln = layernorm_fwd(x, p["lnf_g"], p["lnf_b"])
    z = a @ p["w_head"]
    m = z.max(axis=-1, keepdims=True)
    e = np.exp(z - m)
    se = e.sum(axis=-1, keepdims=True)
    lse = (m + np.log(se))[:, 0]
    t = targets.reshape(-1)
    rows = np.arange(z.shape[0])
    loss_sum = float((lse - z[rows, t]).astype(np.float64).sum())
    dz = e / se
    dz[rows, t] -= 1.0
    dz = dz * z.dtype.type(1.0 / n_tok_total)
    g = {"w_head": a.T @ dz}
    da = dz @ p["w_head"].T
    dx, g["lnf_g"], g["lnf_b"] = layernorm_bwd(da, p["lnf_g"], c_ln)
    return loss_sum, dx, g


def head_loss(cfg, p, x, targets):
    a, _ = layernorm_fwd(x, p["lnf_g"], p["lnf_b"])
    z = a @ p["w_head"]
    m = z.max(axis=-1, keepdims=True)
    lse = (m + np.log(np.exp(z - m).sum(axis=-1, keepdims=True)))[:, 0]
    t = targets.reshape(-1)
    return float((lse - z[np.arange(z.shape[0]), t]).astype(np.float64).sum())


# --------------------------------------------------------------------------
# layer dispatch (profile layers: 0 = embed, 1..L = blocks, L+1 = head)
# --------------------------------------------------------------------------
def layer_fwd(cfg, i, p, x, tok, mbs):
    if i == 0:
        return embed_fwd(cfg, p, tok)
    if i <= cfg.n_layers:
        return block_fwd(cfg, p, x, mbs)
    raise ValueError("head is fused fwd+bwd (head_fwd_bwd)")


# --------------------------------------------------------------------------
# O-5 reference step: no partition, microbatches m ascending
# --------------------------------------------------------------------------
def reference_loss_and_grads(cfg, flat_params, tokens, dtype=np.float32):
    """Unpartitioned step (K = 1, N = 1): loss (mean over M*mbs*s tokens) and
    the flat gradient in oracle layout.  dW accumulated over m ascending
    (reading #22)."""
    flat = np.asarray(flat_params, dtype=dtype)
    M, mbs, _ = tokens.shape
    Lp = cfg.n_profile_layers
    n_tok = M * mbs * cfg.seq_len
    P = [unpack_layer(cfg, flat, i) for i in range(Lp)]
    G = [None] * Lp
    loss_sum = 0.0
    for m in range(M):
        tok = tokens[m, :, :-1]
        tgt = tokens[m, :, 1:]
        caches = [None] * Lp
        x, caches[0] = embed_fwd(cfg, P[0], tok)
        for i in range(1, cfg.n_layers + 1):
            x, caches[i] = block_fwd(cfg, P[i], x, mbs)
        ls, dx, gh = head_fwd_bwd(cfg, P[Lp - 1], x, tgt, n_tok)
        loss_sum += ls
        grads_m = [None] * Lp
        grads_m[Lp - 1] = gh
        for i in range(cfg.n_layers, 0, -1):
            dx, grads_m[i] = block_bwd(cfg, P[i], dx, caches[i], mbs)
        grads_m[0] = embed_bwd(cfg, P[0], dx, caches[0])
        for i in range(Lp):
            if G[i] is None:
                G[i] = {k: v.copy() for k, v in grads_m[i].items()}
            else:
                for k in G[i]:
                    G[i][k] = G[i][k] + grads_m[i][k]
    return loss_sum / n_tok, pack_layers(cfg, G, dtype=dtype)


def reference_loss(cfg, flat_params, tokens, dtype=np.float64):
    """Loss only (for finite differences)."""
    flat = np.asarray(flat_params, dtype=dtype)
    M, mbs, _ = tokens.shape
    Lp = cfg.n_profile_layers
    P = [unpack_layer(cfg, flat, i) for i in range(Lp)]
    total = 0.0
    for m in range(M):
        x, _ = embed_fwd(cfg, P[0], tokens[m, :, :-1])
        for i in range(1, cfg.n_layers + 1):
            x, _ = block_fwd(cfg, P[i], x, mbs)
        total += head_loss(cfg, P[Lp - 1], x, tokens[m, :, 1:])
    return total / (M * mbs * cfg.seq_len)
