"""Seeded synthetic inputs shared by the oracle, the tests and bench.py.

This module holds NO arithmetic of the method (no model math, no schedule,
no planner).  It only defines

* the model configurations of BASELINE.json ``configs`` (GPT shapes),
* the flat parameter layout ("oracle layout") both sides agree on, i.e. the
  list of tensors and their shapes in packing order,
* the seeded draws of SURVEY.md §8(c) O-1 (weights ~ N(0, 0.02^2), tokens
  ~ U{0..V-1}), and the bf16 round-to-nearest-even the harness applies
  before handing weights to the bf16 path (so that parity measures compute
  error only).

The paper describes the workloads only as "GPT-like Transformer based models
with different hidden dimensions and number of layers" (PAPER.md L929-931,
Table 3); the block architecture reading is SURVEY.md §8(c) #1.
"""
from __future__ import annotations

import dataclasses
import math

import numpy as np

SEED_W = 1234
SEED_TOK = 5678


@dataclasses.dataclass(frozen=True)
class GPTConfig:
    n_layers: int      # L transformer blocks
    hidden: int        # h
    n_heads: int
    seq_len: int       # s
    vocab: int         # V
    micro_batch: int   # mbs (micro-batch *size*)

    @property
    def head_dim(self) -> int:
        return self.hidden // self.n_heads

    @property
    def tokens_per_microbatch(self) -> int:
        return self.micro_batch * self.seq_len

    # ---- parameter layout (oracle layout), SURVEY §8(c) O-2 -------------
    def layer_specs(self, i: int):
        """Tensors of profile layer i in packing order.

        Layer 0 = embedding, 1..L = blocks, L+1 = final LN + LM head
        (SURVEY §8(c) #2).  Each entry: (name, shape, init) with init one of
        'normal', 'normal_proj' (std 0.02/sqrt(2L)), 'zeros', 'ones'.
        """
        h, V, s = self.hidden, self.vocab, self.seq_len
        if i == 0:
            return [("wte", (V, h), "normal"), ("wpe", (s, h), "normal")]
        if i == self.n_layers + 1:
            return [("lnf_g", (h,), "ones"), ("lnf_b", (h,), "zeros"),
                    ("w_head", (h, V), "normal")]
        if 1 <= i <= self.n_layers:
            return [
                ("ln1_g", (h,), "ones"), ("ln1_b", (h,), "zeros"),
                ("w_qkv", (h, 3 * h), "normal"), ("b_qkv", (3 * h,), "zeros"),
                ("w_o", (h, h), "normal_proj"), ("b_o", (h,), "zeros"),
                ("ln2_g", (h,), "ones"), ("ln2_b", (h,), "zeros"),
                ("w_1", (h, 4 * h), "normal"), ("b_1", (4 * h,), "zeros"),
                ("w_2", (4 * h, h), "normal_proj"), ("b_2", (h,), "zeros"),
            ]
        raise IndexError(i)

    @property
    def n_profile_layers(self) -> int:
        return self.n_layers + 2

    def layer_numel(self, i: int) -> int:
        return sum(int(np.prod(sh)) for _, sh, _ in self.layer_specs(i))

    def layer_offsets(self):
        offs = [0]
        for i in range(self.n_profile_layers):
            offs.append(offs[-1] + self.layer_numel(i))
        return offs

    @property
    def n_params(self) -> int:
        return self.layer_offsets()[-1]


# BASELINE.json configs.  vocab 50304 for the GPT
# shapes, 512 for tiny.
TINY = GPTConfig(n_layers=4, hidden=256, n_heads=4, seq_len=128, vocab=512, micro_batch=2)
GPT_1_5B = GPTConfig(n_layers=48, hidden=1600, n_heads=25, seq_len=1024, vocab=50304, micro_batch=8)
GPT_13B = GPTConfig(n_layers=40, hidden=5120, n_heads=40, seq_len=2048, vocab=50304, micro_batch=2)
GPT_70B = GPTConfig(n_layers=80, hidden=8192, n_heads=64, seq_len=2048, vocab=50304, micro_batch=1)
# FD-sized model for the oracle pins (SURVEY §8(c) "What pins each part").
MICRO = GPTConfig(n_layers=2, hidden=16, n_heads=2, seq_len=8, vocab=32, micro_batch=2)

CONFIGS = {"tiny": TINY, "1.5b": GPT_1_5B, "13b": GPT_13B, "70b": GPT_70B, "micro": MICRO}


def gen_params(cfg: GPTConfig, seed: int = SEED_W) -> np.ndarray:
    """Flat fp32 parameter vector in oracle layout, drawn in layout order
    from PCG64(seed)."""
    rng = np.random.Generator(np.random.PCG64(seed))
    out = np.empty(cfg.n_params, dtype=np.float32)
    pos = 0
    proj_std = 0.02 / math.sqrt(2 * cfg.n_layers)
    for i in range(cfg.n_profile_layers):
        for _name, shape, init in cfg.layer_specs(i):
            n = int(np.prod(shape))
            if init == "normal":
                out[pos:pos + n] = rng.standard_normal(n) * 0.02
            elif init == "normal_proj":
                out[pos:pos + n] = rng.standard_normal(n) * proj_std
            elif init == "zeros":
                out[pos:pos + n] = 0.0
            elif init == "ones":
                out[pos:pos + n] = 1.0
            else:  # pragma: no cover
                raise ValueError(init)
            pos += n
    assert pos == cfg.n_params
    return out


def perturb_norm_params(cfg: GPTConfig, params: np.ndarray, seed: int = 99, scale: float = 0.1) -> np.ndarray:
    """Optional: make LN gains/biases and linear biases non-trivial so that
    parity tests exercise every term (with the O-1 init they are exactly
    1 / 0 and a dropped bias term would go unnoticed)."""
    rng = np.random.Generator(np.random.PCG64(seed))
    p = params.copy()
    pos = 0
    for i in range(cfg.n_profile_layers):
        for _name, shape, init in cfg.layer_specs(i):
            n = int(np.prod(shape))
            if init == "ones":
                p[pos:pos + n] = 1.0 + scale * rng.standard_normal(n)
            elif init == "zeros":
                p[pos:pos + n] = scale * rng.standard_normal(n)
            pos += n
    return p.astype(np.float32)


def gen_tokens(cfg: GPTConfig, n_microbatches: int, seed: int = SEED_TOK) -> np.ndarray:
    """Tokens [M][mbs][s+1] int32 ~ U{0..V-1}; inputs [..., :s], targets
    [..., 1:]."""
    rng = np.random.Generator(np.random.PCG64(seed))
    return rng.integers(0, cfg.vocab, size=(n_microbatches, cfg.micro_batch, cfg.seq_len + 1),
                        dtype=np.int64).astype(np.int32)


def round_bf16(x: np.ndarray) -> np.ndarray:
    """fp32 -> bf16 -> fp32 with round-to-nearest-even via uint32 bit ops
    (harness input preparation for the bf16 path; NaN/Inf not expected)."""
    x = np.ascontiguousarray(x, dtype=np.float32)
    u = x.view(np.uint32).astype(np.uint64)
    lsb = (u >> 16) & 1
    u = (u + 0x7FFF + lsb) & 0xFFFF0000
    return u.astype(np.uint32).view(np.float32)


def to_bf16_bits(x: np.ndarray) -> np.ndarray:
    """fp32 -> bf16 bit patterns (uint16), RNE."""
    return (round_bf16(x).view(np.uint32) >> 16).astype(np.uint16)


def from_bf16_bits(b: np.ndarray) -> np.ndarray:
    return (b.astype(np.uint32) << 16).view(np.float32)
