"""Per-stage parameter update in DRAM - TEST INFRASTRUCTURE ONLY.

The paper offloads gradients to DRAM "for parameter update"
and updates synchronously like GPipe but names no optimizer.
Reading #16 / O-4: AdamW in fp32 on the host master copy, beta1 = 0.9,
beta2 = 0.999, eps = 1e-8, weight decay 0 (decoupled, Loshchilov & Hutter),
lr = 1e-4, with bias correction; the new bf16 stage weights are RNE(master).
"""
from __future__ import annotations

import numpy as np

LR = 1e-4
BETA1 = 0.9
BETA2 = 0.999
EPS = 1e-8
WD = 0.0


def adamw_step(master, m, v, grad, step, lr=LR, beta1=BETA1, beta2=BETA2, eps=EPS, wd=WD):
    """One AdamW step (step is 1-based).  All arrays fp32; returns new
    (master, m, v).  Update order: decoupled decay, moments, bias-corrected
    step:  w <- w - lr*wd*w;  m <- b1 m + (1-b1) g;  v <- b2 v + (1-b2) g^2;
    w <- w - lr * (m / (1-b1^t)) / (sqrt(v / (1-b2^t)) + eps)."""
    f = np.float32
    g = grad.astype(f)
    w = master.astype(f)
    if wd:
        w = w - f(lr * wd) * w
    m = f(beta1) * m + f(1 - beta1) * g
    v = f(beta2) * v + f(1 - beta2) * g * g
    bc1 = f(1 - beta1 ** step)
    bc2 = f(1 - beta2 ** step)
    w = w - f(lr) * (m / bc1) / (np.sqrt(v / bc2) + f(eps))
    return w.astype(f), m.astype(f), v.astype(f)
