"""Mobius pipeline schedule (PAPER §3.1, Fig 4) -
TEST INFRASTRUCTURE ONLY.

* S (= K) stages can outnumber the N GPUs; stage j runs on GPU
  stage_gpu[j-1] (round-robin residues, reading #4).
* Each GPU runs, for its stages in ascending order, F_{j,1..M}; then for its
  stages in descending order, B_{j,1..M} (Fig 4: F_{1,.} F_{5,.} ... B_{5,.}
  B_{1,.}; the last stage on a GPU runs backward without a reload).
* F_{j,m} needs the activation of F_{j-1,m}; B_{j,m} needs the
  activation-gradient of B_{j+1,m} (Eq 8); B_{K,.} starts after
  F_{K,M} (Eq 11).
* Stage-input checkpoints: F stores x_{j,m}; B recomputes the stage forward
  from it (reading #17); dW of a stage accumulates
  over m ascending (Fig 4, reading #22).

``execute`` runs the real numerics through the per-GPU queues in a
discrete-event order and records the trace; gradients must be bit-identical
to ``model.reference_loss_and_grads`` (synchronous update).
``simulate_times`` is an independent event simulation of the same queues
with given per-stage durations (used to pin the Fig 4 makespan).
"""
from __future__ import annotations

import numpy as np

from . import model as om


def per_gpu_ops(stage_gpu, M, n_gpus=None):
    """Per-GPU op lists [(op, j, m)], j and m 1-based (row a1)."""
    K = len(stage_gpu)
    N = max(stage_gpu) + 1 if n_gpus is None else n_gpus
    q = {g: [] for g in range(N)}
    for g in range(N):
        mine = [j for j in range(1, K + 1) if stage_gpu[j - 1] == g]
        for j in mine:
            q[g] += [("F", j, m) for m in range(1, M + 1)]
        for j in reversed(mine):
            q[g] += [("B", j, m) for m in range(1, M + 1)]
    return q


def _ready(op, done, K):
    kind, j, m = op
    if kind == "F":
        return j == 1 or ("F", j - 1, m) in done
    if j == K:
        return ("F", K, m) in done
    return ("B", j + 1, m) in done


def global_order(stage_gpu, M):
    """Discrete-event order: repeatedly pop any ready queue head (lowest GPU
    first).  Raises on deadlock."""
    K = len(stage_gpu)
    q = per_gpu_ops(stage_gpu, M)
    heads = {g: 0 for g in q}
    done = set()
    order = []
    total = sum(len(v) for v in q.values())
    while len(order) < total:
        progressed = False
        for g in sorted(q):
            if heads[g] < len(q[g]) and _ready(q[g][heads[g]], done, K):
                op = q[g][heads[g]]
                heads[g] += 1
                done.add(op)
                order.append((g,) + op)
                progressed = True
                break
        if not progressed:
            raise RuntimeError("schedule deadlock")
    return order


def simulate_times(stage_gpu, M, Tf, Tb, xfer_p2p=0):
    """Event simulation with per-stage durations Tf[j], Tb[j] (1-based dict
    or list) and free weight transfers.  Returns (makespan, start) with
    start[(op, j, m)]."""
    K = len(stage_gpu)
    order = global_order(stage_gpu, M)
    gpu_free = {}
    end = {}
    start = {}
    N = max(stage_gpu) + 1
    hop = xfer_p2p if N > 1 else 0
    for g, kind, j, m in order:
        t = gpu_free.get(g, 0)
        if kind == "F":
            if j > 1:
                t = max(t, end[("F", j - 1, m)] + hop)
            d = Tf[j]
        else:
            if j == K:
                t = max(t, end[("F", K, M)])
            else:
                t = max(t, end[("B", j + 1, m)] + hop)
            d = Tb[j]
        start[(kind, j, m)] = t
        end[(kind, j, m)] = t + d
        gpu_free[g] = t + d
    return max(end.values()), start


def stage_layers(boundaries, j):
    """Profile layers of stage j (1-based) given boundaries[K+1]."""
    return list(range(boundaries[j - 1], boundaries[j]))


def execute(cfg, flat_params, tokens, boundaries, stage_gpu, dtype=np.float32):
    """Run one Mobius step's numerics through the per-GPU queues.

    boundaries: stage_first_layer list of length K+1 over profile layers.
    Returns (loss, flat_grads, trace) with trace[g] = [(op, j, m), ...]."""
    flat = np.asarray(flat_params, dtype=dtype)
    K = len(stage_gpu)
    M, mbs, _ = tokens.shape
    Lp = cfg.n_profile_layers
    n_tok = M * mbs * cfg.seq_len
    P = [om.unpack_layer(cfg, flat, i) for i in range(Lp)]
    G = [None] * Lp
    ckpt = {}          # (j, m) -> stage input activation (a5)
    act = {}           # (j, m) -> stage output activation, "sent" to j+1 (a3)
    grad_in = {}       # (j, m) -> dL/d(stage j output), "sent" from j+1 (a8)
    head_dx = {}       # m -> dx at the head input (head fwd+bwd runs in F_K)
    head_g = {}
    loss_sum = 0.0
    trace = {}

    def acc(i, gi):
        if G[i] is None:
            G[i] = {k: v.copy() for k, v in gi.items()}
        else:
            for k in G[i]:
                G[i][k] = G[i][k] + gi[k]

    def stage_forward(j, m, x, keep):
        caches = {}
        tok = tokens[m - 1, :, :-1]
        for i in stage_layers(boundaries, j):
            if i == 0:
                x, caches[0] = om.embed_fwd(cfg, P[0], tok)
            elif i <= cfg.n_layers:
                x, caches[i] = om.block_fwd(cfg, P[i], x, mbs)
            else:
                x_head = x
                caches[i] = x_head
        return x, caches

    for g, kind, j, m in global_order(stage_gpu, M):
        trace.setdefault(g, []).append((kind, j, m))
        layers = stage_layers(boundaries, j)
        if kind == "F":
            x_in = None if j == 1 else act[(j - 1, m)]
            ckpt[(j, m)] = x_in
            x, caches = stage_forward(j, m, x_in, keep=False)
            if layers[-1] == Lp - 1:          # head: loss + dx (K9 fwd+bwd)
                ls, dx, gh = om.head_fwd_bwd(cfg, P[Lp - 1], x, tokens[m - 1, :, 1:], n_tok)
                loss_sum += ls
                head_dx[m] = dx
                head_g[m] = gh
            act[(j, m)] = x
        else:
            # recompute the stage forward from its checkpoint (a7)
            x, caches = stage_forward(j, m, ckpt[(j, m)], keep=True)
            if layers[-1] == Lp - 1:
                dx = head_dx.pop(m)
                acc(Lp - 1, head_g.pop(m))
            else:
                dx = grad_in.pop((j, m))
            for i in reversed(layers):
                if i == Lp - 1:
                    continue
                if i == 0:
                    acc(0, om.embed_bwd(cfg, P[0], dx, caches[0]))
                else:
                    dx, gi = om.block_bwd(cfg, P[i], dx, caches[i], mbs)
                    acc(i, gi)
            if j > 1:
                grad_in[(j - 1, m)] = dx
    return loss_sum / n_tok, om.pack_layers(cfg, G, dtype=dtype), trace


def byte_counts(stage_sums_list, stage_gpu, M, grad_bytes, n_gpus=None):
    """O-10 byte accounting per GPU.  stage_sums_list[j-1] has Xf, Xb, A;
    grad_bytes[j-1] = offloaded gradient bytes of stage j.  Loads: every
    stage once in forward, stage j again in backward iff j + N <= K
    (reading #11 -> 2K - N loads per step)."""
    K = len(stage_gpu)
    N = max(stage_gpu) + 1 if n_gpus is None else n_gpus
    h2d = [0] * N
    d2h = [0] * N
    p2p = [0] * N
    for j in range(1, K + 1):
        g = stage_gpu[j - 1]
        h2d[g] += stage_sums_list[j - 1]["Xf"]
        if j + N <= K:
            h2d[g] += stage_sums_list[j - 1]["Xb"]
        d2h[g] += grad_bytes[j - 1]
        if N > 1 and j < K:
            # activation to j+1 (fwd) sent by g; activation-grad back (bwd)
            # sent by stage_gpu[j]
            p2p[g] += M * stage_sums_list[j - 1]["A"]
            p2p[stage_gpu[j]] += M * stage_sums_list[j - 1]["A"]
    return h2d, d2h, p2p
