"""Pins for oracle/schedule.py: the Fig 4 per-GPU order as printed, the
bubble makespan closed form, GPipe as the K = N special case, and the
synchronous-update equivalence (pipelined gradients bit-identical to the
unpartitioned step).  CPU only."""
import os

import numpy as np
import pytest

import synth
from oracle import model as om
from oracle import planner as op
from oracle import schedule as osch

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _read_fig4():
    rows = {}
    for line in open(os.path.join(GOLDEN, "fig4_per_gpu_order.txt")):
        line = line.strip()
        if not line or line.startswith("#"):
            continue
        gpu, ops = line.split(":")
        rows[int(gpu.strip()[1:]) - 1] = ops.split()
    return rows


def test_fig4_per_gpu_order():
    K, N, M = 8, 4, 4
    q = osch.per_gpu_ops(op.sequential_stage_gpu(K, N), M)
    fig = _read_fig4()
    for g in range(N):
        expect = []
        for tok in fig[g]:
            expect += [(tok[0], int(tok[1:]), m) for m in range(1, M + 1)]
        assert q[g] == expect


@pytest.mark.parametrize("K,N,M,expect", [(8, 4, 4, 22), (8, 4, 8, 38), (16, 8, 8, 46), (40, 8, 16, 174)])
def test_unit_time_makespan(K, N, M, expect):
    """Unit F = B = 1, free transfers: makespan = 2((K/N) M + N - 1)
    (Fig 4 gives 22)."""
    sg = op.sequential_stage_gpu(K, N)
    ones = {j: 1 for j in range(1, K + 1)}
    mk, _ = osch.simulate_times(sg, M, ones, ones)
    assert mk == expect == 2 * ((K // N) * M + N - 1)
    # the O-6 recurrence (independent formulation) agrees with the event sim
    layers = op.uniform_profile(K, 1, 1, 1, 0)
    r = op.stage_cost(layers, (1,) * K, N, M, G=10 ** 12, W_h=None, W_p2p=None)
    assert r[0] == expect


@pytest.mark.parametrize("K,N,M,tf,tb", [(6, 3, 3, 2, 5), (8, 2, 4, 3, 4), (5, 5, 2, 1, 3), (7, 3, 2, 4, 9)])
def test_recurrence_equals_event_sim(K, N, M, tf, tb):
    """Free transfers, G = inf: O-6 start times == event-simulation start
    times for every (op, j, m), including K not divisible by N."""
    sg = op.sequential_stage_gpu(K, N)
    T_f = {j: tf + (j % 3) for j in range(1, K + 1)}
    T_b = {j: tb + (j % 2) for j in range(1, K + 1)}
    mk, start = osch.simulate_times(sg, M, T_f, T_b)
    layers = [op.LayerProfile(T_f[j], T_b[j], 1, 1, 1, 1, 0) for j in range(1, K + 1)]
    r = op.stage_cost(layers, (1,) * K, N, M, G=10 ** 12, W_h=None, W_p2p=None)
    assert r[0] == mk
    _, tfm, tbm = r
    for j in range(1, K + 1):
        for m in range(1, M + 1):
            assert tfm[j][m] == start[("F", j, m)]
            assert tbm[j][m] == start[("B", j, m)]


def test_gpipe_is_k_equals_n():
    """K = N: every GPU holds one stage; queue is F_{j,.} then B_{j,.}
    (Fig 3)."""
    q = osch.per_gpu_ops(op.sequential_stage_gpu(4, 4), 3)
    for g in range(4):
        assert q[g] == [("F", g + 1, m) for m in (1, 2, 3)] + [("B", g + 1, m) for m in (1, 2, 3)]


def _bounds(sizes):
    b = [0]
    for s in sizes:
        b.append(b[-1] + s)
    return b


@pytest.mark.parametrize("sizes,N,perm", [
    ((6,), 1, None),                 # unpartitioned
    ((3, 3), 1, None),               # tiny config literal "2 stages" at N=1
    ((2, 1, 2, 1), 2, None),         # K=4 at N=2
    ((1, 1, 1, 1, 1, 1), 2, [1, 0]),  # min-stage, permuted mapping
    ((1, 2, 1, 2), 3, [2, 0, 1]),    # K not divisible by N
])
def test_pipelined_grads_bit_identical(sizes, N, perm):
    cfg = synth.GPTConfig(n_layers=4, hidden=32, n_heads=2, seq_len=16, vocab=64, micro_batch=2)
    w = synth.perturb_norm_params(cfg, synth.gen_params(cfg), scale=0.2)
    tok = synth.gen_tokens(cfg, 3)
    l0, g0 = om.reference_loss_and_grads(cfg, w, tok)
    sg = op.sequential_stage_gpu(len(sizes), N, perm)
    l1, g1, trace = osch.execute(cfg, w, tok, _bounds(sizes), sg)
    assert l1 == l0
    assert np.array_equal(g1, g0)
    q = osch.per_gpu_ops(sg, 3)
    for g in range(N):
        assert trace.get(g, []) == q[g]


def test_byte_counts_2K_minus_N_loads():
    """Reading #11: every stage loads once in forward, stage j reloads in
    backward iff j + N <= K -> 2K - N loads; D2H = gradient bytes once."""
    K, N, M = 8, 4, 4
    sg = op.sequential_stage_gpu(K, N)
    st = [dict(Xf=10, Xb=10, A=3)] * K
    h2d, d2h, p2p = osch.byte_counts(st, sg, M, [5] * K)
    assert sum(h2d) == 10 * (2 * K - N)
    assert h2d == [30, 30, 30, 30]
    assert sum(d2h) == 5 * K
    assert sum(p2p) == 2 * M * 3 * (K - 1)
