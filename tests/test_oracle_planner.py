"""Pins for oracle/planner.py, oracle/mapping.py and oracle/adamw.py:
brute force == literal MILP (scipy/HiGHS) on small instances, the uniform
closed form, MIP optimum <= Fig 9's max-/min-stage baselines, Fig 4b cross
mapping, and the AdamW first-step closed form.  CPU only."""
import os
import random
from fractions import Fraction

import numpy as np
import pytest

from oracle import adamw as oa
from oracle import mapping as omap
from oracle import milp as omilp
from oracle import planner as op

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _rand_layers(rng, Lp, same_act=True):
    act = rng.randint(1, 50)
    out = []
    for _ in range(Lp):
        mem = rng.randint(5, 60)
        out.append(op.LayerProfile(rng.randint(1, 30), rng.randint(2, 60), mem, mem + rng.randint(0, 20),
                                   mem, mem, act if same_act else rng.randint(1, 50)))
    return out


@pytest.mark.parametrize("seed", range(12))
def test_brute_force_equals_literal_milp(seed):
    rng = random.Random(seed)
    Lp = rng.randint(2, 6)
    N = rng.randint(1, 3)
    M = rng.randint(1, 4)
    layers = _rand_layers(rng, Lp)
    G = max(max(l.mem_bwd for l in layers), rng.randint(40, 200))
    W = 10 ** 9           # 1 byte per ns: ceil() is exact, MILP comparable
    best = op.brute_force_partition(layers, N, M, G, W, W)
    assert best is not None
    mk, sizes = best
    milp_best = None
    for K in range(1, Lp + 1):
        v = omilp.solve_literal_mip(layers, K, N, M, G, W, W)
        if v is not None and (milp_best is None or v < milp_best):
            milp_best = v
    assert abs(milp_best - mk) < 1e-6, (milp_best, mk, sizes)


@pytest.mark.parametrize("Lp,N,M,tf,tb,expect", [
    (8, 4, 4, 1, 2, 33), (8, 2, 2, 1, 2, 27), (6, 3, 3, 1, 1, 16), (12, 4, 4, 1, 2, 45), (12, 3, 6, 2, 3, 130)])
def test_uniform_free_transfer_optimum(Lp, N, M, tf, tb, expect):
    """G = W = inf, uniform layers, M >= N, N | L': unique optimum K = L'
    with makespan ((L'/N) M + N - 1)(t_f + t_b)."""
    layers = op.uniform_profile(Lp, tf, tb, 1, 0)
    mk, sizes = op.brute_force_partition(layers, N, M, 10 ** 12, None, None)
    assert sizes == (1,) * Lp
    assert mk == expect == ((Lp // N) * M + N - 1) * (tf + tb)


@pytest.mark.parametrize("seed", range(6))
def test_optimum_le_fig9_baselines(seed):
    rng = random.Random(100 + seed)
    Lp = rng.randint(3, 9)
    layers = _rand_layers(rng, Lp)
    N, M = rng.randint(1, 4), rng.randint(1, 4)
    G = max(l.mem_bwd for l in layers) + rng.randint(0, 80)
    W = 10 ** 9
    mk, _ = op.brute_force_partition(layers, N, M, G, W, W)
    for sizes in (op.max_stage_sizes(layers, G), op.min_stage_sizes(layers)):
        r = op.stage_cost(layers, sizes, N, M, G, W, W)
        assert r is not None and mk <= r[0]


def test_infeasible_cap():
    layers = op.uniform_profile(3, 1, 1, 100, 1)
    assert op.brute_force_partition(layers, 1, 1, 99, 10 ** 9, 10 ** 9) is None


def test_partial_prefetch_remainder():
    """Eq 9 with a partial prefetch: two stages of X bytes on one GPU,
    G - S_1 < X_2, slow link: t_{2,1} = E_1 + (X_2 - (G - S_1))/W."""
    l = op.LayerProfile(t_fwd=10, t_bwd=20, mem_fwd=100, mem_bwd=100, xfer_fwd=100, xfer_bwd=100, act_out=1)
    W = 10 ** 9  # 1 B/ns
    mk, tf, tb = op.stage_cost([l, l], (1, 1), N=1, M=2, G=160, W_h=W, W_p2p=None)
    # stage 1: F at 0,10 -> E=20; prefetch of stage 2 starts at B=0,
    # free 60 B hidden, 40 B after release -> t = max(20, 20+40, 0+100) = 100
    assert tf[2][1] == 100
    # backward: stage 2 resident (2 + 1 > 2); stage 1 reloaded: p=2,
    # B = tb[2][1] = 120, E = 120 + 2*20 = 160 -> max(160, 160+40, 120+100) = 220
    assert tb[2][1] == 120 and tb[1][1] == 220 and mk == 220 + 40


def _read_fig4b():
    d = {}
    for line in open(os.path.join(GOLDEN, "fig4b_cross_mapping.txt")):
        if line.startswith("#") or not line.strip():
            continue
        k, v = line.split(":")
        d[k.strip()] = [int(x) for x in v.split()]
    return d


def test_fig4b_cross_mapping():
    d = _read_fig4b()
    c, perm = omap.cross_mapping(d["K"][0], 4, d["groups"])
    assert perm[(5 - 1) % 4] == d["stage5_gpu"][0]
    assert perm[(6 - 1) % 4] == d["stage6_gpu"][0]
    assert perm == [0, 2, 1, 3]
    seq = omap.contention([j % 4 for j in range(8)], d["groups"])
    assert c < seq
    # hand count for the sequential mapping, groups {0,1},{2,3}, K=8:
    # same-group pairs at distance d with residues (0,1) or (2,3):
    # (0,1) pairs: stages (1,2),(1,6),(5,2)->(2,5),(5,6) -> distances 1,5,3,1; same for (2,3)
    hand = 2 * 2 * (Fraction(1, 1) + Fraction(1, 5) + Fraction(1, 3) + Fraction(1, 1))
    assert seq == hand


def test_topo4_all_ties_sequential():
    c, perm = omap.cross_mapping(8, 4, [0, 0, 0, 0])
    assert perm == [0, 1, 2, 3]


def test_mapping_8gpu_4plus4():
    c, perm = omap.cross_mapping(16, 8, [0, 0, 0, 0, 1, 1, 1, 1])
    assert perm == [0, 4, 1, 5, 2, 6, 3, 7]
    assert c < omap.contention([j % 8 for j in range(16)], [0, 0, 0, 0, 1, 1, 1, 1])


def test_adamw_first_step_closed_form():
    rng = np.random.default_rng(0)
    w = (rng.standard_normal(1000) * 1e-2).astype(np.float32)   # small |w|: fp32 ulp << lr
    g = (rng.standard_normal(1000) * 1e-3).astype(np.float32)
    m = np.zeros_like(w)
    v = np.zeros_like(w)
    w1, m1, v1 = oa.adamw_step(w, m, v, g, 1)
    expect = -oa.LR * g.astype(np.float64) / (np.abs(g.astype(np.float64)) + oa.EPS)
    assert np.allclose(w1.astype(np.float64) - w, expect, rtol=1e-3, atol=1e-9)
    # a constant gradient keeps m_hat = g, v_hat = g^2 -> identical steps
    w2, _, _ = oa.adamw_step(w1, m1, v1, g, 2)
    assert np.allclose(w2.astype(np.float64) - w1, expect, rtol=1e-3, atol=1e-9)


# --- max_stage_sizes pins (Fig 9 "max-stage": "as many Transformer blocks as
# possible without running out of memory") -------------------

def _mem_layers(pairs):
    """Profile layers with only (mem_fwd, mem_bwd) set."""
    return [op.LayerProfile(1, 1, mf, mb, mf, mf, 1) for mf, mb in pairs]


@pytest.mark.parametrize("pairs,G,expect", [
    # hand-worked: forward and backward memory equal, greedy fills to G
    ([(4, 4)] * 5, 10, (2, 2, 1)),
    ([(3, 3), (3, 3), (4, 4), (6, 6), (1, 1)], 10, (3, 2)),
    # mem_bwd binds, mem_fwd does not: forward sums are 2+2+2 = 6 <= 10, but
    # backward sums 4+4 = 8, 8+4 = 12 > 10 -> the stage closes after 2 layers
    ([(2, 4), (2, 4), (2, 4), (2, 4), (2, 4)], 10, (2, 2, 1)),
    # mem_fwd binds, mem_bwd does not
    ([(5, 1), (5, 1), (5, 1)], 10, (2, 1)),
    # a stage exactly at the cap is allowed (Eq 4 is <=)
    ([(5, 5), (5, 5), (5, 5), (5, 5)], 10, (2, 2)),
    # every layer alone at the cap -> one layer per stage
    ([(10, 10)] * 3, 10, (1, 1, 1)),
])
def test_max_stage_sizes_hand_worked(pairs, G, expect):
    assert op.max_stage_sizes(_mem_layers(pairs), G) == expect


@pytest.mark.parametrize("seed", range(25))
def test_max_stage_sizes_is_fewest_stages_largest_first(seed):
    """Brute force over all compositions: the max-stage partition is a
    feasible partition with the fewest stages, and among those the one
    whose stages are filled earliest (lexicographically largest sizes) -
    what packing each stage 'as many blocks as possible' in layer order
    means.  Independent of the greedy loop."""
    rng = random.Random(900 + seed)
    Lp = rng.randint(1, 9)
    pairs = [(rng.randint(1, 9), rng.randint(1, 12)) for _ in range(Lp)]
    G = max(max(p) for p in pairs) + rng.randint(0, 20)
    layers = _mem_layers(pairs)
    best = None
    for sizes in op.compositions(Lp):
        pos, ok = 0, True
        for n in sizes:
            ok &= sum(p[0] for p in pairs[pos:pos + n]) <= G and sum(p[1] for p in pairs[pos:pos + n]) <= G
            pos += n
        if ok:
            key = (-len(sizes), sizes)
            if best is None or key > best:
                best = key
    assert op.max_stage_sizes(layers, G) == best[1]


# --- AdamW weight-decay pins (decoupled decay, O-4) ------------------------

def test_adamw_weight_decay_zero_grad_is_pure_decay():
    """g = 0 at step 1: m = v = 0, the Adam term is 0/(0 + eps) = 0, so the
    step is exactly the decoupled decay w <- w - lr*wd*w."""
    rng = np.random.default_rng(3)
    w = rng.standard_normal(512).astype(np.float32)
    z = np.zeros_like(w)
    w1, m1, v1 = oa.adamw_step(w, z, z, z, 1, lr=1e-2, wd=0.1)
    expect = w.astype(np.float64) * (1 - 1e-2 * 0.1)
    assert np.allclose(w1, expect, rtol=1e-6, atol=0)
    assert not m1.any() and not v1.any()


def test_adamw_weight_decay_first_step_closed_form():
    """Step 1 with wd != 0: dw = -lr*wd*w - lr*g/(|g| + eps) (Loshchilov &
    Hutter's decoupled decay; the decay uses the pre-step weight)."""
    rng = np.random.default_rng(4)
    w = rng.standard_normal(1000).astype(np.float32)
    g = (rng.standard_normal(1000) * 1e-3).astype(np.float32)
    z = np.zeros_like(w)
    lr, wd = 1e-3, 0.05
    w1, _, _ = oa.adamw_step(w, z, z, g, 1, lr=lr, wd=wd)
    w64, g64 = w.astype(np.float64), g.astype(np.float64)
    expect = -lr * wd * w64 - lr * g64 / (np.abs(g64) + oa.EPS)
    # fp32 rounding of w (|w| ~ 1) is ~6e-8 absolute; the step is ~1e-3
    assert np.allclose(w1.astype(np.float64) - w64, expect, rtol=1e-3, atol=3e-7)
    # and the decay term is really there: without it the result differs
    w1_nowd, _, _ = oa.adamw_step(w, z, z, g, 1, lr=lr, wd=0.0)
    assert np.abs(w1 - w1_nowd).max() > 10 * 3e-7
