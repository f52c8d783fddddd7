"""CPU tests of the C-ABI library (no GPU compute): it loads, exports every
symbol include/*.h declares, and its host-side planner / mapper are
bit-exact against the oracle (SURVEY §8(c) pins: O-6/O-7 partition, O-9
mapping, Fig 4b, byte accounting O-10)."""
import os
import random
import re
from fractions import Fraction

import numpy as np
import pytest

import synth
from oracle import mapping as omap
from oracle import planner as op
from oracle import schedule as osch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def mb():
    import paper_conf_asplos_fengxtwls23_b200 as m
    return m


def declared_symbols():
    names = set()
    for h in ("mobius.h", "mobius_kernels.h"):
        src = open(os.path.join(ROOT, "include", h)).read()
        src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
        for m in re.finditer(r"^\s*(?:const\s+)?[a-z_0-9]+\s*\*?\s*(mobius_[a-z_0-9]+)\s*\(", src, flags=re.M):
            names.add(m.group(1))
    return names


def test_library_exports_every_declared_symbol(mb):
    from paper_conf_asplos_fengxtwls23_b200 import _lib
    decl = declared_symbols()
    assert len(decl) >= 25
    missing = [n for n in decl if not hasattr(_lib.lib, n)]
    assert not missing, missing
    assert set(decl) == set(_lib.SIGNATURES), set(decl) ^ set(_lib.SIGNATURES)
    assert not _lib.MISSING
    assert "sm_100a" in mb.build_info()


def test_library_is_sm100a_cubin():
    import subprocess
    lib = os.path.join(ROOT, "paper_conf_asplos_fengxtwls23_b200", "libmobius.so")
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", lib], capture_output=True, text=True).stdout
    assert "sm_100a" in out
    sass = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-sass", lib], capture_output=True, text=True).stdout
    assert "UTCHMMA" in sass and "UTMALDG" in sass and "LDTM" in sass  # tcgen05.mma, TMA, tcgen05.ld


def _rand_layers(rng, Lp):
    act = rng.randint(1, 50)
    out = []
    for _ in range(Lp):
        mem = rng.randint(5, 60)
        out.append(op.LayerProfile(rng.randint(1, 3000), rng.randint(2, 6000), mem, mem + rng.randint(0, 20),
                                   mem, mem + rng.randint(0, 5), act))
    return out


@pytest.mark.parametrize("seed", range(30))
def test_plan_cost_bit_exact(mb, seed):
    rng = random.Random(seed)
    Lp = rng.randint(1, 9)
    layers = _rand_layers(rng, Lp)
    N, M = rng.randint(1, 4), rng.randint(1, 5)
    G = max(l.mem_bwd for l in layers) + rng.randint(0, 100)
    Wh, Wp = rng.choice([None, 7 * 10 ** 8, 3 * 10 ** 9 + 7]), rng.choice([None, 10 ** 9, 13 * 10 ** 8 + 1])
    for sizes in list(op.compositions(Lp))[:64]:
        r = op.stage_cost(layers, sizes, N, M, G, Wh, Wp)
        if r is None:
            with pytest.raises(mb.MobiusError):
                mb.mobius_plan_cost(layers, sizes, N, G, M, Wh, Wp)
            continue
        mk, tf, tb = mb.mobius_plan_cost(layers, sizes, N, G, M, Wh, Wp, want_times=True)
        assert mk == r[0]
        K = len(sizes)
        assert tf.tolist() == [r[1][j][1:] for j in range(1, K + 1)]
        assert tb.tolist() == [r[2][j][1:] for j in range(1, K + 1)]


@pytest.mark.parametrize("seed", range(20))
def test_plan_partition_matches_brute_force(mb, seed):
    rng = random.Random(1000 + seed)
    Lp = rng.randint(2, 10)
    layers = _rand_layers(rng, Lp)
    N, M = rng.randint(1, 4), rng.randint(1, 4)
    G = max(l.mem_bwd for l in layers) + rng.randint(0, 150)
    W = rng.choice([10 ** 9, 5 * 10 ** 8])
    best = op.brute_force_partition(layers, N, M, G, W, W)
    plan = mb.mobius_plan(layers, N, G, M, mb.make_topology(list(range(N)), W, W))
    K = plan.n_stages
    sizes = tuple(plan.stage_first_layer[j + 1] - plan.stage_first_layer[j] for j in range(K))
    assert plan.exhaustive == 1
    assert (plan.makespan_ns, sizes) == best
    # byte accounting (O-10) per GPU
    sg = [plan.stage_gpu[j] for j in range(K)]
    ss = op.stage_sums(layers, sizes)
    h2d, d2h, p2p = osch.byte_counts(ss, sg, M, [s["Xf"] for s in ss], n_gpus=N)
    assert [plan.h2d_bytes[g] for g in range(N)] == h2d
    assert [plan.d2h_bytes[g] for g in range(N)] == d2h
    assert [plan.p2p_bytes[g] for g in range(N)] == p2p


def test_plan_infeasible(mb):
    layers = op.uniform_profile(4, 1, 1, 100, 1)
    with pytest.raises(mb.MobiusError) as e:
        mb.mobius_plan(layers, 1, 99, 2, mb.make_topology([0]))
    assert e.value.code == -2


@pytest.mark.parametrize("K,groups", [(8, [0, 0, 1, 1]), (8, [0, 0, 0, 0]), (8, [0, 1, 1, 1]), (16, [0] * 4 + [1] * 4),
                                      (16, [0, 0, 1, 1, 2, 2, 3, 3]), (5, [0, 1, 0]), (12, [0, 0, 1, 1, 0]),
                                      (3, [0, 0])])
def test_cross_map_matches_oracle(mb, K, groups):
    c_ref, perm_ref = omap.cross_mapping(K, len(groups), groups)
    perm, c, num, den = mb.mobius_cross_map(K, groups)
    assert perm == perm_ref
    assert abs(c - float(c_ref)) < 1e-12 * max(1.0, float(c_ref))
    if den:
        assert Fraction(num, den) == c_ref
    # sequential mapping value
    cs, n2, d2 = mb.mobius_mapping_contention(K, groups, list(range(len(groups))))
    ref_s = omap.contention([j % len(groups) for j in range(K)], groups)
    assert abs(cs - float(ref_s)) < 1e-12 * max(1.0, float(ref_s))


def test_fig4b_through_the_abi(mb):
    perm, c, _, _ = mb.mobius_cross_map(8, [0, 0, 1, 1])
    assert perm == [0, 2, 1, 3]    # stage5 -> P1, stage6 -> P3


def test_large_K_contention_exact_order(mb):
    # K = 82 (70B-class profile) stays exact: compare two permutations whose
    # contentions are mathematically equal by symmetry
    g = [0, 0, 1, 1]
    a, _, _ = mb.mobius_mapping_contention(82, g, [0, 2, 1, 3])
    b, _, _ = mb.mobius_mapping_contention(82, g, [2, 0, 3, 1])
    assert a == b


def test_layer_sizes_match_synth(mb):
    for name in ("tiny", "1.5b", "13b", "70b"):
        c = synth.CONFIGS[name]
        for dt, e in ((mb.BF16, 2), (mb.F32, 4)):
            prof = mb.mobius_layer_sizes(mb.model_cfg(c.n_layers, c.hidden, c.n_heads, c.seq_len, c.vocab,
                                                      c.micro_batch, dtype=dt))
            assert len(prof) == c.n_profile_layers
            for i, p in enumerate(prof):
                assert p.mem_fwd == p.xfer_fwd == c.layer_numel(i) * e
                assert p.act_out == c.micro_batch * c.seq_len * c.hidden * e


def test_tiny_config_cap_forces_swap(mb):
    """configs[0]: 4 MiB cap (reading #19) -> 2 stages cannot be co-resident,
    the planner must split and the second stage is partially prefetched."""
    c = synth.TINY
    prof = mb.mobius_layer_sizes(mb.model_cfg(c.n_layers, c.hidden, c.n_heads, c.seq_len, c.vocab, c.micro_batch))
    for p in prof:
        p.t_fwd_ns, p.t_bwd_ns = 100000, 200000
    plan = mb.mobius_plan(prof, 1, 4 << 20, 2, mb.make_topology([0], 50 * 10 ** 9, 0))
    assert plan.n_stages >= 2
    tot = sum(p.mem_fwd for p in prof)
    assert tot > 4 << 20


@pytest.mark.parametrize("seed", range(10))
def test_fig9_baseline_partitions(mb, seed):
    """max-stage / min-stage (Fig 9) through the ABI equal the
    oracle's construction, are scored by the same Eq 3-11 objective, and the
    MIP optimum is never worse."""
    rng = random.Random(500 + seed)
    Lp = rng.randint(2, 12)
    layers = _rand_layers(rng, Lp)
    N, M = rng.randint(1, 4), rng.randint(1, 4)
    G = max(l.mem_bwd for l in layers) + rng.randint(0, 120)
    W = 10 ** 9
    topo = mb.make_topology(list(range(N)), W, W)
    mip = mb.mobius_plan(layers, N, G, M, topo)
    for algo, ref in ((mb.PARTITION_MAX_STAGE, op.max_stage_sizes(layers, G)),
                      (mb.PARTITION_MIN_STAGE, op.min_stage_sizes(layers))):
        pl = mb.mobius_plan_partition(layers, N, G, M, algo, topo)
        sizes = tuple(pl.stage_first_layer[j + 1] - pl.stage_first_layer[j] for j in range(pl.n_stages))
        assert sizes == ref
        r = op.stage_cost(layers, ref, N, M, G, W, W)
        assert pl.makespan_ns == r[0]
        assert mip.makespan_ns <= pl.makespan_ns


def test_package_fails_loudly_without_library(tmp_path):
    """No CPU or Python fallback: a copy of the package without
    libmobius.so must refuse to import (the product path is the CUDA
    library or nothing)."""
    import shutil
    import subprocess
    import sys
    pkg = os.path.join(ROOT, "paper_conf_asplos_fengxtwls23_b200")
    dst = tmp_path / "paper_conf_asplos_fengxtwls23_b200"
    shutil.copytree(pkg, dst, ignore=shutil.ignore_patterns("*.so", "csrc", "__pycache__"))
    r = subprocess.run([sys.executable, "-c", "import paper_conf_asplos_fengxtwls23_b200"], cwd=tmp_path,
                       capture_output=True, text=True, timeout=300,
                       env={**os.environ, "PYTHONPATH": str(tmp_path)})
    assert r.returncode != 0
    assert "libmobius.so not built" in r.stderr


def _key(pl):
    K = pl.n_stages
    return (pl.makespan_ns, K, tuple(pl.stage_first_layer[j + 1] - pl.stage_first_layer[j] for j in range(K)))


@pytest.mark.parametrize("seed", range(6))
def test_plan_above_20_layers_vs_brute_force(mb, seed, monkeypatch):
    """L' = 21-22 (beyond the enumeration limit): the local search + branch
    and bound against a brute force over all 2^(L'-1) compositions (the same
    C++ recurrence, forced with MOBIUS_PLAN_EXHAUSTIVE_MAX).  A certified
    result (exhaustive = 1) must be the optimum key exactly; an uncertified
    one must be no worse than the brute force's by the key order."""
    rng = random.Random(2100 + seed)
    Lp = 21 + seed % 2
    layers = _rand_layers(rng, Lp)
    N, M = 1 + seed % 3, rng.randint(1, 4)
    G = max(l.mem_bwd for l in layers) + rng.randint(0, 120)
    topo = mb.make_topology(list(range(N)), 10 ** 9, 10 ** 9)
    monkeypatch.delenv("MOBIUS_PLAN_EXHAUSTIVE_MAX", raising=False)
    fast = mb.mobius_plan(layers, N, G, M, topo)
    monkeypatch.setenv("MOBIUS_PLAN_EXHAUSTIVE_MAX", str(Lp))
    brute = mb.mobius_plan(layers, N, G, M, topo)
    assert brute.exhaustive == 1
    if fast.exhaustive:
        assert _key(fast) == _key(brute)
    else:
        assert fast.makespan_ns >= brute.makespan_ns


def test_plan_1p5b_profile_certified_at_n1(mb):
    """The bench's planning problem (GPT-1.5B, L' = 50, N = 1, M = 4, 1 GiB
    ring, measured-shape layer times) is solved to proven optimality by the
    branch and bound (exhaustive = 1) in well under a second."""
    import time
    c = synth.GPT_1_5B
    prof = mb.mobius_layer_sizes(mb.model_cfg(c.n_layers, c.hidden, c.n_heads, c.seq_len, c.vocab, 32))
    for i, p in enumerate(prof):
        f = 6_600_000
        p.t_fwd_ns, p.t_bwd_ns = (200_000, 400_000) if i == 0 else (3 * f, 6 * f) if i == len(prof) - 1 else \
            (f, int(2.3 * f))
    t0 = time.time()
    pl = mb.mobius_plan(prof, 1, 1 << 30, 4, mb.make_topology([0], 55 * 10 ** 9, 0))
    assert pl.exhaustive == 1
    assert time.time() - t0 < 5.0
    assert mb._lib.lib.mobius_plan_search_nodes() > 0
    # the certificate's partition is no worse than Fig 9's max-stage baseline
    mx = mb.mobius_plan_partition(prof, 1, 1 << 30, 4, mb.PARTITION_MAX_STAGE, mb.make_topology([0], 55 * 10 ** 9, 0))
    assert pl.makespan_ns <= mx.makespan_ns


def _pair_from(solo, groups, share=0.5, noise=0.0):
    """Synthetic concurrent bandwidths: GPUs of one uplink group halve each
    other's bandwidth, others do not interfere."""
    n = len(solo)
    return [[(solo[i] * (share if groups[i] == groups[j] else 1.0 - noise)) if i != j else 0.0 for j in range(n)]
            for i in range(n)]


@pytest.mark.parametrize("groups", [[0, 0, 1, 1], [0, 1, 1, 1], [0, 0, 0, 0], [0, 1, 2, 3],
                                    [0, 0, 0, 0, 1, 1, 1, 1], [0, 1, 0, 1, 2, 2, 3, 3]])
def test_topology_from_measured_bandwidth(mb, groups):
    """GPUs whose concurrent pinned H2D falls below 0.8 x
    solo share an uplink group (Topo 2+2, 1+3, 4, and 8-GPU layouts); group
    ids are numbered by first member; host W = median solo."""
    n = len(groups)
    solo = [55.0 + i for i in range(n)]
    t = mb.mobius_topology_from_bw(solo, _pair_from(solo, groups, noise=0.05), 0.8)
    got = [t.group[i] for i in range(n)]
    canon, ids = [], {}
    for g in groups:
        ids.setdefault(g, len(ids))
        canon.append(ids[g])
    assert got == canon
    assert t.host_bw_Bps == int(sorted(solo)[n // 2] * 1e9)
    # the measured groups feed the cross mapping: adjacent stages avoid sharing
    if 1 < len(set(groups)) < n and n <= 8:
        perm, c, _, _ = mb.mobius_cross_map(2 * n, got)
        seq, _, _ = mb.mobius_mapping_contention(2 * n, got, list(range(n)))
        assert c <= seq


def test_topology_from_bw_threshold_edge(mb):
    """Exactly at the threshold the pair is not contended (strict <);
    contention is judged on the worse of the two directions."""
    solo = [50.0, 50.0]
    t = mb.mobius_topology_from_bw(solo, [[0, 40.0], [40.0, 0]], 0.8)
    assert [t.group[0], t.group[1]] == [0, 1]
    t = mb.mobius_topology_from_bw(solo, [[0, 50.0], [39.0, 0]], 0.8)
    assert [t.group[0], t.group[1]] == [0, 0]
