"""Model partition (PAPER §3.2) - TEST INFRASTRUCTURE ONLY.

``stage_cost`` is the optimum of the paper's MIP (Eq 3-11, Table 2
P:L662-705) for a FIXED partition, written as the earliest-start recurrence
(the survey checked it equal to an LP solve of the
literal constraints on 269 random instances).  ``brute_force_partition``
enumerates all compositions (O-7).  Everything is exact integer arithmetic
(reading #14): times in int64 ns, bytes in int64, transfer times
ceil(bytes * 1e9 / W).

Readings used: #5 physical K (reload j in backward iff
j + N <= K), #6 separate host (W_h) and P2P (W_p2p) bandwidths - W_p2p is
not charged when N == 1, #7 memory (mem_*) vs transfer (xfer_*) bytes, #8
the prefetch window is stage j-N's execution window, #9 the objective is
the MIP makespan (Eq 3), #13 tie-break key (makespan, K, sizes).
"""
from __future__ import annotations

import dataclasses
import itertools
from typing import Optional, Sequence


@dataclasses.dataclass(frozen=True)
class LayerProfile:
    """One profile layer (Table 2 per-layer quantities)."""
    t_fwd: int      # ns per microbatch  (contributes to T^f)
    t_bwd: int      # ns per microbatch  (T^b)
    mem_fwd: int    # bytes counted against G in forward  (S^f)
    mem_bwd: int    # bytes counted against G in backward (S^b)
    xfer_fwd: int   # bytes uploaded before forward
    xfer_bwd: int   # bytes uploaded before backward (reload)
    act_out: int    # activation (= activation-gradient) bytes at the output


def ceil_xfer_ns(nbytes: int, bw_Bps: Optional[int]) -> int:
    """ceil(bytes * 1e9 / W) in exact integers; W None/0 => free."""
    if not bw_Bps or nbytes <= 0:
        return 0
    return -((-nbytes * 10 ** 9) // bw_Bps)


def stage_sums(layers: Sequence[LayerProfile], sizes: Sequence[int]):
    """Per-stage sums for a composition ``sizes`` (layers per stage)."""
    st = []
    pos = 0
    for n in sizes:
        ls = layers[pos:pos + n]
        st.append(dict(
            Tf=sum(l.t_fwd for l in ls), Tb=sum(l.t_bwd for l in ls),
            Sf=sum(l.mem_fwd for l in ls), Sb=sum(l.mem_bwd for l in ls),
            Xf=sum(l.xfer_fwd for l in ls), Xb=sum(l.xfer_bwd for l in ls),
            A=ls[-1].act_out))
        pos += n
    assert pos == len(layers)
    return st


def feasible(st, G: int) -> bool:
    """Eq 4: S^e_j <= G for every stage and function."""
    return all(s["Sf"] <= G and s["Sb"] <= G for s in st)


def stage_cost(layers, sizes, N: int, M: int, G: int, W_h: int, W_p2p: Optional[int]):
    """Earliest start times of every F_{j,m} / B_{j,m} and the Eq 3
    objective t^b_{1,M} + T^b_1.  Returns (makespan, tf, tb) with
    tf[j][m], tb[j][m] 1-based lists (index 0 unused).  None if infeasible."""
    st = stage_sums(layers, sizes)
    if not feasible(st, G):
        return None
    K = len(st)
    S = [None] + st                      # 1-based
    p2p = (lambda b: 0) if N == 1 else (lambda b: ceil_xfer_ns(b, W_p2p))
    tf = [[0] * (M + 1) for _ in range(K + 1)]
    tb = [[0] * (M + 1) for _ in range(K + 2)]

    def prefetch_bound(X, Sp_mem, B, E):
        # Eq 5/6/9 combined: P <= min(G - S_p, W*D_p, X);  t >= E + (X-P)/W
        return max(E,
                   E + ceil_xfer_ns(max(0, X - (G - Sp_mem)), W_h),
                   B + ceil_xfer_ns(X, W_h))

    # forward, j ascending (Eq 8, 9, 10)
    for j in range(1, K + 1):
        for m in range(1, M + 1):
            c = [0]
            if m > 1:
                c.append(tf[j][m - 1] + S[j]["Tf"])                               # Eq 10
            if j > 1:
                c.append(tf[j - 1][m] + S[j - 1]["Tf"] + p2p(S[j - 1]["A"]))     # Eq 8
            if m == 1 and j > N:
                p = j - N
                c.append(prefetch_bound(S[j]["Xf"], S[p]["Sf"], tf[p][1], tf[p][M] + S[p]["Tf"]))  # Eq 9
            tf[j][m] = max(c)
    # backward, j descending
    for j in range(K, 0, -1):
        for m in range(1, M + 1):
            c = []
            if m > 1:
                c.append(tb[j][m - 1] + S[j]["Tb"])                               # Eq 10
            if j < K:
                c.append(tb[j + 1][m] + S[j + 1]["Tb"] + p2p(S[j]["A"]))         # Eq 8 (bwd)
            if j == K and m == 1:
                c.append(tf[K][M] + S[K]["Tf"])                                   # Eq 11
            if m == 1 and j + N <= K:
                p = j + N
                c.append(prefetch_bound(S[j]["Xb"], S[p]["Sb"], tb[p][1], tb[p][M] + S[p]["Tb"]))  # Eq 9
            tb[j][m] = max(c)
    makespan = tb[1][M] + S[1]["Tb"]                                              # Eq 3
    return makespan, tf, tb


def compositions(n: int):
    """All compositions of n (ordered tuples of positive ints summing to n)."""
    for cuts in range(1 << (n - 1)):
        sizes = []
        run = 1
        for b in range(n - 1):
            if cuts >> b & 1:
                sizes.append(run)
                run = 1
            else:
                run += 1
        sizes.append(run)
        yield tuple(sizes)


def brute_force_partition(layers, N, M, G, W_h, W_p2p):
    """O-7: minimise key (makespan, K, sizes) over all feasible
    compositions.  Returns (makespan, sizes) or None if none is feasible."""
    best = None
    for sizes in compositions(len(layers)):
        r = stage_cost(layers, sizes, N, M, G, W_h, W_p2p)
        if r is None:
            continue
        key = (r[0], len(sizes), sizes)
        if best is None or key < best:
            best = key
    if best is None:
        return None
    return best[0], best[2]


def sequential_stage_gpu(K: int, N: int, perm: Sequence[int] = None):
    """Stage j (1-based) -> GPU perm[(j-1) mod N] (reading #4)."""
    perm = list(range(N)) if perm is None else list(perm)
    return [perm[(j - 1) % N] for j in range(1, K + 1)]


def max_stage_sizes(layers, G):
    """Fig 9 baseline: greedily put as many layers per stage
    as memory allows."""
    sizes, cur, cs_f, cs_b = [], 0, 0, 0
    for l in layers:
        if cur and (cs_f + l.mem_fwd > G or cs_b + l.mem_bwd > G):
            sizes.append(cur)
            cur, cs_f, cs_b = 0, 0, 0
        cur += 1
        cs_f += l.mem_fwd
        cs_b += l.mem_bwd
    sizes.append(cur)
    return tuple(sizes)


def min_stage_sizes(layers):
    """Fig 9 baseline: one layer per stage."""
    return tuple([1] * len(layers))


def uniform_profile(Lp, t_f, t_b, mem, act, xfer=None):
    xfer = mem if xfer is None else xfer
    return [LayerProfile(t_f, t_b, mem, mem, xfer, xfer, act) for _ in range(Lp)]


def all_partitions_of_K(n, K):
    for c in itertools.combinations(range(1, n), K - 1):
        b = (0,) + c + (n,)
        yield tuple(b[i + 1] - b[i] for i in range(K))
