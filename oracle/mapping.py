"""Cross mapping (PAPER §3.3) - TEST INFRASTRUCTURE ONLY.

contention(Stage_i, Stage_j) = shared(i, j) / |i - j|            (Eq 12)
minimise  sum_{i<j} contention(Stage_i, Stage_j)                  (Eq 13)

shared(i, j) = number of GPUs under the CPU root complex holding both
stages, 0 if the two GPUs sit under different root complexes.
Readings: #4 stage j runs on residue (j-1) mod N and a mapping
is a permutation of residues; #12 same-GPU pairs are excluded (they are
serialised on one GPU); #13 ties broken by the GPU vector lexicographically;
#14 exact rational arithmetic (fractions.Fraction).
"""
from __future__ import annotations

import itertools
from fractions import Fraction
from typing import Sequence


def contention(stage_gpu: Sequence[int], group: Sequence[int]) -> Fraction:
    """Eq 13 objective for a concrete stage -> GPU vector (0-based stages)."""
    size = {}
    for g in group:
        size[g] = size.get(g, 0) + 1
    total = Fraction(0)
    K = len(stage_gpu)
    for i in range(K):
        for j in range(i + 1, K):
            gi, gj = stage_gpu[i], stage_gpu[j]
            if gi != gj and group[gi] == group[gj]:
                total += Fraction(size[group[gi]], j - i)
    return total


def cross_mapping(K: int, N: int, group: Sequence[int]):
    """Brute force over all N! residue permutations (Eq 13).  Returns
    (contention, perm) where stage j (1-based) -> GPU perm[(j-1) mod N]."""
    best = None
    for perm in itertools.permutations(range(N)):
        sg = [perm[(j - 1) % N] for j in range(1, K + 1)]
        c = contention(sg, group)
        key = (c, perm)
        if best is None or key < best:
            best = key
    return best[0], list(best[1])
