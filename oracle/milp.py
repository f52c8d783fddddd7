"""Literal MIP of PAPER §3.2 (Eq 3-11, Table 2) solved with
scipy.optimize.milp (HiGHS) - TEST INFRASTRUCTURE ONLY.

Used only to pin ``planner.stage_cost`` / ``brute_force_partition`` (O-8).
For a given physical stage count K the variables are

  B[i, j]  in {0,1}   layer i in stage j (i = 1..L', j = 1..K)
  t^f_{j,m}, t^b_{j,m} >= 0  start times
  P^f_j, P^b_j >= 0   prefetched bytes

and the constraints are Eq 4-11 as printed, with stage sums written as
linear functions of B (S^e_j = sum_i B_ij mem_i, T^e_j = sum_i B_ij t_i,
X^e_j = sum_i B_ij xfer_i).  Products of B with times (D_j in Eq 6) are
avoided by using the printed form W * D_{j-N} with D linear in t and T,
which is already linear once T is a linear function of B.  Contiguity:
each layer in exactly one stage, stage of layer i+1 >= stage of layer i,
every stage non-empty (physical K, reading #5).  Transfer terms use the
same ceil(bytes*1e9/W) rounding as the recurrence only when bytes are
constant, so this cross-check is restricted to profiles where every layer
has the same act_out (as for GPT blocks) and W_h divides 1e9*xfer exactly
in the test instances.
"""
from __future__ import annotations

import numpy as np
from scipy.optimize import Bounds, LinearConstraint, milp


def solve_literal_mip(layers, K, N, M, G, W_h, W_p2p):
    """Returns the optimal Eq 3 objective for exactly K non-empty stages, or
    None if infeasible.  Times in ns (continuous)."""
    Lp = len(layers)
    act = layers[0].act_out
    assert all(l.act_out == act for l in layers), "uniform act_out required"
    comm = 0.0 if (N == 1 or not W_p2p) else act * 1e9 / W_p2p
    inv_wh = 1e9 / W_h

    # variable indexing
    nB = Lp * K
    def iB(i, j):   # 0-based
        return i * K + j
    base_tf = nB
    def itf(j, m):
        return base_tf + j * M + m
    base_tb = base_tf + K * M
    def itb(j, m):
        return base_tb + j * M + m
    base_pf = base_tb + K * M
    base_pb = base_pf + K
    nvar = base_pb + K

    rows, lo, hi = [], [], []

    def add(coefs, l, h):
        r = np.zeros(nvar)
        for k, v in coefs:
            r[k] += v
        rows.append(r)
        lo.append(l)
        hi.append(h)

    def T_terms(j, e, scale=1.0):
        return [(iB(i, j), scale * (layers[i].t_fwd if e == "f" else layers[i].t_bwd)) for i in range(Lp)]

    def S_terms(j, e, scale=1.0):
        return [(iB(i, j), scale * (layers[i].mem_fwd if e == "f" else layers[i].mem_bwd)) for i in range(Lp)]

    def X_terms(j, e, scale=1.0):
        return [(iB(i, j), scale * (layers[i].xfer_fwd if e == "f" else layers[i].xfer_bwd)) for i in range(Lp)]

    inf = np.inf
    # each layer in exactly one stage
    for i in range(Lp):
        add([(iB(i, j), 1) for j in range(K)], 1, 1)
    # every stage non-empty
    for j in range(K):
        add([(iB(i, j), 1) for i in range(Lp)], 1, inf)
    # contiguity: stage index non-decreasing in i:  sum_j j*B[i+1,j] - sum_j j*B[i,j] in [0, 1]
    for i in range(Lp - 1):
        add([(iB(i + 1, j), j) for j in range(K)] + [(iB(i, j), -j) for j in range(K)], 0, 1)
    # Eq 4 memory
    for j in range(K):
        for e in "fb":
            add(S_terms(j, e), -inf, G)
    # Eq 5: P^f_j <= G - S^f_{j-N};  P^b_j <= G - S^b_{j+N}
    for j in range(K):
        if j - N >= 0:
            add([(base_pf + j, 1)] + S_terms(j - N, "f"), -inf, G)
        if j + N <= K - 1:
            add([(base_pb + j, 1)] + S_terms(j + N, "b"), -inf, G)
    # Eq 6: P <= W * D_{j-N},  D = T + t_{.,M} - t_{.,1}  (Eq 7);  P <= X_j
    for j in range(K):
        if j - N >= 0:
            p = j - N
            add([(base_pf + j, inv_wh)] + T_terms(p, "f", -1.0) + [(itf(p, M - 1), -1), (itf(p, 0), 1)], -inf, 0)
        if j + N <= K - 1:
            p = j + N
            add([(base_pb + j, inv_wh)] + T_terms(p, "b", -1.0) + [(itb(p, M - 1), -1), (itb(p, 0), 1)], -inf, 0)
        add([(base_pf + j, 1)] + X_terms(j, "f", -1.0), -inf, 0)
        add([(base_pb + j, 1)] + X_terms(j, "b", -1.0), -inf, 0)
    # Eq 8: t^f_{j,m} >= t^f_{j-1,m} + T^f_{j-1} + A/W ;  bwd mirrored
    for j in range(1, K):
        for m in range(M):
            add([(itf(j, m), 1), (itf(j - 1, m), -1)] + T_terms(j - 1, "f", -1.0), comm, inf)
    for j in range(K - 1):
        for m in range(M):
            add([(itb(j, m), 1), (itb(j + 1, m), -1)] + T_terms(j + 1, "b", -1.0), comm, inf)
    # Eq 9: t^f_{j,1} >= t^f_{j-N,M} + T^f_{j-N} + (X_j - P_j)/W
    for j in range(K):
        if j - N >= 0:
            p = j - N
            add([(itf(j, 0), 1), (itf(p, M - 1), -1)] + T_terms(p, "f", -1.0)
                + X_terms(j, "f", -inv_wh) + [(base_pf + j, inv_wh)], 0, inf)
        if j + N <= K - 1:
            p = j + N
            add([(itb(j, 0), 1), (itb(p, M - 1), -1)] + T_terms(p, "b", -1.0)
                + X_terms(j, "b", -inv_wh) + [(base_pb + j, inv_wh)], 0, inf)
    # Eq 10: sequential microbatches
    for j in range(K):
        for m in range(1, M):
            add([(itf(j, m), 1), (itf(j, m - 1), -1)] + T_terms(j, "f", -1.0), 0, inf)
            add([(itb(j, m), 1), (itb(j, m - 1), -1)] + T_terms(j, "b", -1.0), 0, inf)
    # Eq 11: backward after forward of the last stage
    add([(itb(K - 1, 0), 1), (itf(K - 1, M - 1), -1)] + T_terms(K - 1, "f", -1.0), 0, inf)

    c = np.zeros(nvar)
    c[itb(0, M - 1)] = 1.0
    for k, v in T_terms(0, "b"):
        c[k] += v
    integrality = np.zeros(nvar)
    integrality[:nB] = 1
    lb = np.zeros(nvar)
    ub = np.full(nvar, np.inf)
    ub[:nB] = 1
    res = milp(c, constraints=LinearConstraint(np.array(rows), lo, hi), integrality=integrality,
               bounds=Bounds(lb, ub), options={"mip_rel_gap": 0, "presolve": True})
    if res.status != 0:
        return None
    return float(res.fun)
