"""Copy/compute overlap of one Mobius step from its device timeline
(`MobiusContext.read_timeline()`, include/mobius.h mobius_read_timeline).

The paper's claim for the prefetcher (Eq 5/6) is that the
swap-in of stage j+N runs while stage j computes; `overlap_summary` measures
how much of the stage-load (H2D) copy time lies inside compute intervals and
how much of it the compute stream had to wait for.  Pure interval
arithmetic on the event times - no model numerics."""
from __future__ import annotations

from typing import Dict, Iterable, List, Tuple

Interval = Tuple[float, float]


def _union(iv: Iterable[Interval]) -> List[Interval]:
    out: List[Interval] = []
    for a, b in sorted(x for x in iv if x[1] > x[0]):
        if out and a <= out[-1][1]:
            out[-1] = (out[-1][0], max(out[-1][1], b))
        else:
            out.append((a, b))
    return out


def _intersect_len(a: List[Interval], b: List[Interval]) -> float:
    i = j = 0
    tot = 0.0
    while i < len(a) and j < len(b):
        lo, hi = max(a[i][0], b[j][0]), min(a[i][1], b[j][1])
        if hi > lo:
            tot += hi - lo
        if a[i][1] < b[j][1]:
            i += 1
        else:
            j += 1
    return tot


def overlap_summary(timeline) -> Dict[str, float]:
    """timeline: [(kind, stage, t0_ms, t1_ms)] with kind in h2d/fwd/bwd/d2h.
    Returns copy and compute busy times (interval unions, ms), the copy time
    hidden under compute, and the step span."""
    h2d = _union((t0, t1) for k, _, t0, t1 in timeline if k == "h2d")
    d2h = _union((t0, t1) for k, _, t0, t1 in timeline if k == "d2h")
    comp = _union((t0, t1) for k, _, t0, t1 in timeline if k in ("fwd", "bwd"))
    h2d_ms = sum(b - a for a, b in h2d)
    d2h_ms = sum(b - a for a, b in d2h)
    comp_ms = sum(b - a for a, b in comp)
    hid = _intersect_len(h2d, comp)
    hid_d = _intersect_len(d2h, comp)
    t_all = [t for _, _, t0, t1 in timeline for t in (t0, t1)]
    return {"h2d_ms": h2d_ms, "h2d_hidden_ms": hid, "h2d_hidden_frac": hid / h2d_ms if h2d_ms else 1.0,
            "d2h_ms": d2h_ms, "d2h_hidden_ms": hid_d, "compute_busy_ms": comp_ms,
            "span_ms": (max(t_all) - min(t_all)) if t_all else 0.0, "n_h2d_parts": len([x for x in timeline if x[0] == "h2d"])}
