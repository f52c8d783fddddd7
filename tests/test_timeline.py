"""Host-side overlap arithmetic of the step timeline (CPU; the timeline
itself is checked on the GPU in test_gpu_step.py)."""
import random

from paper_conf_asplos_fengxtwls23_b200.timeline import overlap_summary


def brute(timeline, kinds_a, kinds_b, step=0.01):
    def cov(kinds, t):
        return any(k in kinds and t0 <= t < t1 for k, _, t0, t1 in timeline)
    lo = min(t0 for _, _, t0, _ in timeline)
    hi = max(t1 for _, _, _, t1 in timeline)
    n = int(round((hi - lo) / step))
    a = sum(cov(kinds_a, lo + (i + 0.5) * step) for i in range(n)) * step
    ab = sum(cov(kinds_a, lo + (i + 0.5) * step) and cov(kinds_b, lo + (i + 0.5) * step) for i in range(n)) * step
    return a, ab


def test_overlap_hand_example():
    # load 0 exposed (0-2), stage 1 computes 2-6 while load 2 runs 3-5 (hidden), load 3 runs 5-7 (half hidden)
    tl = [("h2d", 1, 0.0, 2.0), ("fwd", 1, 2.0, 6.0), ("h2d", 2, 3.0, 5.0), ("h2d", 3, 5.0, 7.0),
          ("bwd", 1, 7.0, 8.0), ("d2h", 1, 8.0, 9.0)]
    s = overlap_summary(tl)
    assert abs(s["h2d_ms"] - 6.0) < 1e-12
    assert abs(s["h2d_hidden_ms"] - 3.0) < 1e-12
    assert abs(s["compute_busy_ms"] - 5.0) < 1e-12
    assert abs(s["d2h_hidden_ms"]) < 1e-12
    assert abs(s["span_ms"] - 9.0) < 1e-12 and s["n_h2d_parts"] == 3


def test_overlap_random_vs_brute_force():
    rnd = random.Random(3)
    for _ in range(20):
        tl = []
        for k in ("h2d", "fwd", "bwd", "d2h"):
            for j in range(rnd.randint(1, 4)):
                a = round(rnd.uniform(0, 5), 2)
                tl.append((k, j + 1, a, round(a + rnd.uniform(0.05, 2), 2)))
        s = overlap_summary(tl)
        a, ab = brute(tl, {"h2d"}, {"fwd", "bwd"})
        assert abs(s["h2d_ms"] - a) < 0.05 and abs(s["h2d_hidden_ms"] - ab) < 0.05
