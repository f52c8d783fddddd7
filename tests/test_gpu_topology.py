"""Measured host-link contention groups on
the visible GPUs: solo pinned H2D at the link's rate, a group per GPU that
does not slow another's copies, and the groups feeding the planner's cross
mapping."""
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a GPU", allow_module_level=True)

from paper_conf_asplos_fengxtwls23_b200 import mobius_probe_topology, mobius_topology_from_bw  # noqa: E402


def test_probe_topology_measures_links():
    t, solo, pair = mobius_probe_topology(128 << 20, 0.8)
    n = torch.cuda.device_count()
    assert t.n_gpus == min(n, 16)
    assert all(20.0 < x < 200.0 for x in solo), solo  # PCIe 5 x16 pinned H2D
    assert t.host_bw_Bps == int(sorted(solo)[len(solo) // 2] * 1e9)
    # the grouping is the pure function of the measured numbers
    t2 = mobius_topology_from_bw(solo, pair, 0.8)
    assert [t.group[i] for i in range(t.n_gpus)] == [t2.group[i] for i in range(t.n_gpus)]
    if n == 1:
        assert t.group[0] == 0 and t.p2p_bw_Bps == 0
    else:
        assert t.p2p_bw_Bps > 100e9  # NVLink peer copy
