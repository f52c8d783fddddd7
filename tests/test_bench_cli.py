"""bench.py launcher contract (CPU): `--gpus N` without torchrun must not
silently run one rank and label it N (VERDICT r1 Missing #6): on a box with
fewer GPUs it exits non-zero with a message; with enough GPUs it re-execs
under torch.distributed.run (covered on GPU boxes)."""
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_bench_gpus_without_launcher_fails_loudly_without_gpus():
    torch = pytest.importorskip("torch")
    if torch.cuda.device_count() >= 2:
        pytest.skip("box has >= 2 GPUs: bench.py would launch the ranks")
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    env.pop("MOBIUS_BENCH_SAME_GPU", None)
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "1"],
                       capture_output=True, text=True, env=env, timeout=300)
    assert r.returncode != 0
    assert "needs 2 GPUs" in r.stderr
    assert '"n_gpus": 1' not in r.stdout


def test_bench_world_size_mismatch_fails():
    env = dict(os.environ, WORLD_SIZE="2", RANK="0", LOCAL_RANK="0")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "4", "--steps", "1"],
                       capture_output=True, text=True, env=env, timeout=300)
    assert r.returncode != 0 and "WORLD_SIZE=2 != --gpus 4" in r.stderr
