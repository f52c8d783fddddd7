"""Multi-rank plumbing (torch.distributed only carries bytes and scalars; the
data path - activations / activation-gradients between pipeline stages -
runs inside libmobius over CUDA-IPC mappings).

SPMD: every rank (one process per GPU) computes the same plan
(mobius_plan is deterministic), creates its MobiusContext, then
``connect(ctx, group)`` all-gathers the export blobs and maps the
neighbours' receive buffers."""
from __future__ import annotations

from typing import Optional, Sequence

import torch.distributed as dist


def exchange_blobs(blob: bytes, group=None) -> Sequence[bytes]:
    world = dist.get_world_size(group)
    out = [None] * world
    dist.all_gather_object(out, blob, group=group)
    return out


def connect(ctx, group=None) -> None:
    ctx.dist_connect(exchange_blobs(ctx.dist_export(), group))
    dist.barrier(group=group)


def plan_digest(plan) -> tuple:
    K = plan.n_stages
    return (K, tuple(plan.stage_first_layer[j] for j in range(K + 1)), tuple(plan.stage_gpu[j] for j in range(K)),
            plan.makespan_ns)


def check_same_plan(plan, group=None) -> bool:
    """Every rank must hold the same partition/mapping (SPMD contract)."""
    world = dist.get_world_size(group)
    out = [None] * world
    dist.all_gather_object(out, plan_digest(plan), group=group)
    return all(o == out[0] for o in out)


def max_over_ranks(x: float, device: Optional[str] = None, group=None) -> float:
    import torch
    t = torch.tensor([float(x)], dtype=torch.float64, device=device or "cpu")
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return float(t.item())
