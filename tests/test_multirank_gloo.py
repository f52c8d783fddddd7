"""N > 1 host logic on CPU with world_size-2 gloo process groups: every rank
derives the same plan (mobius_plan is deterministic, SPMD contract of
include/mobius.h), the export-blob exchange and the max-over-ranks timing
reduction used by bench.py, and the per-rank op lists of the oracle's
N=2 schedule (Fig 4 rule) cover every (op, stage, microbatch) once."""
import os
import socket

import pytest
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import synth
        from oracle import schedule as osch
        from paper_conf_asplos_fengxtwls23_b200 import (make_topology, mobius_layer_sizes, mobius_plan, model_cfg)
        from paper_conf_asplos_fengxtwls23_b200 import dist as mdist

        c = synth.GPT_1_5B
        prof = mobius_layer_sizes(model_cfg(c.n_layers, c.hidden, c.n_heads, c.seq_len, c.vocab, c.micro_batch))
        for i, p in enumerate(prof):
            p.t_fwd_ns = 900_000 if 0 < i < len(prof) - 1 else 300_000
            p.t_bwd_ns = 2 * p.t_fwd_ns
        plan = mobius_plan(prof, world, 1 << 30, 4 * world, make_topology([0, 1], 55 * 10 ** 9, 700 * 10 ** 9))
        same = mdist.check_same_plan(plan)
        blobs = mdist.exchange_blobs(f"rank{rank}".encode())
        mx = mdist.max_over_ranks(10.0 + rank)
        K = plan.n_stages
        sg = [plan.stage_gpu[j] for j in range(K)]
        mine = osch.per_gpu_ops(sg, 4 * world, n_gpus=world)[rank]
        q.put((rank, same, blobs, mx, len(mine), K, sg))
    finally:
        dist.destroy_process_group()


def test_two_rank_plan_and_plumbing():
    world = 2
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    res.sort()
    for rank, same, blobs, mx, n_ops, K, sg in res:
        assert same
        assert blobs == [b"rank0", b"rank1"]
        assert mx == 11.0
        assert K >= 2 and set(sg) == {0, 1}
        # round robin: stage j on gpu_perm[j mod 2]
        assert all(sg[j] == sg[j % 2] for j in range(K))
    # every (op, stage, mb) exactly once across ranks: 2 * K * M ops
    assert sum(r[4] for r in res) == 2 * res[0][5] * 4 * world
