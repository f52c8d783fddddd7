"""Stage swap-in sweep (BASELINE configs[4]; Fig 7 / Fig 10 analog, SURVEY
§8(d) C5 / §8(f) f3): host->HBM copy bandwidth of a stage-sized pinned
buffer, 1 MiB .. 4 GiB, measured

  solo        - the copy alone (the host-link peak the roofline uses),
  with_d2h    - while the gradient offload (D2H) of another stage runs,
  with_gemm   - while the compute stream runs bf16 GEMMs (swap-in hidden
                behind compute),

and, when launched with torchrun over N GPUs, every rank swapping at once,
with the per-rank and aggregate bandwidth (host-link contention when GPUs
share an uplink); the summary line gives the discovered contention groups
and the cross mapping mobius_cross_map derives from them.
Copies use the same DMA path as the
runtime's prefetcher (pinned cudaMemcpyAsync on a high-priority stream).
This is a link-characterisation tool, not the bench contract.

usage: python tools/swap_sweep.py [--max-gib 4] [--out profiles/swap_sweep.jsonl]
       torchrun --nproc-per-node N tools/swap_sweep.py ...
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

MiB = 1 << 20


def timed_copy(dst, src, stream, iters):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(stream):
        dst.copy_(src, non_blocking=True)
        a.record(stream)
        for _ in range(iters):
            dst.copy_(src, non_blocking=True)
        b.record(stream)
    b.synchronize()
    return iters * src.numel() / (a.elapsed_time(b) * 1e-3) / 1e9


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--max-gib", type=float, default=4.0)
    ap.add_argument("--out", default="")
    args = ap.parse_args()
    rank = int(os.environ.get("RANK", 0))
    world = int(os.environ.get("WORLD_SIZE", 1))
    local = int(os.environ.get("LOCAL_RANK", 0))
    torch.cuda.set_device(local)
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    from paper_conf_asplos_fengxtwls23_b200 import (mobius_cross_map, mobius_mapping_contention,
                                                    mobius_probe_topology)
    probe = None
    if rank == 0:  # measured contention groups (SURVEY #12): concurrent pinned H2D < 0.8 x solo
        topo, solo, pair = mobius_probe_topology(256 << 20, 0.8)
        probe = {"solo_GBps": solo, "pair_GBps": pair, "p2p_GBps": topo.p2p_bw_Bps / 1e9,
                 "groups": [topo.group[i] for i in range(topo.n_gpus)]}
    if world > 1:
        obj = [probe]
        dist.broadcast_object_list(obj, src=0)
        probe = obj[0]
    groups = probe["groups"][:max(world, 1)]
    hi = torch.cuda.Stream(priority=-1)
    lo = torch.cuda.Stream(priority=0)
    comp = torch.cuda.Stream(priority=0)
    sizes = []
    s = MiB
    while s <= args.max_gib * (1 << 30):
        sizes.append(s)
        s *= 4
    gemm_a = torch.randn(8192, 8192, device="cuda", dtype=torch.bfloat16)
    lines = []
    for nbytes in sizes:
        host = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
        dev = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
        iters = max(2, min(50, (2 << 30) // nbytes))
        if world > 1:
            dist.barrier()
        solo = timed_copy(dev, host, hi, iters)
        # concurrent D2H offload of an equal-sized gradient
        dev2 = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
        host2 = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
        with torch.cuda.stream(lo):
            for _ in range(iters + 2):
                host2.copy_(dev2, non_blocking=True)
        with_d2h = timed_copy(dev, host, hi, iters)
        torch.cuda.synchronize()
        # concurrent compute
        with torch.cuda.stream(comp):
            for _ in range(max(4, iters // 2)):
                gemm_a @ gemm_a
        with_gemm = timed_copy(dev, host, hi, iters)
        torch.cuda.synchronize()
        rec = {"rank": rank, "world": world, "stage_MiB": nbytes / MiB, "h2d_GBps_solo": solo,
               "h2d_GBps_with_d2h": with_d2h, "h2d_GBps_with_gemm": with_gemm}
        if world > 1:
            t = torch.tensor([solo, with_d2h, with_gemm], device="cuda", dtype=torch.float64)
            dist.all_reduce(t)
            rec.update({"aggregate_GBps_solo": t[0].item(), "aggregate_GBps_with_d2h": t[1].item(),
                        "aggregate_GBps_with_gemm": t[2].item()})
        lines.append(rec)
        if rank == 0:
            print(json.dumps(rec), flush=True)
        del host, dev, dev2, host2
    if rank == 0:
        perm, cont, num, den = mobius_cross_map(2 * max(world, 1), groups)
        seq = mobius_mapping_contention(2 * max(world, 1), groups, list(range(len(groups))))[0]
        summary = {"summary": True, "groups": groups, "probe": probe, "cross_map": list(perm),
                   "cross_contention": cont, "sequential_contention": seq,
                   "note": "N=1: no host-link contention between GPUs; cross vs sequential differs only for N>1 "
                           "(end-to-end comparison: bench.py --mapping cross|sequential --topology probe)"}
        print(json.dumps(summary))
        if args.out:
            with open(args.out, "w") as f:
                for r in lines + [summary]:
                    f.write(json.dumps(r) + "\n")
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
