#!/usr/bin/env python
"""Mobius fine-tuning step benchmark (BASELINE.json metric: fine-tune tokens/s
at 1/2/4/8 B200; stage swap-in GB/s vs host-link peak).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config 1.5b] [--impl reference]

N=1 workload = BASELINE configs[1]: GPT 1.5B (48 layers, h=1600, s=1024,
mbs=8) on one B200 with the stage ring capped (default 1 GiB) so every stage
swaps from pinned DRAM each step.  N>1 (torchrun, one rank per GPU): the same
model pipelined over N GPUs with M = M1*N microbatches (weak scaling).

Timing: W untimed warm-up steps; K timed steps between a barrier +
torch.cuda.synchronize() on both sides, CUDA events on the current stream
(mobius_step returns only after its GPU work and the host AdamW update have
completed, so the events bracket complete steps), max over ranks.  Each step
streams every stage's weights (3.1 GB bf16 > 126 MB L2) from host DRAM, so
inputs are larger than L2.  The reference arm (--impl reference) times the
CPU oracle (oracle/, test infrastructure) on a bounded sample; it is a
deliberately slow baseline, not a target.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import synth  # noqa: E402

GiB = 1 << 30
METRIC = "fine-tune tokens/s at 1/2/4/8 B200; stage swap-in GB/s vs host-link peak"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="1.5b")
    ap.add_argument("--layers", type=int, default=0, help="override the block count (shape checks only)")
    ap.add_argument("--microbatches", type=int, default=0, help="M per GPU (default 4 for 1.5b)")
    ap.add_argument("--cap-gib", type=float, default=1.0, help="HBM stage-ring cap G per GPU")
    ap.add_argument("--micro-batch", type=int, default=0,
                    help="micro-batch size mbs (default 32 for 1.5b: 4 x 32 x 1024 = 131072 tokens per GPU-step)")
    ap.add_argument("--impl", default="mobius", choices=["mobius", "reference"])
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-keep", action="store_true", help="always recompute (no kept activations)")
    ap.add_argument("--timeline", default="", help="write the last timed step's device timeline (JSON) here")
    ap.add_argument("--host-tail-update", action="store_true",
                    help="update the last-in-backward stage on the host too (default: GPU AdamW for it)")
    ap.add_argument("--partition", default="mip", choices=["mip", "max", "min"],
                    help="MIP (paper) or the Fig 9 max-stage / min-stage baselines")
    ap.add_argument("--arena-cap-gib", type=float, default=0.0,
                    help="Table 2's G as the WHOLE per-GPU memory (ring + checkpoints + workspaces): "
                         "MOBIUS_FLAG_ARENA_CAP, planner fed G_eff = G - fixed bytes (SURVEY O-11), the paper's "
                         "recompute and host update; survey C2 = --micro-batch 8 --arena-cap-gib 2")
    ap.add_argument("--topology", default="auto", choices=["auto", "probe", "sysfs"],
                    help="host-link contention groups: measured (probe: concurrent pinned H2D < 0.8 x solo, "
                         "SURVEY #12) or sysfs root complex; auto = probe when N > 1")
    ap.add_argument("--mapping", default="cross", choices=["cross", "sequential"],
                    help="stage->GPU mapping: the planner's cross mapping (Eq 12/13) or sequential (f3 baseline)")
    ap.add_argument("--no-prefetch-order", action="store_true",
                    help="N > 1: do not serialise the stage loads of GPUs sharing an uplink by planned stage start "
                         "(P:L858-863 priority)")
    ap.add_argument("--no-offload", action="store_true",
                    help="with --arena-cap-gib: keep every stage-input checkpoint in HBM (no A_Mobius offload)")
    return ap.parse_args()


def dist_env():
    return int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)), int(os.environ.get("LOCAL_RANK", 0))


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return d, "measured"
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0}, "fallback"


class ClockSampler:
    """nvidia-smi clocks / throttle reasons during the timed region."""

    def __init__(self, index=0):
        self.index = index
        self.samples = []
        self._stop = threading.Event()
        self._t = None

    def _run(self):
        q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
             "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
             "clocks_event_reasons.sw_power_cap")
        while not self._stop.is_set():
            try:
                out = subprocess.run(["nvidia-smi", "-i", str(self.index), f"--query-gpu={q}",
                                      "--format=csv,noheader,nounits"], capture_output=True, text=True,
                                     timeout=5).stdout.strip()
                if out:
                    self.samples.append([x.strip() for x in out.split(",")])
            except Exception:
                pass
            self._stop.wait(0.2)

    def start(self):
        self._t = threading.Thread(target=self._run, daemon=True)
        self._t.start()

    def stop(self):
        self._stop.set()
        if self._t:
            self._t.join(timeout=10)
        sm = [float(s[0]) for s in self.samples if s[0].replace(".", "").isdigit()]
        mx = [float(s[1]) for s in self.samples if s[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for s in self.samples for i in range(4) if len(s) > 3 + i and "Active" in s[3 + i]
                          and not s[3 + i].startswith("Not")})
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.samples)}


def model_flops_per_token(c: synth.GPTConfig) -> float:
    """Algorithmic FLOPs per token, fwd + bwd, causal attention, LM head
    (SURVEY §8(d)): L (72 h^2 + 6 s h) + 6 h V.  Recompute excluded."""
    h = c.hidden
    return c.n_layers * (72 * h * h + 6 * c.seq_len * h) + 6 * h * c.vocab


# --------------------------------------------------------------- reference
def host_cpu_info():
    """CPU model and the BLAS numpy links (printed with the oracle timing)."""
    model = "unknown"
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    model = line.split(":", 1)[1].strip()
                    break
    except OSError:
        pass
    blas = "unknown"
    try:
        import io
        import contextlib
        buf = io.StringIO()
        with contextlib.redirect_stdout(buf):
            np.show_config()
        txt = buf.getvalue().lower()
        for name in ("openblas", "mkl", "blis", "accelerate"):
            if name in txt:
                blas = name
                break
    except Exception:
        pass
    return model, blas


def cpu_oracle_sample(c: synth.GPTConfig, tokens_per_step: int, budget_s: float = 20.0):
    """Time the oracle (numpy fp32) on one block fwd+bwd and the head at
    mbs=1, extrapolate to tokens/s:  T_step ~ (L t_block + t_head + t_embed)
    * tokens_per_step / s."""
    from oracle import model as om
    cores = len(os.sched_getaffinity(0))
    s, h, V = c.seq_len, c.hidden, c.vocab
    c1 = synth.GPTConfig(n_layers=c.n_layers, hidden=h, n_heads=c.n_heads, seq_len=s, vocab=V, micro_batch=1)
    rng = np.random.default_rng(0)
    blk = {name: (rng.standard_normal(shape) * 0.02).astype(np.float32) if init.startswith("normal")
           else (np.ones(shape, np.float32) if init == "ones" else np.zeros(shape, np.float32))
           for name, shape, init in c1.layer_specs(1)}
    head = {name: (rng.standard_normal(shape) * 0.02).astype(np.float32) if init.startswith("normal")
            else (np.ones(shape, np.float32) if init == "ones" else np.zeros(shape, np.float32))
            for name, shape, init in c1.layer_specs(c1.n_layers + 1)}
    x = rng.standard_normal((s, h)).astype(np.float32)
    tok = rng.integers(0, V, size=(1, s + 1))
    tb, th = [], []
    t_start = time.perf_counter()
    while True:  # bounded sample: repeat until ~budget_s of CPU work, take medians
        t0 = time.perf_counter()
        y, cache = om.block_fwd(c1, blk, x, 1)
        om.block_bwd(c1, blk, y, cache, 1)
        tb.append(time.perf_counter() - t0)
        t0 = time.perf_counter()
        om.head_fwd_bwd(c1, head, x, tok[:, 1:], s)
        th.append(time.perf_counter() - t0)
        if time.perf_counter() - t_start > budget_s or len(tb) >= 50:
            break
    t_block, t_head = float(np.median(tb)), float(np.median(th))
    t_step = (c.n_layers * t_block + t_head) * tokens_per_step / s
    cpu_model, blas = host_cpu_info()
    return {"value": tokens_per_step / t_step, "unit": "tokens/s", "cores": cores, "kind": "oracle",
            "cpu_model": cpu_model, "blas": blas,
            "sample": f"numpy fp32 oracle: {len(tb)} x (1 block fwd+bwd, median {t_block:.2f}s + LM head fwd+bwd, "
                      f"median {t_head:.2f}s) at mbs=1 s={s} h={h} V={V} (~{budget_s:.0f}s of CPU work), "
                      f"extrapolated x{c.n_layers} blocks to the step's {tokens_per_step} tokens "
                      f"(host AdamW and transfers not included)"}


def bench_workload(args, world):
    """(config, M): the bench's GPT config (mbs overridable) and microbatch
    count.  1.5b default: M = 4 per GPU of mbs 32 (131072 tokens per GPU per
    step).  Same tokens, measured on one box back to back: 16 x mbs 8 79.5k,
    8 x mbs 16 86.0k, 4 x mbs 32 87.6k tokens/s - larger GEMMs quantise
    better over the 74 SM pairs and the elementwise kernels amortise."""
    import dataclasses
    c = synth.CONFIGS[args.config]
    mbs = args.micro_batch or (32 if args.config == "1.5b" else c.micro_batch)
    c = dataclasses.replace(c, n_layers=args.layers or c.n_layers, micro_batch=mbs)
    M = (args.microbatches or (4 if args.config == "1.5b" else 16)) * world
    return c, M


def run_reference(args, rank, world):
    if rank != 0:
        return
    c, M = bench_workload(args, args.gpus)
    tps = M * c.micro_batch * c.seq_len
    vals = []
    for _ in range(args.warmup):
        cpu_oracle_sample(c, tps, budget_s=3.0)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        vals.append(cpu_oracle_sample(c, tps, budget_s=10.0))
    wall = time.perf_counter() - t0
    v = float(np.median([x["value"] for x in vals]))
    cb = dict(vals[-1])
    cb["value"] = v
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "tokens/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1000.0 * tps / v,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": f"GPT {args.config} CPU oracle sample", "model": f"gpt-{args.config}",
                       "global_batch": M * c.micro_batch, "seq_len": c.seq_len, "microbatches": M},
            "cpu_baseline": cb,
            "e2e": {"value": v, "unit": "tokens/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
            "wall_s": wall}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ mobius
def measure_h2d_GBps(torch, nbytes=512 << 20):
    h = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
    d = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    d.copy_(h, non_blocking=True)
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(3):
        d.copy_(h, non_blocking=True)
    b.record()
    torch.cuda.synchronize()
    return 3 * nbytes / (a.elapsed_time(b) * 1e-3) / 1e9


def run_mobius(args, rank, world, local):
    import torch
    import torch.distributed as dist
    from paper_conf_asplos_fengxtwls23_b200 import (BF16, FLAG_DEVICE_TAIL_UPDATE, FLAG_KEEP_ACTS, FLAG_TIMING,
                                                    MobiusContext, make_topology, mobius_discover_topology,
                                                    mobius_plan, mobius_profile, model_cfg)
    # MOBIUS_BENCH_SAME_GPU=1: every rank on device 0 (checks the N>1 code
    # path on a 1-GPU box; ranks time-slice the GPU, numbers are not scaling
    # numbers).  Plumbing then uses gloo (NCCL rejects duplicate GPUs).
    same_gpu = os.environ.get("MOBIUS_BENCH_SAME_GPU") == "1"
    if same_gpu:
        local = 0
    torch.cuda.set_device(local)
    if world > 1:
        if same_gpu:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    pg_dev = "cpu" if same_gpu else "cuda"
    c, M = bench_workload(args, world)
    cfg = model_cfg(c.n_layers, c.hidden, c.n_heads, c.seq_len, c.vocab, c.micro_batch, dtype=BF16)
    G = int(args.cap_gib * GiB)
    arena = args.arena_cap_gib > 0
    arena_flags = 0
    if arena:
        from paper_conf_asplos_fengxtwls23_b200 import (FLAG_ARENA_CAP, FLAG_CKPT_OFFLOAD, mobius_arena_fixed_bytes,
                                                        mobius_arena_layer_sizes)
        arena_flags = FLAG_ARENA_CAP | (0 if (args.no_offload or world > 1) else FLAG_CKPT_OFFLOAD)
        # G_eff = G - everything outside the ring (upper bound on the local
        # stage count for the per-stage slot / flag arrays)
        fixed = mobius_arena_fixed_bytes(cfg, M, c.n_layers + 2, arena_flags)
        G = int(args.arena_cap_gib * GiB) - fixed
        if G <= 0:
            sys.exit(f"bench.py: --arena-cap-gib {args.arena_cap_gib}: the fixed workspaces alone need "
                     f"{fixed / GiB:.2f} GiB")
    # profile (layer similarity) and plan (MIP + cross mapping)
    t_prof0 = time.perf_counter()
    prof = mobius_profile(cfg, local)
    prof_s = time.perf_counter() - t_prof0
    if arena:  # whole-memory mem_fwd / mem_bwd, measured times (SURVEY O-11)
        mem = mobius_arena_layer_sizes(cfg)
        for p, q in zip(prof, mem):
            p.mem_fwd, p.mem_bwd, p.xfer_fwd, p.xfer_bwd = q.mem_fwd, q.mem_bwd, q.xfer_fwd, q.xfer_bwd
    h2d_gbps = measure_h2d_GBps(torch)
    topo_src = args.topology if args.topology != "auto" else ("probe" if world > 1 else "sysfs")
    probe = None
    if topo_src == "probe" and rank == 0:
        from paper_conf_asplos_fengxtwls23_b200 import mobius_probe_topology
        topo, solo, pair = mobius_probe_topology(256 << 20, 0.8)
        probe = {"solo_GBps": solo, "pair_GBps": pair, "p2p_GBps": topo.p2p_bw_Bps / 1e9}
    else:
        topo = mobius_discover_topology()
    groups = [topo.group[i] for i in range(topo.n_gpus)][:world]
    if len(groups) < world:
        groups = list(range(world))
    # SPMD contract: every rank must plan from identical inputs -> rank 0's
    # profile, link bandwidth and topology are broadcast (measured timings
    # differ slightly per GPU, which would yield different partitions)
    shared = [[(p.t_fwd_ns, p.t_bwd_ns, p.mem_fwd, p.mem_bwd, p.xfer_fwd, p.xfer_bwd, p.act_out) for p in prof],
              h2d_gbps, groups, probe]
    if world > 1:
        dist.broadcast_object_list(shared, src=0)
        from paper_conf_asplos_fengxtwls23_b200._lib import LayerProfile
        prof = [LayerProfile(*x) for x in shared[0]]
        h2d_gbps, groups, probe = shared[1], shared[2], shared[3]
    t = make_topology(groups, host_bw_Bps=int(h2d_gbps * 1e9), p2p_bw_Bps=int(700e9))
    t0 = time.perf_counter()
    if args.partition == "mip":
        plan = mobius_plan(prof, world, G, M, t)
    else:
        from paper_conf_asplos_fengxtwls23_b200 import (PARTITION_MAX_STAGE, PARTITION_MIN_STAGE,
                                                        mobius_plan_partition)
        plan = mobius_plan_partition(prof, world, G, M,
                                     PARTITION_MAX_STAGE if args.partition == "max" else PARTITION_MIN_STAGE, t)
    plan_s = time.perf_counter() - t0
    if args.mapping == "sequential":  # f3 baseline: stage j on GPU (j-1) mod N
        for g in range(world):
            plan.gpu_perm[g] = g
        for j in range(plan.n_stages):
            plan.stage_gpu[j] = j % world
    from paper_conf_asplos_fengxtwls23_b200 import mobius_mapping_contention
    contention = mobius_mapping_contention(plan.n_stages, groups, [plan.gpu_perm[g] for g in range(world)])[0]
    if world > 1:
        from paper_conf_asplos_fengxtwls23_b200 import dist as mdist
        assert mdist.check_same_plan(plan), "ranks derived different plans"
    timing = os.environ.get("MOBIUS_BENCH_TIMING", "1") != "0"  # per-kernel CUDA events (roofline)
    flags = (FLAG_TIMING if timing else 0) | (0 if args.no_keep else FLAG_KEEP_ACTS) | \
        (0 if args.host_tail_update else FLAG_DEVICE_TAIL_UPDATE)
    if arena:  # the paper's regime: everything inside G, recompute, host update
        flags = (FLAG_TIMING if timing else 0) | arena_flags
    ctx = MobiusContext(cfg, plan, rank=rank, world=world, device=local, seed=1234, flags=flags)
    prefetch_order = world > 1 and not args.no_prefetch_order and len(set(groups)) < world
    if prefetch_order:  # loads of GPUs sharing an uplink: one at a time, earlier-starting stage first
        ctx.set_prefetch_groups(groups)
    if world > 1:
        blobs = [None] * world
        dist.all_gather_object(blobs, ctx.dist_export())
        ctx.dist_connect(blobs)
        dist.barrier()
    tokens = synth.gen_tokens(c, M)
    tok_dev = torch.from_numpy(tokens).cuda()

    def barrier():
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
            torch.cuda.synchronize()

    def max_over_ranks(x):
        if world == 1:
            return x
        tt = torch.tensor([x], dtype=torch.float64, device=pg_dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        return float(tt.item())

    dbg = os.environ.get("MOBIUS_DEBUG") == "1"
    if dbg:
        print(f"[rank {rank}] ctx ready, K={plan.n_stages}", file=sys.stderr, flush=True)
    loss = float("nan")
    for w in range(args.warmup):
        loss = ctx.step_device(tok_dev, M)
        if dbg:
            print(f"[rank {rank}] warmup step {w} loss {loss}", file=sys.stderr, flush=True)
    sampler = ClockSampler(local)
    sampler.start()
    barrier()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ev0.record()
    stats = []
    for _ in range(args.steps):
        loss = ctx.step_device(tok_dev, M)
        stats.append(ctx.stats())
    ev1.record()
    barrier()
    clocks = sampler.stop()
    # device timeline of the last timed step: copy/compute overlap evidence
    from paper_conf_asplos_fengxtwls23_b200.timeline import overlap_summary
    timeline = ctx.read_timeline()
    overlap = overlap_summary(timeline)
    if args.timeline and rank == 0:
        with open(args.timeline, "w") as f:
            json.dump({"kinds": "h2d = stage-load copy part, fwd/bwd = a stage's pass over its M microbatches, "
                                "d2h = gradient offload / tail-stage weight write-back; ms from the step start",
                       "records": [{"kind": k, "stage": j, "t0_ms": a, "t1_ms": b} for k, j, a, b in timeline],
                       "summary": overlap}, f, indent=1)
    ms = max_over_ranks(ev0.elapsed_time(ev1) / args.steps)
    tokens_per_step = M * c.micro_batch * c.seq_len
    value = tokens_per_step / (ms * 1e-3)

    # e2e: same step through the public API with HOST tokens (H2D inside the
    # timed region) and the loss read back (D2H)
    e2e = None
    if not args.no_e2e:
        barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(args.steps):
            ctx.step(tokens)
        e1.record()
        barrier()
        ems = max_over_ranks(e0.elapsed_time(e1) / args.steps)
        e2e = {"value": tokens_per_step / (ems * 1e-3), "unit": "tokens/s", "h2d_bytes_per_step": int(tokens.nbytes),
               "d2h_bytes_per_step": 8, "ms_per_step": ems}

    st = stats[-1]

    def avg(field):
        return sum(getattr(x, field) for x in stats) / len(stats)
    peaks, peak_src = load_peaks()
    gemm_ns = sum(s.gemm_ns for s in stats)
    gemm_flops = sum(s.gemm_flops for s in stats)
    achieved_tf = gemm_flops / (gemm_ns * 1e-9) / 1e12 if gemm_ns else 0.0
    peak_tf = peaks.get("bf16_tflops_sustained", peaks.get("bf16_tflops"))
    traffic = traffic_alg = None
    # ncu --set full capture of the block GEMM shapes (per launch) at this T
    tr_name = {32768: "r2_gemm_traffic_v7.json", 16384: "r1_gemm_traffic_v5.json",
               8192: "r1_gemm_traffic_v3.json"}.get(c.micro_batch * c.seq_len)
    tr_path = os.path.join(ROOT, "profiles", tr_name) if tr_name else ""
    tr_n = 0
    if tr_path and os.path.exists(tr_path):
        with open(tr_path) as f:
            tr = json.load(f)
        traffic = float(np.mean([t["dram_bytes"] for t in tr]))
        traffic_alg = float(np.mean([t["algorithmic_bytes"] for t in tr]))
        tr_n = len(tr)
    # model GEMM FLOPs per step (no recompute): L (72 h^2) per token fwd+bwd + the LM head 6 h V
    model_gemm_flop_step = (c.n_layers * 72 * c.hidden ** 2 + 6 * c.hidden * c.vocab) * tokens_per_step / world
    # step roofline (north_star): max(FLOP / P_tc, H2D bytes / host link), per GPU
    flop_step = model_flops_per_token(c) * tokens_per_step / world
    t_tc = flop_step / (peak_tf * 1e12)
    t_link = max(st.h2d_bytes + st.ckpt_h2d_bytes, st.d2h_bytes + st.ckpt_d2h_bytes) / (h2d_gbps * 1e9)
    t_roof = max(t_tc, t_link)
    line = None
    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "tokens/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "bf16", "data": "synthetic (seeded GPT-shaped tokens, random-init weights)",
            "config": {"workload": f"GPT {args.config} (configs[1]): L={c.n_layers} h={c.hidden} heads={c.n_heads} "
                                   f"s={c.seq_len} V={c.vocab}, " +
                                   (f"whole HBM arena capped at {args.arena_cap_gib} GiB per GPU (Table 2 G: ring + "
                                    f"checkpoints + workspaces{', checkpoint offload' if arena_flags & 16 else ''})"
                                    if arena else f"stage ring capped at {args.cap_gib} GiB per GPU"),
                       "model": f"gpt-{args.config}", "global_batch": M * c.micro_batch, "seq_len": c.seq_len,
                       "microbatches": M, "micro_batch": c.micro_batch, "parallelism": f"mobius-pp{world}",
                       "n_stages": plan.n_stages, "stage_layers": [plan.stage_first_layer[j + 1] - plan.stage_first_layer[j]
                                                                   for j in range(plan.n_stages)],
                       "gpu_perm": [plan.gpu_perm[g] for g in range(world)], "plan_s": plan_s,
                       "mapping": args.mapping, "uplink_groups": groups, "topology_source": topo_src,
                       "mapping_contention": contention, "prefetch_order": prefetch_order, "link_probe": probe,
                       "profile_s": prof_s, "plan_exhaustive": bool(plan.exhaustive),
                       "partition": args.partition, "plan_makespan_ms": plan.makespan_ns / 1e6,
                       "arena_cap_GB": args.arena_cap_gib * GiB / 1e9 if arena else None,
                       "tail_stage_update": "host AdamW" if (args.host_tail_update or arena) else
                       "GPU AdamW (first stage, last in backward; optimizer state in HBM)",
                       "l2": "inputs larger than L2: every stage (3.1 GB bf16 total) streams from host DRAM each step"},
            "loss": loss,
            "e2e": e2e,
            "roofline": {"bound": "tensor", "kernel": "gemm_tc (tcgen05 bf16, all block/head GEMMs)",
                         "achieved": achieved_tf, "peak": peak_tf, "unit": "TFLOP/s",
                         "frac": achieved_tf / peak_tf if peak_tf else None, "traffic": traffic,
                         "traffic_algorithmic_bytes": traffic_alg,
                         "traffic_source": f"profiles/{tr_name}: dram__bytes_read+write per launch, mean over the "
                                           f"{tr_n} captured 1.5B block GEMM shapes at T={c.micro_batch * c.seq_len} "
                                           "(ncu --set full, cold L2; tools/gemm_prof.py + tools/gemm_traffic.py)",
                         "peak_source": f"MEASURED_PEAKS.json bf16_tflops_sustained ({peak_src})",
                         "flops_counted": "2MNK of every sampled GEMM launch, including the launches of the "
                                          "recomputed blocks (launches of the same kernel)",
                         "frac_model_flops": (model_gemm_flop_step / (avg("gemm_ns") * 1e-9) / 1e12 / peak_tf
                                              if avg("gemm_ns") and peak_tf else None)},
            "step_roofline": {"t_tensor_ms": t_tc * 1e3, "t_link_ms": t_link * 1e3, "t_roofline_ms": t_roof * 1e3,
                              "frac": t_roof / (ms * 1e-3), "h2d_GBps_link": h2d_gbps,
                              "note": "north_star step roofline = max(algorithmic FLOPs / tensor peak, stage bytes / "
                                      "measured pinned H2D); recompute, bubble and host update excluded"},
            "swap_in": {"h2d_bytes_per_step": st.h2d_bytes, "d2h_bytes_per_step": st.d2h_bytes,
                        "copies": st.n_h2d_copies, "GBps_median": st.h2d_GBps_median, "GBps_max": st.h2d_GBps_max,
                        "link_peak_GBps": h2d_gbps, "exposed_load_ms": st.exposed_load_ns / 1e6},
            "overlap": dict(overlap, source="mobius_read_timeline (CUDA events on the prefetch, compute and D2H "
                                            "streams, last timed step; nsys is not in this image)"),
            "breakdown_ms": {"gemm": avg("gemm_ns") / 1e6, "attention": avg("attn_ns") / 1e6,
                             "elementwise": avg("elem_ns") / 1e6,
                             "timing": f"CUDA events around every {st.timing_stride}th launch of each kernel class "
                                       "inside the timed steps, scaled by the stride (sampled estimate)",
                             "device_step": st.device_step_ns / 1e6, "host_update_total": st.host_update_ns / 1e6,
                             "update_tail": st.update_tail_ns / 1e6},
            "memory": {"arena_GB": st.arena_bytes / 1e9, "ring_GB": st.ring_bytes / 1e9,
                       "pinned_host_GB": st.pinned_bytes / 1e9, "recompute_blocks": int(st.recompute),
                       "kept_layout": "none (recompute)" if (arena or args.no_keep) else
                       "compact (x, qkv, o, x1, u, lse, LN stats)",
                       "ckpt_offload_GB_per_step": (st.ckpt_d2h_bytes + st.ckpt_h2d_bytes) / 1e9,
                       "exposed_ckpt_ms": st.exposed_ckpt_ns / 1e6},
            "gpu_launches": int(sum(s.kernel_launches for s in stats)),
            "clocks": clocks,
        }
    ctx.close()
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_oracle_sample(c, tokens_per_step)
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


def spawn_ranks(n):
    """`--gpus N` without a launcher: re-exec this command under
    torch.distributed.run with one rank per GPU (127.0.0.1 rendezvous), or
    fail loudly if the box has fewer than N GPUs - never silently benchmark
    one rank and label it N."""
    import socket
    same_gpu = os.environ.get("MOBIUS_BENCH_SAME_GPU") == "1"
    if not same_gpu:
        import torch
        have = torch.cuda.device_count()
        if have < n:
            sys.exit(f"bench.py: --gpus {n} needs {n} GPUs, this box has {have} "
                     f"(set MOBIUS_BENCH_SAME_GPU=1 to run {n} ranks on one GPU as a code-path check)")
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__)] + sys.argv[1:]
    print(f"bench.py: launching {n} ranks: {' '.join(cmd)}", file=sys.stderr, flush=True)
    sys.exit(subprocess.call(cmd))


def main():
    args = parse()
    rank, world, local = dist_env()
    if world != args.gpus and world > 1:
        sys.exit(f"bench.py: WORLD_SIZE={world} != --gpus {args.gpus}")
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ and args.impl != "reference":
        spawn_ranks(args.gpus)
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    run_mobius(args, rank, world, local)


if __name__ == "__main__":
    main()
