"""Python binding of include/mobius.h: same names, argument marshalling
only (numpy arrays / torch device tensors -> pointers).  Nothing here
computes any part of the method."""
from __future__ import annotations

import ctypes as C
from typing import Optional, Sequence

import numpy as np

from . import _lib as L
from ._lib import (BF16, F32, FLAG_ARENA_CAP, FLAG_CKPT_OFFLOAD, FLAG_DEVICE_TAIL_UPDATE, FLAG_KEEP_ACTS,  # noqa: F401
                   FLAG_TIMING, MobiusError, check, lib)

__all__ = ["mobius_plan", "mobius_plan_partition", "PARTITION_MIP", "PARTITION_MAX_STAGE", "PARTITION_MIN_STAGE", "mobius_plan_cost", "mobius_cross_map", "mobius_mapping_contention",
           "mobius_discover_topology", "mobius_topology_from_bw", "mobius_probe_topology", "mobius_layer_sizes", "mobius_profile", "MobiusContext", "model_cfg",
           "make_topology", "plan_from_sizes", "kt", "BF16", "F32", "FLAG_TIMING", "FLAG_KEEP_ACTS", "FLAG_DEVICE_TAIL_UPDATE", "FLAG_ARENA_CAP", "FLAG_CKPT_OFFLOAD",
           "mobius_arena_layer_sizes", "mobius_arena_fixed_bytes", "MobiusError",
           "build_info"]


def build_info() -> str:
    return lib.mobius_build_info().decode()


def model_cfg(n_layers, hidden, n_heads, seq_len, vocab, micro_batch, dtype=BF16, lr=1e-4, beta1=0.9, beta2=0.999,
              eps=1e-8, weight_decay=0.0) -> L.ModelCfg:
    return L.ModelCfg(n_layers, hidden, n_heads, seq_len, vocab, micro_batch, dtype, lr, beta1, beta2, eps,
                      weight_decay)


def _profile_array(layers) -> "C.Array":
    arr = (L.LayerProfile * len(layers))()
    for i, l in enumerate(layers):
        if isinstance(l, L.LayerProfile):
            arr[i] = l
        else:  # any object with the oracle LayerProfile attribute names
            arr[i] = L.LayerProfile(l.t_fwd, l.t_bwd, l.mem_fwd, l.mem_bwd, l.xfer_fwd, l.xfer_bwd, l.act_out)
    return arr


def make_topology(groups: Sequence[int], host_bw_Bps: int = 0, p2p_bw_Bps: int = 0) -> L.Topology:
    t = L.Topology()
    t.n_gpus = len(groups)
    for i, g in enumerate(groups):
        t.group[i] = g
    t.host_bw_Bps = host_bw_Bps
    t.p2p_bw_Bps = p2p_bw_Bps
    return t


def mobius_discover_topology() -> L.Topology:
    t = L.Topology()
    check(lib.mobius_discover_topology(C.byref(t)))
    return t


def mobius_topology_from_bw(solo: Sequence[float], pair, threshold: float = 0.8) -> L.Topology:
    """pair: n x n array-like of GB/s (row i: GPU i while column j copies)."""
    n = len(solo)
    so = (C.c_double * n)(*solo)
    pa = (C.c_double * (n * n))(*[float(pair[i][j]) for i in range(n) for j in range(n)])
    t = L.Topology()
    check(lib.mobius_topology_from_bw(n, so, pa, threshold, C.byref(t)))
    return t


def mobius_probe_topology(nbytes: int = 256 << 20, threshold: float = 0.8):
    """(topology, solo GB/s list, pair GB/s n x n list) measured on the visible GPUs."""
    so = (C.c_double * L.MAX_GPUS)()
    pa = (C.c_double * (L.MAX_GPUS * L.MAX_GPUS))()
    t = L.Topology()
    check(lib.mobius_probe_topology(nbytes, threshold, C.byref(t), so, pa))
    n = t.n_gpus
    return t, list(so[:n]), [[pa[i * n + j] for j in range(n)] for i in range(n)]


def mobius_plan(layers, n_gpus: int, hbm_cap_bytes: int, n_microbatches: int,
                topo: Optional[L.Topology] = None) -> L.Plan:
    arr = _profile_array(layers)
    out = L.Plan()
    check(lib.mobius_plan(arr, len(layers), n_gpus, hbm_cap_bytes, n_microbatches,
                          C.byref(topo) if topo is not None else None, C.byref(out)))
    return out


PARTITION_MIP, PARTITION_MAX_STAGE, PARTITION_MIN_STAGE = 0, 1, 2


def mobius_plan_partition(layers, n_gpus: int, hbm_cap_bytes: int, n_microbatches: int, algo: int,
                          topo: Optional[L.Topology] = None) -> L.Plan:
    arr = _profile_array(layers)
    out = L.Plan()
    check(lib.mobius_plan_partition(arr, len(layers), n_gpus, hbm_cap_bytes, n_microbatches,
                                    C.byref(topo) if topo is not None else None, algo, C.byref(out)))
    return out


def mobius_plan_cost(layers, sizes: Sequence[int], n_gpus, hbm_cap_bytes, M, host_bw, p2p_bw, want_times=False):
    arr = _profile_array(layers)
    K = len(sizes)
    sz = (C.c_int * K)(*sizes)
    mk = C.c_int64()
    tf = (C.c_int64 * (K * M))() if want_times else None
    tb = (C.c_int64 * (K * M))() if want_times else None
    check(lib.mobius_plan_cost(arr, len(layers), sz, K, n_gpus, hbm_cap_bytes, M, host_bw or 0, p2p_bw or 0,
                               C.byref(mk), tf, tb))
    if want_times:
        return mk.value, np.array(tf[:], dtype=np.int64).reshape(K, M), np.array(tb[:], dtype=np.int64).reshape(K, M)
    return mk.value


def mobius_cross_map(n_stages: int, groups: Sequence[int]):
    N = len(groups)
    g = (C.c_int * N)(*groups)
    perm = (C.c_int * N)()
    c = C.c_double()
    num = C.c_int64()
    den = C.c_int64()
    check(lib.mobius_cross_map(n_stages, N, g, perm, C.byref(c), C.byref(num), C.byref(den)))
    return list(perm), c.value, num.value, den.value


def mobius_mapping_contention(n_stages: int, groups: Sequence[int], perm: Sequence[int]):
    N = len(groups)
    c = C.c_double()
    num = C.c_int64()
    den = C.c_int64()
    check(lib.mobius_mapping_contention(n_stages, N, (C.c_int * N)(*groups), (C.c_int * N)(*perm), C.byref(c),
                                        C.byref(num), C.byref(den)))
    return c.value, num.value, den.value


def mobius_layer_sizes(cfg: L.ModelCfg):
    out = (L.LayerProfile * L.MAX_LAYERS)()
    n = C.c_int()
    check(lib.mobius_layer_sizes(C.byref(cfg), out, C.byref(n)))
    return [out[i] for i in range(n.value)]


def mobius_arena_layer_sizes(cfg: L.ModelCfg):
    out = (L.LayerProfile * L.MAX_LAYERS)()
    n = C.c_int()
    check(lib.mobius_arena_layer_sizes(C.byref(cfg), out, C.byref(n)))
    return [out[i] for i in range(n.value)]


def mobius_arena_fixed_bytes(cfg: L.ModelCfg, n_microbatches: int, n_local_stages: int, flags: int) -> int:
    b = C.c_int64()
    check(lib.mobius_arena_fixed_bytes(C.byref(cfg), n_microbatches, n_local_stages, flags, C.byref(b)))
    return b.value


def mobius_profile(cfg: L.ModelCfg, device: int = 0):
    out = (L.LayerProfile * L.MAX_LAYERS)()
    n = C.c_int()
    check(lib.mobius_profile(C.byref(cfg), device, out, C.byref(n)))
    return [out[i] for i in range(n.value)]


def plan_from_sizes(sizes: Sequence[int], n_gpus: int, n_microbatches: int, perm: Optional[Sequence[int]] = None,
                    hbm_cap_bytes: int = 0) -> L.Plan:
    """Hand-built plan (fixed partition, round-robin over ``perm``)."""
    p = L.Plan()
    K = len(sizes)
    p.n_stages = K
    p.n_gpus = n_gpus
    p.n_microbatches = n_microbatches
    p.n_layers = int(sum(sizes))
    p.hbm_cap_bytes = hbm_cap_bytes
    perm = list(range(n_gpus)) if perm is None else list(perm)
    pos = 0
    p.stage_first_layer[0] = 0
    for j, s in enumerate(sizes):
        pos += s
        p.stage_first_layer[j + 1] = pos
        p.stage_gpu[j] = perm[j % n_gpus]
    for g in range(n_gpus):
        p.gpu_perm[g] = perm[g]
    return p


class MobiusContext:
    """One rank's mobius_ctx (SPMD: every rank constructs one)."""

    def __init__(self, cfg: L.ModelCfg, plan: L.Plan, rank: int = 0, world: int = 1, device: int = 0,
                 init_params: Optional[np.ndarray] = None, seed: int = 1234, flags: int = 0):
        self.cfg = cfg
        self.plan = plan
        self._ctx = C.c_void_p()
        d = L.Dist(rank, world, device, flags)
        ptr = None
        if init_params is not None:
            self._init = np.ascontiguousarray(init_params, dtype=np.float32)
            ptr = self._init.ctypes.data_as(C.c_void_p)
        check(lib.mobius_create(C.byref(cfg), C.byref(plan), C.byref(d), ptr, seed, C.byref(self._ctx)))
        if init_params is not None:
            del self._init

    # -- multi-rank plumbing (CUDA IPC handles travel over torch.distributed)
    def dist_export(self) -> bytes:
        buf = (C.c_char * 4096)()
        n = C.c_size_t()
        check(lib.mobius_dist_export(self._ctx, buf, 4096, C.byref(n)))
        return bytes(buf[:n.value])

    def dist_connect(self, blobs: Sequence[bytes]):
        ln = max(len(b) for b in blobs)
        flat = b"".join(b.ljust(ln, b"\0") for b in blobs)
        check(lib.mobius_dist_connect(self._ctx, flat, ln))

    def set_prefetch_groups(self, groups: Sequence[int]):
        g = (C.c_int * len(groups))(*groups)
        check(lib.mobius_set_prefetch_groups(self._ctx, g, len(groups)))

    def read_prefetch_tickets(self):
        buf = (C.c_int32 * 1024)()
        n = C.c_size_t()
        check(lib.mobius_read_prefetch_tickets(self._ctx, buf, 1024, C.byref(n)))
        return list(buf[:n.value])

    def step(self, tokens: np.ndarray) -> float:
        tok = np.ascontiguousarray(tokens, dtype=np.int32)
        loss = C.c_float()
        check(lib.mobius_step(self._ctx, tok.ctypes.data_as(C.c_void_p), tok.shape[0], C.byref(loss)))
        return loss.value

    def step_device(self, tokens_dev, n_microbatches: int) -> float:
        loss = C.c_float()
        check(lib.mobius_step_device(self._ctx, C.c_void_p(tokens_dev.data_ptr()), n_microbatches, C.byref(loss)))
        return loss.value

    def read_grads(self, n: int) -> np.ndarray:
        out = np.full(n, np.nan, dtype=np.float32)
        check(lib.mobius_read_grads(self._ctx, out.ctypes.data_as(C.c_void_p), n))
        return out

    def read_params(self, n: int) -> np.ndarray:
        out = np.full(n, np.nan, dtype=np.float32)
        check(lib.mobius_read_params(self._ctx, out.ctypes.data_as(C.c_void_p), n))
        return out

    def read_trace(self):
        cap = 1 << 16
        buf = (C.c_int32 * (3 * cap))()
        n = C.c_size_t()
        check(lib.mobius_read_trace(self._ctx, buf, cap, C.byref(n)))
        return [("F" if buf[3 * i] == 0 else "B", buf[3 * i + 1], buf[3 * i + 2]) for i in range(n.value)]

    def read_timeline(self):
        """Device timeline of the last step: list of (kind, stage, t0_ms, t1_ms),
        kind in h2d / fwd / bwd / d2h (include/mobius.h mobius_read_timeline)."""
        n = C.c_size_t()
        check(lib.mobius_read_timeline(self._ctx, None, 0, C.byref(n)))
        buf = (L.TimelineEvent * max(1, n.value))()
        check(lib.mobius_read_timeline(self._ctx, buf, n.value, C.byref(n)))
        return [(L.TL_KINDS[e.kind], e.stage, e.t0_ms, e.t1_ms) for e in buf[:n.value]]

    def stats(self) -> L.StepStats:
        s = L.StepStats()
        check(lib.mobius_stats(self._ctx, C.byref(s)))
        return s

    def close(self):
        if self._ctx:
            lib.mobius_destroy(self._ctx)
            self._ctx = C.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class _KT:
    """Kernel-level test entries (include/mobius_kernels.h) on torch tensors."""

    @staticmethod
    def _p(t):
        return None if t is None else C.c_void_p(t.data_ptr())

    def gemm(self, dtype, M, N, K, A, lda, a_mn, B, ldb, b_mn, Cm, ldc, c_f32=False, epi=0, alpha=1.0, bias=None,
             R=None, ldr=0, AUX=None, ldx=0, causal=0, accumulate=False, nb1=1, nb2=1, abs_=(0, 0), bbs=(0, 0),
             cbs=(0, 0), a_off=0, b_off=0, c_off=0):
        esz = 2 if dtype == BF16 else 4
        ce = 4 if (c_f32 or dtype == F32) else 2
        pa = C.c_void_p(A.data_ptr() + a_off * esz)
        pb = C.c_void_p(B.data_ptr() + b_off * esz)
        pc = C.c_void_p(Cm.data_ptr() + c_off * ce)
        check(lib.mobius_kt_gemm(dtype, M, N, K, nb1, nb2, pa, lda, abs_[0], abs_[1], int(a_mn), pb, ldb, bbs[0],
                                 bbs[1], int(b_mn), pc, ldc, cbs[0], cbs[1], int(c_f32), epi, alpha, self._p(bias),
                                 self._p(R), ldr, self._p(AUX), ldx, causal, int(accumulate)))

    def gemm_config(self, two_cta=-1, stream_k=-1):
        check(lib.mobius_kt_gemm_config(int(two_cta), int(stream_k)))

    def layernorm_fwd(self, dtype, x, g, b, y, mu, rstd, rows, h):
        check(lib.mobius_kt_layernorm_fwd(dtype, *map(self._p, (x, g, b, y, mu, rstd)), rows, h))

    def layernorm_bwd(self, dtype, dy, x, g, mu, rstd, dres, dx, dg, db, rows, h):
        check(lib.mobius_kt_layernorm_bwd(dtype, *map(self._p, (dy, x, g, mu, rstd, dres, dx, dg, db)), rows, h))

    def softmax_fwd(self, dtype, S, P, B, s, scale):
        check(lib.mobius_kt_softmax_fwd(dtype, self._p(S), self._p(P), B, s, scale))

    def softmax_bwd(self, dtype, P, dP, dS, B, s, scale):
        check(lib.mobius_kt_softmax_bwd(dtype, self._p(P), self._p(dP), self._p(dS), B, s, scale))

    def cross_entropy(self, dtype, logits, tok, loss_rows, rows, V, s, inv_ntok):
        check(lib.mobius_kt_cross_entropy(dtype, self._p(logits), self._p(tok), self._p(loss_rows), rows, V, s,
                                          inv_ntok))

    def embed_fwd(self, dtype, tok, wte, wpe, x, mbs, s, h):
        check(lib.mobius_kt_embed_fwd(dtype, *map(self._p, (tok, wte, wpe, x)), mbs, s, h))

    def embed_bwd(self, dtype, tok, dx, dwte, dwpe, mbs, s, h, V=None):
        V = dwte.shape[0] if V is None else V
        check(lib.mobius_kt_embed_bwd(dtype, *map(self._p, (tok, dx, dwte, dwpe)), mbs, s, h, V))

    def colsum(self, dtype, X, ld, rows, n, out):
        check(lib.mobius_kt_colsum(dtype, self._p(X), ld, rows, n, self._p(out)))

    def attention(self, dtype, mbs, s, nh, dh, qkv, o, dout=None, dqkv=None):
        check(lib.mobius_kt_attention(dtype, mbs, s, nh, dh, *map(self._p, (qkv, o, dout, dqkv))))

    def block(self, dtype, h, nh, s, mbs, w, x, y, dy=None, dx=None, grads=None):
        check(lib.mobius_kt_block(dtype, h, nh, s, mbs, *map(self._p, (w, x, y, dy, dx, grads))))


kt = _KT()
