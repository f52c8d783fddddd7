"""ctypes binding of libmobius (include/mobius.h, include/mobius_kernels.h).

Argument marshalling only: every step of the hot path runs inside
libmobius.so.  There is no Python or CPU fallback - if the shared library
is missing this module raises at import.
"""
from __future__ import annotations

import ctypes as C
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
# MOBIUS_LIB_PATH: an alternative build of the same library (kernel A/B
# timing tools only); there is no other implementation behind the binding
LIB_PATH = os.environ.get("MOBIUS_LIB_PATH") or os.path.join(_HERE, "libmobius.so")

MAX_GPUS = 16
MAX_LAYERS = 256
BF16 = 0
F32 = 1

STATUS = {0: "MOBIUS_OK", -1: "MOBIUS_EINVAL", -2: "MOBIUS_EINFEASIBLE", -3: "MOBIUS_ENOMEM",
          -4: "MOBIUS_ECUDA", -5: "MOBIUS_ENCCL", -6: "MOBIUS_ETOPO", -7: "MOBIUS_ESTATE"}


class MobiusError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"{STATUS.get(code, code)}: {msg}")
        self.code = code


class ModelCfg(C.Structure):
    _fields_ = [("n_layers", C.c_int), ("hidden", C.c_int), ("n_heads", C.c_int), ("seq_len", C.c_int),
                ("vocab", C.c_int), ("micro_batch", C.c_int), ("dtype", C.c_int), ("lr", C.c_float),
                ("beta1", C.c_float), ("beta2", C.c_float), ("eps", C.c_float), ("weight_decay", C.c_float)]


class LayerProfile(C.Structure):
    _fields_ = [("t_fwd_ns", C.c_int64), ("t_bwd_ns", C.c_int64), ("mem_fwd", C.c_int64), ("mem_bwd", C.c_int64),
                ("xfer_fwd", C.c_int64), ("xfer_bwd", C.c_int64), ("act_out", C.c_int64)]


class Topology(C.Structure):
    _fields_ = [("n_gpus", C.c_int), ("group", C.c_int * MAX_GPUS), ("host_bw_Bps", C.c_int64),
                ("p2p_bw_Bps", C.c_int64)]


class Plan(C.Structure):
    _fields_ = [("n_stages", C.c_int), ("n_gpus", C.c_int), ("n_microbatches", C.c_int), ("n_layers", C.c_int),
                ("stage_first_layer", C.c_int * (MAX_LAYERS + 1)), ("stage_gpu", C.c_int * MAX_LAYERS),
                ("gpu_perm", C.c_int * MAX_GPUS), ("hbm_cap_bytes", C.c_int64), ("makespan_ns", C.c_int64),
                ("exhaustive", C.c_int), ("contention", C.c_double), ("contention_num", C.c_int64),
                ("contention_den", C.c_int64), ("h2d_bytes", C.c_int64 * MAX_GPUS),
                ("d2h_bytes", C.c_int64 * MAX_GPUS), ("p2p_bytes", C.c_int64 * MAX_GPUS)]


class Dist(C.Structure):
    _fields_ = [("rank", C.c_int), ("world", C.c_int), ("device", C.c_int), ("flags", C.c_int)]


class TimelineEvent(C.Structure):
    _fields_ = [("kind", C.c_int32), ("stage", C.c_int32), ("t0_ms", C.c_double), ("t1_ms", C.c_double)]


TL_KINDS = {0: "h2d", 1: "fwd", 2: "bwd", 3: "d2h", 4: "d2d", 5: "ckpt_d2h", 6: "ckpt_h2d"}


class StepStats(C.Structure):
    _fields_ = [("step_ns", C.c_int64), ("device_step_ns", C.c_int64), ("h2d_bytes", C.c_int64),
                ("d2h_bytes", C.c_int64), ("p2p_bytes", C.c_int64), ("n_h2d_copies", C.c_int64),
                ("h2d_GBps_median", C.c_double), ("h2d_GBps_max", C.c_double), ("gemm_ns", C.c_int64),
                ("gemm_flops", C.c_int64), ("gemm_launches", C.c_int64), ("attn_ns", C.c_int64),
                ("elem_ns", C.c_int64), ("kernel_launches", C.c_int64), ("exposed_load_ns", C.c_int64),
                ("update_tail_ns", C.c_int64), ("arena_bytes", C.c_int64), ("ring_bytes", C.c_int64),
                ("pinned_bytes", C.c_int64), ("host_update_ns", C.c_int64), ("n_local_stages", C.c_int),
                ("recompute", C.c_int), ("timing_stride", C.c_int), ("d2d_bytes", C.c_int64),
                ("ckpt_d2h_bytes", C.c_int64), ("ckpt_h2d_bytes", C.c_int64), ("exposed_ckpt_ns", C.c_int64)]


FLAG_TIMING = 1
FLAG_KEEP_ACTS = 2
FLAG_DEVICE_TAIL_UPDATE = 4
FLAG_ARENA_CAP = 8
FLAG_CKPT_OFFLOAD = 16

P = C.c_void_p
I = C.c_int
I64 = C.c_int64
F = C.c_float

# name -> (restype, argtypes); every symbol declared in include/*.h
SIGNATURES = {
    "mobius_plan": (I, [C.POINTER(LayerProfile), I, I, I64, I, C.POINTER(Topology), C.POINTER(Plan)]),
    "mobius_plan_partition": (I, [C.POINTER(LayerProfile), I, I, I64, I, C.POINTER(Topology), I, C.POINTER(Plan)]),
    "mobius_plan_search_nodes": (I64, []),
    "mobius_plan_cost": (I, [C.POINTER(LayerProfile), I, C.POINTER(C.c_int), I, I, I64, I, I64, I64,
                             C.POINTER(I64), C.POINTER(I64), C.POINTER(I64)]),
    "mobius_cross_map": (I, [I, I, C.POINTER(C.c_int), C.POINTER(C.c_int), C.POINTER(C.c_double),
                             C.POINTER(I64), C.POINTER(I64)]),
    "mobius_mapping_contention": (I, [I, I, C.POINTER(C.c_int), C.POINTER(C.c_int), C.POINTER(C.c_double),
                                      C.POINTER(I64), C.POINTER(I64)]),
    "mobius_discover_topology": (I, [C.POINTER(Topology)]),
    "mobius_topology_from_bw": (I, [I, P, P, C.c_double, C.POINTER(Topology)]),
    "mobius_probe_topology": (I, [I64, C.c_double, C.POINTER(Topology), P, P]),
    "mobius_layer_sizes": (I, [C.POINTER(ModelCfg), C.POINTER(LayerProfile), C.POINTER(C.c_int)]),
    "mobius_profile": (I, [C.POINTER(ModelCfg), I, C.POINTER(LayerProfile), C.POINTER(C.c_int)]),
    "mobius_arena_layer_sizes": (I, [C.POINTER(ModelCfg), C.POINTER(LayerProfile), C.POINTER(C.c_int)]),
    "mobius_arena_fixed_bytes": (I, [C.POINTER(ModelCfg), I, I, I, C.POINTER(I64)]),
    "mobius_create": (I, [C.POINTER(ModelCfg), C.POINTER(Plan), C.POINTER(Dist), P, C.c_uint64, C.POINTER(P)]),
    "mobius_dist_export": (I, [P, P, C.c_size_t, C.POINTER(C.c_size_t)]),
    "mobius_dist_connect": (I, [P, P, C.c_size_t]),
    "mobius_set_prefetch_groups": (I, [P, P, I]),
    "mobius_read_prefetch_tickets": (I, [P, P, C.c_size_t, C.POINTER(C.c_size_t)]),
    "mobius_step": (I, [P, P, I, C.POINTER(F)]),
    "mobius_step_device": (I, [P, P, I, C.POINTER(F)]),
    "mobius_read_grads": (I, [P, P, C.c_size_t]),
    "mobius_read_params": (I, [P, P, C.c_size_t]),
    "mobius_read_trace": (I, [P, P, C.c_size_t, C.POINTER(C.c_size_t)]),
    "mobius_stats": (I, [P, C.POINTER(StepStats)]),
    "mobius_read_timeline": (I, [P, P, C.c_size_t, C.POINTER(C.c_size_t)]),
    "mobius_destroy": (None, [P]),
    "mobius_last_error": (C.c_char_p, []),
    "mobius_build_info": (C.c_char_p, []),
    "mobius_kt_gemm_config": (I, [I, I]),
    "mobius_kt_gemm": (I, [I, I, I, I, I, I, P, I64, I64, I64, I, P, I64, I64, I64, I, P, I64, I64, I64, I, I, F,
                           P, P, I64, P, I64, I, I]),
    "mobius_kt_layernorm_fwd": (I, [I, P, P, P, P, P, P, I, I]),
    "mobius_kt_layernorm_bwd": (I, [I, P, P, P, P, P, P, P, P, P, I, I]),
    "mobius_kt_softmax_fwd": (I, [I, P, P, I, I, F]),
    "mobius_kt_softmax_bwd": (I, [I, P, P, P, I, I, F]),
    "mobius_kt_cross_entropy": (I, [I, P, P, P, I, I, I, F]),
    "mobius_kt_embed_fwd": (I, [I, P, P, P, P, I, I, I]),
    "mobius_kt_embed_bwd": (I, [I, P, P, P, P, I, I, I, I]),
    "mobius_kt_colsum": (I, [I, P, I64, I, I, P]),
    "mobius_kt_block": (I, [I, I, I, I, I, P, P, P, P, P, P]),
    "mobius_kt_attention": (I, [I, I, I, I, I, P, P, P, P]),
}


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} not built; run __graft_entry__.build() "
                          "(python -m paper_conf_asplos_fengxtwls23_b200.build)")
    lib = C.CDLL(LIB_PATH)
    for name, (res, args) in SIGNATURES.items():
        fn = getattr(lib, name, None)
        if fn is None:
            MISSING.append(name)
            continue
        fn.restype = res
        fn.argtypes = args
    return lib


MISSING: list = []


lib = _load()


def check(rc):
    if rc != 0:
        raise MobiusError(rc, (lib.mobius_last_error() or b"").decode())
    return rc
