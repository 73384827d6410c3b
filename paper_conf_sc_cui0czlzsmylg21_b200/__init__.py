"""Python binding of libabacus.so (include/abacus.h) -- argument marshalling only.

Every step of the candidate search runs in the CUDA library; PyTorch is used
for device memory, streams and process groups.  There is no CPU fallback:
importing works anywhere (so the CPU test-suite can check the exported
symbols), but every call needs the built library and an sm_100 GPU and raises
otherwise.
"""
from __future__ import annotations

import ctypes as C
import os
from typing import List, Optional, Sequence

import numpy as np

from . import _build

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = _build.LIB

# ---- constants (include/abacus.h) ------------------------------------------
ABACUS_OK, ABACUS_E_INVALID, ABACUS_E_DUP_MODEL, ABACUS_E_NOT_LOADED = 0, -1, -2, -3
ABACUS_E_CUDA, ABACUS_E_NCCL, ABACUS_E_DEVICE = -4, -5, -6
ABACUS_FP32, ABACUS_BF16, ABACUS_FP16 = 0, 1, 2
ABACUS_SPACE_GRID, ABACUS_SPACE_CHAIN, ABACUS_SPACE_AUTO = 0, 1, 2
ABACUS_DECIDE_OK, ABACUS_DECIDE_DROP, ABACUS_DECIDE_NONE = 0, 1, 2
K_MAX = 4

EXPORTED = ["abacus_create", "abacus_destroy", "abacus_last_error", "abacus_load_predictor",
            "abacus_encode_candidates", "abacus_encode_groups", "abacus_predict_batch",
            "abacus_select_group", "abacus_search", "abacus_search_batch", "abacus_search_mway", "abacus_search_grid", "abacus_search_sharded", "abacus_search_whatif",
            "abacus_combine_decisions", "abacus_nccl_unique_id",
            "abacus_nccl_comm_init", "abacus_nccl_comm_destroy", "abacus_peer_export", "abacus_peer_comm_init",
            "abacus_peer_comm_destroy", "abacus_kernel_launches",
            "abacus_last_kernel_ms", "abacus_set_timing", "abacus_set_stream", "abacus_abi_version",
            "abacus_train_begin", "abacus_train_step", "abacus_train_epoch", "abacus_train_params"]


class abacus_adam_t(C.Structure):
    _fields_ = [("beta1", C.c_float), ("beta2", C.c_float), ("eps", C.c_float)]


class abacus_slot_t(C.Structure):
    _fields_ = [("model_id", C.c_int32), ("start_op", C.c_int32), ("batch", C.c_int32),
                ("seqlen", C.c_int32), ("end_lo", C.c_int32), ("end_hi", C.c_int32),
                ("allow_absent", C.c_int32)]


class abacus_grid_t(C.Structure):
    _fields_ = [("k", C.c_int32), ("slot", abacus_slot_t * K_MAX)]


class _gslot(C.Structure):
    _fields_ = [("model_id", C.c_int32), ("ops", C.c_int32), ("ope", C.c_int32),
                ("batch", C.c_int32), ("seqlen", C.c_int32)]


class abacus_group_t(C.Structure):
    _fields_ = [("k", C.c_int32), ("slot", _gslot * K_MAX)]


class abacus_variant_t(C.Structure):
    _fields_ = [("batch", C.c_int32 * K_MAX), ("seqlen", C.c_int32 * K_MAX)]


class abacus_query_t(C.Structure):
    _fields_ = [("model_id", C.c_int32), ("next_op", C.c_int32), ("batch", C.c_int32),
                ("seqlen", C.c_int32), ("qos_ms", C.c_double), ("t_start_ms", C.c_double)]


class abacus_decision_t(C.Structure):
    _fields_ = [("status", C.c_int32), ("critical", C.c_int32), ("order", C.c_int32 * 4),
                ("end_op", C.c_int32 * 4), ("key", C.c_uint64), ("index", C.c_uint64),
                ("evaluated", C.c_uint64), ("total_ops", C.c_int32), ("headroom_ms", C.c_float),
                ("pred_ms", C.c_float), ("pred_critical_only_ms", C.c_float)]


class AbacusError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__("abacus error %d: %s" % (code, msg))
        self.code = code


_lib = None


def lib():
    """Load libabacus.so (fails loudly if it was not built: there is no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError("libabacus.so is not built (run __graft_entry__.build()); "
                               "the CUDA path has no CPU fallback")
        L = C.CDLL(LIB_PATH)
        P = C.POINTER
        vp = C.c_void_p
        L.abacus_create.argtypes = [C.c_int, C.c_int32, P(C.c_int32), C.c_int32, P(vp)]
        L.abacus_destroy.argtypes = [vp]
        L.abacus_destroy.restype = None
        L.abacus_last_error.argtypes = [vp]
        L.abacus_last_error.restype = C.c_char_p
        L.abacus_load_predictor.argtypes = [vp, P(C.c_float), C.c_size_t, C.c_int]
        L.abacus_encode_candidates.argtypes = [vp, P(abacus_grid_t), C.c_uint64, C.c_uint64, vp, vp]
        L.abacus_encode_groups.argtypes = [vp, vp, C.c_uint64, vp, vp, vp]
        L.abacus_predict_batch.argtypes = [vp, vp, C.c_uint64, vp, vp]
        L.abacus_select_group.argtypes = [vp, P(abacus_grid_t), C.c_uint64, C.c_uint64, vp, C.c_float, vp, vp]
        L.abacus_search.argtypes = [vp, P(abacus_query_t), C.c_int32, C.c_double, C.c_double, C.c_int32,
                                    C.c_uint64, P(abacus_decision_t)]
        L.abacus_search_batch.argtypes = [vp, P(abacus_query_t), P(C.c_int32), P(C.c_double), P(C.c_double),
                                          C.c_int32, C.c_int32, C.c_uint64, P(abacus_decision_t)]
        L.abacus_search_mway.argtypes = [vp, P(abacus_query_t), C.c_int32, C.c_double, C.c_double, C.c_int32,
                                         P(abacus_decision_t), P(C.c_int32)]
        L.abacus_search_grid.argtypes = [vp, P(abacus_grid_t), C.c_float, C.c_uint64, C.c_uint64, vp,
                                         P(abacus_decision_t)]
        L.abacus_search_sharded.argtypes = [vp, P(abacus_query_t), C.c_int32, C.c_double, C.c_double, C.c_int32,
                                            C.c_uint64, vp, P(abacus_decision_t)]
        L.abacus_search_whatif.argtypes = [vp, P(abacus_grid_t), P(abacus_variant_t), C.c_int32, C.c_float,
                                           P(abacus_decision_t), P(abacus_decision_t), P(C.c_int32)]
        L.abacus_combine_decisions.argtypes = [P(abacus_decision_t), C.c_int32, C.c_int32, P(abacus_decision_t)]
        L.abacus_nccl_unique_id.argtypes = [P(C.c_uint8)]
        L.abacus_nccl_comm_init.argtypes = [vp, C.c_int32, C.c_int32, P(C.c_uint8), P(vp)]
        L.abacus_peer_export.argtypes = [vp, P(C.c_uint8)]
        L.abacus_peer_comm_init.argtypes = [vp, C.c_int32, C.c_int32, P(C.c_uint8), P(vp)]
        L.abacus_peer_comm_destroy.argtypes = [vp]
        L.abacus_peer_comm_destroy.restype = None
        L.abacus_nccl_comm_destroy.argtypes = [vp]
        L.abacus_nccl_comm_destroy.restype = None
        L.abacus_kernel_launches.argtypes = [vp]
        L.abacus_kernel_launches.restype = C.c_uint64
        L.abacus_last_kernel_ms.argtypes = [vp]
        L.abacus_last_kernel_ms.restype = C.c_float
        L.abacus_set_timing.argtypes = [vp, C.c_int]
        L.abacus_set_stream.argtypes = [vp, vp]
        L.abacus_abi_version.argtypes = []
        L.abacus_train_begin.argtypes = [vp, P(C.c_float), C.c_size_t, P(abacus_adam_t)]
        L.abacus_train_step.argtypes = [vp, vp, vp, C.c_uint64, C.c_float, vp, vp]
        L.abacus_train_epoch.argtypes = [vp, vp, vp, C.c_uint64, C.c_uint32, C.c_float, vp, vp]
        L.abacus_train_params.argtypes = [vp, P(C.c_float), P(C.c_float)]
        _lib = L
    return _lib


def _check(ctx, rc):
    if rc != ABACUS_OK:
        msg = lib().abacus_last_error(ctx).decode() if ctx else ""
        raise AbacusError(rc, msg)


def _ptr(t) -> Optional[int]:
    if t is None:
        return None
    if isinstance(t, int):
        return t
    return t.data_ptr()


def _stream(stream) -> Optional[int]:
    if stream is None:
        return None
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


def make_grid(slots) -> abacus_grid_t:
    """slots: objects with model_id, start_op, batch, seqlen, end_lo, end_hi, allow_absent"""
    g = abacus_grid_t()
    g.k = len(slots)
    for j, s in enumerate(slots):
        g.slot[j] = abacus_slot_t(s.model_id, s.start_op, s.batch, s.seqlen, s.end_lo, s.end_hi, s.allow_absent)
    return g


def make_groups(groups) -> "bytes":
    """list of lists of (model, ops, ope, bs, seqlen) -> packed abacus_group_t records"""
    arr = (abacus_group_t * len(groups))()
    for i, g in enumerate(groups):
        arr[i].k = len(g)
        for j, s in enumerate(g):
            arr[i].slot[j] = _gslot(*s)
    return bytes(arr)


# ---- the C ABI, same names ------------------------------------------------
def abacus_create(device: int, ops_per_model: Sequence[int], k_max: int = K_MAX) -> int:
    n = len(ops_per_model)
    arr = (C.c_int32 * n)(*ops_per_model)
    out = C.c_void_p()
    _check(None, lib().abacus_create(device, n, arr, k_max, C.byref(out)))
    return out.value


def abacus_destroy(ctx: int) -> None:
    lib().abacus_destroy(ctx)


def abacus_last_error(ctx: int) -> str:
    return lib().abacus_last_error(ctx).decode()


def abacus_load_predictor(ctx: int, params, precision: int) -> None:
    p = np.ascontiguousarray(params, dtype=np.float32)
    _check(ctx, lib().abacus_load_predictor(ctx, p.ctypes.data_as(C.POINTER(C.c_float)), p.size, precision))


def abacus_encode_candidates(ctx, grid: abacus_grid_t, first: int, count: int, d_features, stream=None):
    _check(ctx, lib().abacus_encode_candidates(ctx, C.byref(grid), first, count, _ptr(d_features),
                                               _stream(stream)))


def abacus_encode_groups(ctx, d_groups, count: int, d_features, d_bad=None, stream=None):
    _check(ctx, lib().abacus_encode_groups(ctx, _ptr(d_groups), count, _ptr(d_features), _ptr(d_bad),
                                           _stream(stream)))


def abacus_predict_batch(ctx, d_features, count: int, d_latency_ms, stream=None):
    _check(ctx, lib().abacus_predict_batch(ctx, _ptr(d_features), count, _ptr(d_latency_ms), _stream(stream)))


def abacus_select_group(ctx, grid: abacus_grid_t, first: int, count: int, d_latency_ms, headroom_ms: float,
                        d_best_key, stream=None):
    _check(ctx, lib().abacus_select_group(ctx, C.byref(grid), first, count, _ptr(d_latency_ms),
                                          float(headroom_ms), _ptr(d_best_key), _stream(stream)))


def abacus_search(ctx, queries, now_ms: float, inflight_pred_ms: float, space: int = ABACUS_SPACE_GRID,
                  grid_budget: int = 2**40) -> abacus_decision_t:
    k = len(queries)
    qa = (abacus_query_t * k)(*[abacus_query_t(q.model_id, q.next_op, q.batch, q.seqlen, q.qos_ms,
                                               q.t_start_ms) for q in queries])
    out = abacus_decision_t()
    _check(ctx, lib().abacus_search(ctx, qa, k, float(now_ms), float(inflight_pred_ms), space, grid_budget,
                                    C.byref(out)))
    return out


def abacus_search_batch(ctx, decisions, space: int = ABACUS_SPACE_GRID, grid_budget: int = 2**40):
    """decisions: sequence of (queries, now_ms, inflight_pred_ms); returns a list of decisions."""
    n = len(decisions)
    qa = (abacus_query_t * (4 * n))()
    ka = (C.c_int32 * n)()
    now = (C.c_double * n)()
    inf = (C.c_double * n)()
    for i, (queries, now_ms, inflight) in enumerate(decisions):
        ka[i] = len(queries)
        now[i] = float(now_ms)
        inf[i] = float(inflight)
        for j, q in enumerate(queries):
            qa[4 * i + j] = abacus_query_t(q.model_id, q.next_op, q.batch, q.seqlen, q.qos_ms, q.t_start_ms)
    out = (abacus_decision_t * n)()
    _check(ctx, lib().abacus_search_batch(ctx, qa, ka, now, inf, n, space, grid_budget, out))
    return list(out)


def abacus_search_mway(ctx, queries, now_ms: float, inflight_pred_ms: float, ways: int):
    """Returns (decision, rounds)."""
    k = len(queries)
    qa = (abacus_query_t * k)(*[abacus_query_t(q.model_id, q.next_op, q.batch, q.seqlen, q.qos_ms,
                                               q.t_start_ms) for q in queries])
    out = abacus_decision_t()
    rounds = C.c_int32()
    _check(ctx, lib().abacus_search_mway(ctx, qa, k, float(now_ms), float(inflight_pred_ms), int(ways),
                                         C.byref(out), C.byref(rounds)))
    return out, int(rounds.value)


def abacus_search_grid(ctx, grid: abacus_grid_t, headroom_ms: float, first: int, count: int,
                       nccl_comm: Optional[int] = None) -> abacus_decision_t:
    out = abacus_decision_t()
    _check(ctx, lib().abacus_search_grid(ctx, C.byref(grid), float(headroom_ms), first, count, nccl_comm,
                                         C.byref(out)))
    return out


def abacus_search_sharded(ctx, queries, now_ms: float, inflight_pred_ms: float, space: int = ABACUS_SPACE_GRID,
                          grid_budget: int = 2**40, nccl_comm: Optional[int] = None) -> abacus_decision_t:
    k = len(queries)
    qa = (abacus_query_t * k)(*[abacus_query_t(q.model_id, q.next_op, q.batch, q.seqlen, q.qos_ms,
                                               q.t_start_ms) for q in queries])
    out = abacus_decision_t()
    _check(ctx, lib().abacus_search_sharded(ctx, qa, k, float(now_ms), float(inflight_pred_ms), space, grid_budget,
                                            nccl_comm, C.byref(out)))
    return out


def abacus_search_whatif(ctx, grid: abacus_grid_t, variants, headroom_ms: float):
    """variants: sequence of (batch per slot, seqlen per slot).  Returns
    (per-variant decisions, best decision, best variant index or -1)."""
    n = len(variants)
    va = (abacus_variant_t * max(n, 1))()
    for i, (bs, sl) in enumerate(variants):
        for j in range(min(len(bs), K_MAX)):
            va[i].batch[j] = int(bs[j])
            va[i].seqlen[j] = int(sl[j])
    per = (abacus_decision_t * max(n, 1))()
    best = abacus_decision_t()
    bv = C.c_int32()
    _check(ctx, lib().abacus_search_whatif(ctx, C.byref(grid), va, n, float(headroom_ms), per, C.byref(best),
                                           C.byref(bv)))
    return list(per)[:n], best, int(bv.value)


def abacus_combine_decisions(per_rank: Sequence[abacus_decision_t], drop_test: bool = False) -> abacus_decision_t:
    """Host-side a6 combine of per-rank sweep decisions (rank order); needs no GPU."""
    n = len(per_rank)
    arr = (abacus_decision_t * max(n, 1))(*per_rank)
    out = abacus_decision_t()
    _check(None, lib().abacus_combine_decisions(arr, n, 1 if drop_test else 0, C.byref(out)))
    return out


def abacus_nccl_unique_id() -> bytes:
    buf = (C.c_uint8 * 128)()
    _check(None, lib().abacus_nccl_unique_id(buf))
    return bytes(buf)


def abacus_nccl_comm_init(ctx, nranks: int, rank: int, uid: bytes) -> int:
    buf = (C.c_uint8 * 128)(*uid)
    out = C.c_void_p()
    _check(ctx, lib().abacus_nccl_comm_init(ctx, nranks, rank, buf, C.byref(out)))
    return out.value


def abacus_nccl_comm_destroy(comm: int) -> None:
    lib().abacus_nccl_comm_destroy(comm)


PEER_BLOB = 128


def abacus_peer_export(ctx) -> bytes:
    buf = (C.c_uint8 * PEER_BLOB)()
    _check(ctx, lib().abacus_peer_export(ctx, buf))
    return bytes(buf)


def abacus_peer_comm_init(ctx, nranks: int, rank: int, blobs: Sequence[bytes]) -> int:
    raw = b"".join(blobs)
    buf = (C.c_uint8 * len(raw))(*raw)
    out = C.c_void_p()
    _check(ctx, lib().abacus_peer_comm_init(ctx, nranks, rank, buf, C.byref(out)))
    return out.value


def abacus_peer_comm_destroy(comm: int) -> None:
    lib().abacus_peer_comm_destroy(comm)


def peer_comm_from_process_group(ctx, group=None) -> int:
    """Every rank exports its mailbox, torch.distributed all-gathers the blobs,
    every rank opens the others' mailboxes (CUDA IPC)."""
    import torch.distributed as dist
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    blobs = [None] * world
    dist.all_gather_object(blobs, abacus_peer_export(ctx), group=group)
    return abacus_peer_comm_init(ctx, world, rank, blobs)


def abacus_kernel_launches(ctx) -> int:
    return int(lib().abacus_kernel_launches(ctx))


def abacus_last_kernel_ms(ctx) -> float:
    return float(lib().abacus_last_kernel_ms(ctx))


def abacus_set_timing(ctx, on: bool) -> None:
    _check(ctx, lib().abacus_set_timing(ctx, 1 if on else 0))


def abacus_set_stream(ctx, stream) -> None:
    _check(ctx, lib().abacus_set_stream(ctx, _stream(stream)))


def abacus_train_begin(ctx, params, beta1: float = 0.9, beta2: float = 0.999, eps: float = 1e-8) -> None:
    p = np.ascontiguousarray(params, dtype=np.float32)
    opt = abacus_adam_t(beta1, beta2, eps)
    _check(ctx, lib().abacus_train_begin(ctx, p.ctypes.data_as(C.POINTER(C.c_float)), p.size, C.byref(opt)))


def abacus_train_step(ctx, d_features, d_latency_ms, count: int, lr: float, d_grad=None, stream=None) -> None:
    _check(ctx, lib().abacus_train_step(ctx, _ptr(d_features), _ptr(d_latency_ms), count, lr, _ptr(d_grad),
                                        _stream(stream)))


def abacus_train_epoch(ctx, d_features, d_latency_ms, count: int, batch: int, lr: float, d_losses=None,
                       stream=None) -> None:
    _check(ctx, lib().abacus_train_epoch(ctx, _ptr(d_features), _ptr(d_latency_ms), count, batch, lr,
                                         _ptr(d_losses), _stream(stream)))


def abacus_train_params(ctx, n_params: int):
    """Returns (params float32 array, last step's loss)."""
    out = np.zeros(n_params, dtype=np.float32)
    loss = C.c_float()
    _check(ctx, lib().abacus_train_params(ctx, out.ctypes.data_as(C.POINTER(C.c_float)), C.byref(loss)))
    return out, float(loss.value)


def abacus_abi_version() -> int:
    return int(lib().abacus_abi_version())


# ---- NCCL bootstrap over a torch process group -------------------------------
def nccl_comm_from_process_group(ctx, group=None) -> int:
    """Rank 0 draws an ncclUniqueId, torch.distributed broadcasts the 128 bytes,
    every rank creates its communicator on the ctx's device."""
    import torch
    import torch.distributed as dist
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    uid = abacus_nccl_unique_id() if rank == 0 else bytes(128)
    obj = [uid]
    dist.broadcast_object_list(obj, src=0, group=group)
    return abacus_nccl_comm_init(ctx, world, rank, obj[0])


def shard_range(T: int, rank: int, world: int):
    """Contiguous shard [floor(rT/G), floor((r+1)T/G)) of the candidate index space."""
    a = (rank * T) // world
    b = ((rank + 1) * T) // world
    return a, b - a
