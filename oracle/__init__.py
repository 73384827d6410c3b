"""fp64 CPU oracle for the Abacus candidate search -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline``
/ ``--impl reference`` legs may import this package.  It shares no code with
the CUDA path (``paper_conf_sc_cui0czlzsmylg21_b200``) and never imports it.

``abacus_oracle.c`` is the oracle proper (plain C, double precision, one
thread); this module is ctypes marshalling plus :mod:`oracle.brute`, a
pure-Python brute force for tiny inputs.  Parity pins: tests/test_oracle_*.py.
Parity unpinned: predicted values on real workloads (the paper's trained
weights and profiled data are not available; SURVEY §8(c) last row).
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "abacus_oracle.c")
LIB = os.path.join(HERE, "liboracle.so")


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (plain -O2, no FMA contraction)."""
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-std=c11",
                               "-shared", "-fPIC", "-o", LIB, SRC, "-lm"])
    return LIB


class Present(C.Structure):
    _fields_ = [("model_id", C.c_int32), ("ops", C.c_int32), ("ope", C.c_int32),
                ("bs", C.c_int32), ("seqlen", C.c_int32)]


class GSlot(C.Structure):
    _fields_ = [("model_id", C.c_int32), ("start_op", C.c_int32), ("batch", C.c_int32),
                ("seqlen", C.c_int32), ("end_lo", C.c_int32), ("end_hi", C.c_int32),
                ("allow_absent", C.c_int32)]


class QueryC(C.Structure):
    _fields_ = [("model_id", C.c_int32), ("next_op", C.c_int32), ("batch", C.c_int32),
                ("seqlen", C.c_int32), ("qos_ms", C.c_double), ("t_start_ms", C.c_double)]


class SweepResult(C.Structure):
    _fields_ = [("best_key", C.c_uint64), ("best_index", C.c_uint64), ("best_y", C.c_double),
                ("y0", C.c_double), ("feasible", C.c_uint64), ("evaluated", C.c_uint64),
                ("hash", C.c_uint64), ("maxkey_strict", C.c_uint64), ("maxkey_loose", C.c_uint64),
                ("best_sum_n", C.c_int32), ("pad", C.c_int32)]


class Decision(C.Structure):
    _fields_ = [("status", C.c_int32), ("critical", C.c_int32), ("order", C.c_int32 * 4),
                ("end_op", C.c_int32 * 4), ("space_used", C.c_int32), ("total_ops", C.c_int32),
                ("key", C.c_uint64), ("index", C.c_uint64), ("evaluated", C.c_uint64),
                ("feasible", C.c_uint64), ("maxkey_strict", C.c_uint64), ("maxkey_loose", C.c_uint64),
                ("headroom_ms", C.c_double), ("pred_ms", C.c_double),
                ("pred_critical_only_ms", C.c_double), ("h", C.c_double * 4)]


class MWay(C.Structure):
    _fields_ = [("status", C.c_int32), ("rounds", C.c_int32), ("predictions", C.c_int32),
                ("total_ops", C.c_int32), ("u", C.c_uint64), ("headroom_ms", C.c_double),
                ("pred_ms", C.c_double), ("pred_critical_only_ms", C.c_double), ("end_op", C.c_int32 * 4),
                ("order", C.c_int32 * 4)]


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
        L = _lib
        P = C.POINTER
        L.orc_splitmix64.restype = C.c_uint64
        L.orc_splitmix64.argtypes = [C.c_uint64]
        L.orc_fnv1a64.restype = C.c_uint64
        L.orc_fnv1a64.argtypes = [P(C.c_int16), C.c_int32]
        L.orc_headroom.restype = C.c_double
        L.orc_headroom.argtypes = [C.c_double] * 4
        L.orc_order.restype = None
        L.orc_order.argtypes = [C.c_int32, P(C.c_double), P(C.c_int32), P(C.c_int32)]
        L.orc_encode.restype = C.c_int32
        L.orc_encode.argtypes = [C.c_int32, C.c_int32, C.c_int32, P(Present), P(C.c_int16)]
        L.orc_encode_groups.restype = C.c_int32
        L.orc_encode_groups.argtypes = [C.c_int32, C.c_int32, C.c_int64, P(Present), P(C.c_int16)]
        L.orc_mlp64.restype = C.c_double
        L.orc_mlp64.argtypes = [P(C.c_float), C.c_int32, P(C.c_int16)]
        L.orc_mlp64_batch.restype = None
        L.orc_mlp64_batch.argtypes = [P(C.c_float), C.c_int32, P(C.c_int16), C.c_int64, P(C.c_double)]
        L.orc_round_bf16.restype = C.c_double
        L.orc_round_bf16.argtypes = [C.c_double]
        L.orc_mlp64_emu.restype = C.c_double
        L.orc_mlp64_emu.argtypes = [P(C.c_float), C.c_int32, P(C.c_int16), C.c_int32]
        L.orc_mlp64_emu_batch.restype = None
        L.orc_mlp64_emu_batch.argtypes = [P(C.c_float), C.c_int32, P(C.c_int16), C.c_int64,
                                          C.c_int32, P(C.c_double)]
        L.orc_grid_size.restype = C.c_uint64
        L.orc_grid_size.argtypes = [C.c_int32, P(GSlot)]
        L.orc_sweep.restype = C.c_int32
        L.orc_sweep.argtypes = [C.c_int32, C.c_int32, P(C.c_float), C.c_int32, P(GSlot), C.c_double,
                                C.c_uint64, C.c_uint64, C.c_double, C.c_int32, P(C.c_double),
                                P(C.c_int16), P(C.c_int32), P(SweepResult)]
        L.orc_sweep_shell.restype = C.c_int32
        L.orc_sweep_shell.argtypes = [C.c_int32, C.c_int32, P(C.c_float), C.c_int32, P(GSlot), C.c_double,
                                      C.c_int32, C.c_double, C.c_int32, P(SweepResult)]
        L.orc_search.restype = C.c_int32
        L.orc_search.argtypes = [C.c_int32, C.c_int32, P(C.c_int32), P(C.c_float), P(QueryC),
                                 C.c_int32, C.c_double, C.c_double, C.c_int32, C.c_uint64,
                                 C.c_double, C.c_int32, P(Decision)]
        L.orc_search_mway.restype = C.c_int32
        L.orc_search_mway.argtypes = [C.c_int32, C.c_int32, P(C.c_int32), P(C.c_float), P(QueryC), C.c_int32,
                                      C.c_double, C.c_double, C.c_int32, C.c_int32, P(MWay)]
    return _lib


def _f32(p):
    p = np.ascontiguousarray(p, dtype=np.float32)
    return p, p.ctypes.data_as(C.POINTER(C.c_float))


def _i16(x):
    x = np.ascontiguousarray(x, dtype=np.int16)
    return x, x.ctypes.data_as(C.POINTER(C.c_int16))


# ----------------------------------------------------------------------------
def splitmix64(z: int) -> int:
    return int(lib().orc_splitmix64(z & (2**64 - 1)))


def fnv1a64(x) -> int:
    x, px = _i16(x)
    return int(lib().orc_fnv1a64(px, x.size))


def headroom(qos, t_start, now, inflight) -> float:
    return float(lib().orc_headroom(qos, t_start, now, inflight))


def order(h, model_ids):
    k = len(h)
    ha = (C.c_double * k)(*h)
    ma = (C.c_int32 * k)(*model_ids)
    o = (C.c_int32 * k)()
    lib().orc_order(k, ha, ma, o)
    return list(o)


def encode(n_models, kmax, present):
    """present: list of (model, ops, ope, bs, seqlen) -> int16[n_models + 4 kmax]"""
    n = len(present)
    arr = (Present * max(n, 1))(*[Present(*p) for p in present])
    x = np.zeros(n_models + 4 * kmax, dtype=np.int16)
    rc = lib().orc_encode(n_models, kmax, n, arr, x.ctypes.data_as(C.POINTER(C.c_int16)))
    if rc != 0:
        raise ValueError("orc_encode rejected the group")
    return x


def encode_groups(n_models, kmax, groups):
    """groups: list of lists of (model, ops, ope, bs, seqlen) -> int16[count, D]"""
    cnt = len(groups)
    a = np.zeros((cnt, kmax, 5), dtype=np.int32)
    for i, g in enumerate(groups):
        for j, s in enumerate(g):
            a[i, j] = s
    x = np.zeros((cnt, n_models + 4 * kmax), dtype=np.int16)
    rc = lib().orc_encode_groups(n_models, kmax, cnt, a.ctypes.data_as(C.POINTER(Present)),
                                 x.ctypes.data_as(C.POINTER(C.c_int16)))
    if rc != 0:
        raise ValueError("orc_encode_groups rejected a group")
    return x


def mlp64(params, x) -> float:
    p, pp = _f32(params)
    x, px = _i16(x)
    return float(lib().orc_mlp64(pp, x.size, px))


def mlp64_batch(params, X):
    p, pp = _f32(params)
    X, px = _i16(X)
    cnt, d = X.shape
    y = np.zeros(cnt, dtype=np.float64)
    lib().orc_mlp64_batch(pp, d, px, cnt, y.ctypes.data_as(C.POINTER(C.c_double)))
    return y


def round_bf16(v: float) -> float:
    return float(lib().orc_round_bf16(v))


def mlp64_emu_batch(params, X, flags=15):
    p, pp = _f32(params)
    X, px = _i16(X)
    cnt, d = X.shape
    y = np.zeros(cnt, dtype=np.float64)
    lib().orc_mlp64_emu_batch(pp, d, px, cnt, flags, y.ctypes.data_as(C.POINTER(C.c_double)))
    return y


def _gslots(grid):
    k = len(grid)
    return (GSlot * k)(*[GSlot(s.model_id, s.start_op, s.batch, s.seqlen, s.end_lo, s.end_hi,
                               s.allow_absent) for s in grid])


def grid_size(grid) -> int:
    return int(lib().orc_grid_size(len(grid), _gslots(grid)))


def sweep(params, grid, H, first=0, count=None, eps=1e-4, n_models=8, kmax=4, emu_flags=0,
          want_y=False, want_x=False, want_ope=False):
    """Sweep [first, first+count) of a grid; returns (SweepResult, y, x, ope)."""
    T = grid_size(grid)
    if count is None:
        count = T - first
    count = max(0, min(count, T - first))
    p, pp = _f32(params)
    d = n_models + 4 * kmax
    k = len(grid)
    y = np.zeros(count, dtype=np.float64) if want_y else None
    x = np.zeros((count, d), dtype=np.int16) if want_x else None
    o = np.zeros((count, k), dtype=np.int32) if want_ope else None
    r = SweepResult()
    rc = lib().orc_sweep(n_models, kmax, pp, k, _gslots(grid), float(H), first, count, eps, emu_flags,
                         y.ctypes.data_as(C.POINTER(C.c_double)) if want_y else None,
                         x.ctypes.data_as(C.POINTER(C.c_int16)) if want_x else None,
                         o.ctypes.data_as(C.POINTER(C.c_int32)) if want_ope else None, C.byref(r))
    if rc != 0:
        raise ValueError("orc_sweep rejected the grid")
    return r, y, x, o


def whatif(params, grid, variants, H, eps=1e-4, n_models=8, kmax=4):
    """What-if sweep (bs / seqlen as swept grid dimensions;
    the batch size is chosen by the load balancer at run time and inputs differ
    in length).  ``variants`` is a list of (batch per slot, seqlen
    per slot); variant v replaces the grid slots' bs and seqlen (Fig.-8
    features) and its candidates take the indices
    v * T + t (variant the most significant digit, T = |grid|).  The selection
    rule is the grid's (max sum_n, then max index, reading c12) over all
    variants: among groups of equal size the later variant wins.
    Returns (per-variant SweepResults, (best key over all variants, its
    variant or -1, its grid index t), (maxkey_strict, maxkey_loose) with the
    per-variant acceptance keys lifted to global indices)."""
    T = grid_size(grid)
    per = []
    best = (0, -1, 0)
    strict = loose = 0
    for v, (bss, sls) in enumerate(variants):
        g = [type(s)(s.model_id, s.start_op, int(bss[j]), int(sls[j]), s.end_lo, s.end_hi, s.allow_absent)
             for j, s in enumerate(grid)]
        r, _, _, _ = sweep(params, g, H, eps=eps, n_models=n_models, kmax=kmax)
        per.append(r)
        lift = lambda key: ((key >> 40) << 40) | (v * T + (key & ((1 << 40) - 1))) if key else 0  # noqa: E731
        if r.best_key and lift(r.best_key) > best[0]:
            best = (lift(r.best_key), v, r.best_index)
        strict = max(strict, lift(r.maxkey_strict))
        loose = max(loose, lift(r.maxkey_loose))
    return per, best, (strict, loose)


def sweep_shell(params, grid, H, nsum_min, eps=1e-4, n_models=8, kmax=4, emu_flags=0):
    """The whole grid restricted to candidates with sum_n >= nsum_min (orc_sweep_shell)."""
    p, pp = _f32(params)
    r = SweepResult()
    rc = lib().orc_sweep_shell(n_models, kmax, pp, len(grid), _gslots(grid), float(H), int(nsum_min), eps,
                               emu_flags, C.byref(r))
    if rc != 0:
        raise ValueError("orc_sweep_shell rejected the grid")
    return r


def search(params, queries, now, inflight, space=0, budget=2**40, eps=1e-4, n_models=8, kmax=4,
           ops_per_model=None, emu_flags=0):
    if ops_per_model is None:
        import synth
        ops_per_model = synth.OPS_PER_MODEL
    opm = np.ascontiguousarray(ops_per_model, dtype=np.int32)
    k = len(queries)
    qa = (QueryC * k)(*[QueryC(q.model_id, q.next_op, q.batch, q.seqlen, q.qos_ms, q.t_start_ms)
                        for q in queries])
    p, pp = _f32(params)
    out = Decision()
    rc = lib().orc_search(n_models, kmax, opm.ctypes.data_as(C.POINTER(C.c_int32)), pp, qa, k,
                          float(now), float(inflight), space, budget, eps, emu_flags, C.byref(out))
    if rc != 0:
        raise ValueError("orc_search rejected the queries (rc=%d)" % rc)
    return out


def search_mway(params, queries, now, inflight, ways, n_models=8, kmax=4, ops_per_model=None, emu_flags=0):
    """The paper's multi-way search over the chain (rounds of batched probes)."""
    if ops_per_model is None:
        import synth
        ops_per_model = synth.OPS_PER_MODEL
    opm = np.ascontiguousarray(ops_per_model, dtype=np.int32)
    k = len(queries)
    qa = (QueryC * k)(*[QueryC(q.model_id, q.next_op, q.batch, q.seqlen, q.qos_ms, q.t_start_ms)
                        for q in queries])
    p, pp = _f32(params)
    out = MWay()
    rc = lib().orc_search_mway(n_models, kmax, opm.ctypes.data_as(C.POINTER(C.c_int32)), pp, qa, k,
                               float(now), float(inflight), int(ways), emu_flags, C.byref(out))
    if rc != 0:
        raise ValueError("orc_search_mway rejected the queries (rc=%d)" % rc)
    return out


def key_parts(key: int):
    """(sum_n + 1, t) from a 64-bit key"""
    return key >> 40, key & ((1 << 40) - 1)
