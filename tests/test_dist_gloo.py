"""Multi-process (gloo, CPU, world sizes 2 and 4) coverage of the cross-GPU
combine step a6 through the PRODUCT's combine.

Each rank takes its contiguous shard [floor(rT/G), floor((r+1)T/G)) of a
grid, builds the record abacus_search_grid returns for that shard without a
communicator -- here computed by the fp64 oracle, since there is no GPU --,
all ranks exchange the records (gloo all-gather, the collective the NCCL path
runs as ncclAllGather), and every rank merges them with
libabacus.so's abacus_combine_decisions: the same combine_results function the
device finalize kernel runs after the NCCL all-gather.  The merged decision
must equal the UNSHARDED oracle's: key, y(t*), y(0) (taken from the rank
whose shard holds index 0 -- the round-1 bug took it from the winner),
evaluated count, end ops and, for scheduling decisions (drop_test), the
status including DROP (reading c14).  The per-decision sharding
of abacus_search_sharded is the decision case: a1 on every rank, the
decision's GRID sharded, combined with the drop test."""
import ctypes as C
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synth
import paper_conf_sc_cui0czlzsmylg21_b200 as ab


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _cases():
    """(name, grid, H, drop_test, order) cases: sweep grids and decision grids."""
    params = synth.weights(1)
    out = []
    g1 = [synth.GridSlot(1, 1, 8, 0, 1, 60, 1), synth.GridSlot(5, 1, 8, 0, 1, 40, 1),
          synth.GridSlot(7, 100, 4, 64, 100, 140, 1)]
    _, y, _, _ = oracle.sweep(params, g1, 0.0, want_y=True)
    for q in (0.02, 0.5, 0.97):
        out.append(("sweep_q%g" % q, g1, float(np.float32(np.quantile(y, q))), False, None))
    out.append(("sweep_none", g1, float(np.float32(y.min() * 0.5)), False, None))
    # tiny grid: T = 3 < world 4 (empty shards, index 0 on a later rank)
    out.append(("sweep_tiny", [synth.GridSlot(5, 38, 2, 0, 39, 40, 1)], 1e3, False, None))
    # scheduling decisions (config 2 queries): a1 by the oracle's order, GRID sharded
    for i, (qs, now, infl) in enumerate(synth.cfg2_decisions(6)):
        d = oracle.search(params, qs, now, infl, space=0)
        order = [d.order[j] for j in range(len(qs))]
        grid = []
        for j, qi in enumerate(order):
            qq = qs[qi]
            L = synth.L(qq.model_id)
            grid.append(synth.GridSlot(qq.model_id, qq.next_op, qq.batch, qq.seqlen,
                                       L if j == 0 else qq.next_op, L, 0 if j == 0 else 1))
        H = float(np.float32(d.headroom_ms))
        out.append(("decision%d" % i, grid, H, True, (qs, now, infl)))
        if i == 0:  # the same decision with the headroom cut below y(critical alone): DROP
            out.append(("decision_drop", grid, float(np.float32(d.pred_critical_only_ms * 0.9)), True, None))
    return out


def _shard_record(params, grid, H, first, count):
    """The per-rank record abacus_search_grid returns for shard [first, first+count)
    (nccl_comm NULL), computed by the fp64 oracle."""
    r, _, _, _ = oracle.sweep(params, grid, H, first=first, count=count)
    d = ab.abacus_decision_t()
    d.status = ab.ABACUS_DECIDE_OK if r.best_key else ab.ABACUS_DECIDE_NONE
    d.critical = 0
    for j in range(4):
        d.order[j] = j if j < len(grid) else -1
    d.key = r.best_key
    d.index = r.best_index if r.best_key else 0
    d.evaluated = r.evaluated
    d.headroom_ms = H
    d.pred_ms = float(r.best_y) if r.best_key else float("nan")
    d.pred_critical_only_ms = float(r.y0)  # NaN unless index 0 is in this shard
    if r.best_key:
        _, _, _, ope = oracle.sweep(params, grid, H, first=r.best_index, count=1, want_ope=True)
        for j in range(len(grid)):
            d.end_op[j] = int(ope[0, j])
        d.total_ops = (r.best_key >> 40) - 1
    return bytes(d)


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        params = synth.weights(1)
        res = []
        for name, grid, H, drop, _ in _cases():
            T = oracle.grid_size(grid)
            first, count = ab.shard_range(T, rank, world)
            mine = _shard_record(params, grid, H, first, count)
            gathered = [None] * world
            dist.all_gather_object(gathered, mine)
            recs = [ab.abacus_decision_t.from_buffer_copy(b) for b in gathered]
            d = ab.abacus_combine_decisions(recs, drop_test=drop)
            res.append((name, bytes(d), first, count))
        q.put((rank, res))
    finally:
        dist.destroy_process_group()


def _run(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = dict(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    return out


def _f32(v):
    return float(np.float32(v))


@pytest.mark.parametrize("world", [2, 4])
def test_sharded_combine_gloo(world):
    out = _run(world)
    params = synth.weights(1)
    cases = {c[0]: c for c in _cases()}
    names = [r[0] for r in out[0]]
    for ci, name in enumerate(names):
        _, grid, H, drop, dec = cases[name]
        T = oracle.grid_size(grid)
        # shards partition [0, T) contiguously, in rank order
        parts = [(out[r][ci][2], out[r][ci][3]) for r in range(world)]
        assert parts[0][0] == 0 and sum(c for _, c in parts) == T
        assert all(parts[i][0] + parts[i][1] == parts[i + 1][0] for i in range(world - 1))
        ds = [ab.abacus_decision_t.from_buffer_copy(out[r][ci][1]) for r in range(world)]
        for d in ds[1:]:  # every rank returns the same decision
            assert bytes(d) == bytes(ds[0]), name
        d = ds[0]
        full, _, _, _ = oracle.sweep(params, grid, H)  # the unsharded oracle
        assert d.evaluated == T, name
        assert d.key == full.best_key, (name, d.key, full.best_key)
        assert _f32(d.pred_critical_only_ms) == _f32(full.y0), (name, d.pred_critical_only_ms, full.y0)
        dropped = drop and not (full.y0 <= H)
        if dropped:
            assert d.status == ab.ABACUS_DECIDE_DROP and d.total_ops == 0 and list(d.end_op) == [0] * 4, name
            assert _f32(d.pred_ms) == _f32(full.y0), name
        elif full.best_key:
            assert d.status == ab.ABACUS_DECIDE_OK, name
            assert _f32(d.pred_ms) == _f32(full.best_y), name
            assert d.index == full.best_index and d.total_ops == (full.best_key >> 40) - 1, name
            _, _, _, ope = oracle.sweep(params, grid, H, first=full.best_index, count=1, want_ope=True)
            assert list(d.end_op)[:len(grid)] == [int(v) for v in ope[0]], name
        else:
            assert d.status == ab.ABACUS_DECIDE_NONE and d.key == 0, name
        if dec is not None:  # the decision equals the unsharded oracle decision (abacus_search semantics)
            qs, now, infl = dec
            od = oracle.search(params, qs, now, infl, space=0)
            assert d.status == od.status, name
            if od.status == ab.ABACUS_DECIDE_OK:
                assert d.key == od.key and _f32(d.pred_ms) == _f32(od.pred_ms), name
    statuses = {ab.abacus_decision_t.from_buffer_copy(out[0][i][1]).status for i in range(len(names))}
    assert statuses == {ab.ABACUS_DECIDE_OK, ab.ABACUS_DECIDE_DROP, ab.ABACUS_DECIDE_NONE}, statuses


def test_combine_rejects_inconsistent_records():
    a = ab.abacus_decision_t()
    a.headroom_ms = 1.0
    b = ab.abacus_decision_t()
    b.headroom_ms = 2.0
    with pytest.raises(ab.AbacusError):
        ab.abacus_combine_decisions([a, b])
    b.headroom_ms = 1.0
    b.key = 5  # key without status OK
    b.status = ab.ABACUS_DECIDE_NONE
    with pytest.raises(ab.AbacusError):
        ab.abacus_combine_decisions([a, b])
    with pytest.raises(ab.AbacusError):
        ab.abacus_combine_decisions([])


def test_combine_y0_from_index0_rank_not_winner():
    """Rank 0 holds index 0 (y0 = 3.5) but rank 1 wins: y0 must be rank 0's."""
    a = ab.abacus_decision_t()
    a.status, a.key, a.pred_ms, a.pred_critical_only_ms, a.evaluated = 0, (5 << 40) | 3, 7.0, 3.5, 10
    a.headroom_ms = 9.0
    b = ab.abacus_decision_t()
    b.status, b.key, b.pred_ms, b.pred_critical_only_ms, b.evaluated = 0, (9 << 40) | 12, 8.5, float("nan"), 11
    b.headroom_ms = 9.0
    b.end_op[0] = 4
    d = ab.abacus_combine_decisions([a, b])
    assert d.key == b.key and d.pred_ms == 8.5 and d.pred_critical_only_ms == 3.5 and d.evaluated == 21
    assert d.index == 12 and d.end_op[0] == 4 and d.status == ab.ABACUS_DECIDE_OK
    d = ab.abacus_combine_decisions([b, a])  # index 0 on the later rank
    assert d.pred_critical_only_ms == 3.5
    a.pred_critical_only_ms = 9.5  # above H: a decision drops
    d = ab.abacus_combine_decisions([a, b], drop_test=True)
    assert d.status == ab.ABACUS_DECIDE_DROP and d.pred_ms == 9.5 and d.total_ops == 0


def test_shard_range_partitions():
    for T in (1, 7, 5043, 9_188_218_208):
        for G in (1, 2, 3, 4, 8):
            parts = [ab.shard_range(T, r, G) for r in range(G)]
            assert parts[0][0] == 0 and sum(c for _, c in parts) == T
            assert all(parts[i][0] + parts[i][1] == parts[i + 1][0] for i in range(G - 1))
            assert max(c for _, c in parts) - min(c for _, c in parts) <= 1
