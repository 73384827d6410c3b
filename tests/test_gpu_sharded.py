"""GPU parity of the cross-GPU combine (a6) and the per-decision sharded search
(SURVEY §8(e)).

This run has one GPU, so a real multi-rank NCCL communicator cannot be made
(NCCL refuses two ranks on one device).  Coverage instead:
  * every shard of a G-way partition (G = 2, 3, 4, 8) is searched on the GPU
    by abacus_search_grid without a communicator -- exactly what each rank of
    a G-GPU run computes -- and the records are merged by the product's
    abacus_combine_decisions (the combine_results function the device
    finalize kernel runs after the NCCL all-gather).  The merged decision must
    equal the unsharded GPU search bit for bit (key, y(t*), y(0), end ops,
    evaluated) and be acceptable to the fp64 oracle (reading c18);
  * scheduling decisions are sharded the same way over their GRID (a1 by the
    product on one rank, then shards) with the drop test, against
    abacus_search and oracle.search;
  * abacus_search_sharded and abacus_search_grid through a real 1-rank NCCL
    communicator (ncclAllGather + finalize kernel) against the local path
    and the oracle.
The multi-rank host logic (shards, gather, combine) is also run with gloo at
world sizes 2 and 4 in tests/test_dist_gloo.py."""
import numpy as np
import pytest

import oracle
import synth
import paper_conf_sc_cui0czlzsmylg21_b200 as ab
from gpu_util import EPS, NAMES, Ctx, accept_key

pytestmark = pytest.mark.gpu
PRECS = [ab.ABACUS_FP32, ab.ABACUS_FP16, ab.ABACUS_BF16]


@pytest.fixture(scope="module")
def ctx():
    c = Ctx(params=synth.weights(1), precision=ab.ABACUS_FP32)
    yield c
    c.close()


@pytest.fixture(scope="module")
def comm(ctx):
    cm = ab.abacus_nccl_comm_init(ctx.h, 1, 0, ab.abacus_nccl_unique_id())
    yield cm
    ab.abacus_nccl_comm_destroy(cm)


def _same(a, b):
    return (a.status, a.key, a.index, a.evaluated, list(a.end_op), a.total_ops, np.float32(a.pred_ms).tobytes(),
            np.float32(a.pred_critical_only_ms).tobytes()) == \
           (b.status, b.key, b.index, b.evaluated, list(b.end_op), b.total_ops, np.float32(b.pred_ms).tobytes(),
            np.float32(b.pred_critical_only_ms).tobytes())


def _grids(params):
    g1 = [synth.GridSlot(1, 1, 8, 0, 1, 60, 1), synth.GridSlot(5, 1, 8, 0, 1, 40, 1),
          synth.GridSlot(7, 100, 4, 64, 100, 140, 1)]
    out = [g1, synth.cfg1_grids()[2][1], [synth.GridSlot(5, 38, 2, 0, 39, 40, 1)]]
    return out


@pytest.mark.parametrize("prec", PRECS, ids=[NAMES[p] for p in PRECS])
def test_shard_records_combine_equals_unsharded(ctx, prec):
    ctx.load(ctx.params, prec)
    eps = EPS[prec]
    for slots in _grids(ctx.params):
        T = oracle.grid_size(slots)
        grid = ab.make_grid(slots)
        _, y, _, _ = oracle.sweep(ctx.params, slots, 0.0, want_y=True)
        for q in (0.05, 0.5, 0.95):
            H = float(np.float32(np.quantile(y, q)))
            whole = ab.abacus_search_grid(ctx.h, grid, H, 0, T)
            assert np.isfinite(whole.pred_critical_only_ms)
            ref, _, _, _ = oracle.sweep(ctx.params, slots, H, eps=eps)
            assert accept_key(whole.key, ref.maxkey_strict, ref.maxkey_loose)
            assert abs(whole.pred_critical_only_ms - ref.y0) <= eps * abs(ref.y0)
            for G in (2, 3, 4, 8):
                recs = []
                for r in range(G):
                    first, count = ab.shard_range(T, r, G)
                    d = ab.abacus_search_grid(ctx.h, grid, H, first, count)
                    assert (first == 0 and count > 0) == bool(np.isfinite(d.pred_critical_only_ms)), (r, G)
                    recs.append(d)
                merged = ab.abacus_combine_decisions(recs)
                assert _same(merged, whole), (NAMES[prec], T, q, G)


@pytest.mark.parametrize("prec", PRECS, ids=[NAMES[p] for p in PRECS])
def test_sharded_decisions_combine_with_drop(ctx, prec):
    """A decision's GRID split over G shards + combine(drop_test) == abacus_search."""
    ctx.load(ctx.params, prec)
    decs = synth.cfg2_decisions(12)
    # one decision whose critical query alone cannot fit (DROP)
    qs, now, infl = decs[0]
    qs = [synth.Query(q.model_id, 1, 32, q.seqlen, q.qos_ms, q.t_start_ms) for q in qs]
    qs[0].qos_ms = 1.0
    decs.append((qs, now, infl))
    seen = set()
    for qs, now, infl in decs:
        ref = ab.abacus_search(ctx.h, qs, now, infl, ab.ABACUS_SPACE_GRID)
        seen.add(ref.status)
        order = [ref.order[j] for j in range(len(qs))]
        slots = []
        for j, qi in enumerate(order):
            q = qs[qi]
            L = synth.L(q.model_id)
            slots.append(synth.GridSlot(q.model_id, q.next_op, q.batch, q.seqlen, L if j == 0 else q.next_op, L,
                                        0 if j == 0 else 1))
        T = oracle.grid_size(slots)
        for G in (2, 4, 8):
            recs = [ab.abacus_search_grid(ctx.h, ab.make_grid(slots), ref.headroom_ms, *ab.shard_range(T, r, G))
                    for r in range(G)]
            m = ab.abacus_combine_decisions(recs, drop_test=True)
            assert m.status == ref.status and m.key == ref.key and m.evaluated == ref.evaluated
            assert np.float32(m.pred_ms) == np.float32(ref.pred_ms)
            assert np.float32(m.pred_critical_only_ms) == np.float32(ref.pred_critical_only_ms)
            # end ops: grid slot j is caller query order[j]
            assert [m.end_op[j] for j in range(len(qs))] == [ref.end_op[order[j]] for j in range(len(qs))]
        od = oracle.search(ctx.params, qs, now, infl, space=0, eps=EPS[prec])
        if abs(od.pred_critical_only_ms - od.headroom_ms) > EPS[prec] * abs(od.headroom_ms):
            assert ref.status == od.status
        if od.status == ab.ABACUS_DECIDE_OK and ref.status == ab.ABACUS_DECIDE_OK:
            assert accept_key(ref.key, od.maxkey_strict, od.maxkey_loose)
    assert ab.ABACUS_DECIDE_DROP in seen and ab.ABACUS_DECIDE_OK in seen


@pytest.mark.parametrize("prec", PRECS, ids=[NAMES[p] for p in PRECS])
def test_search_sharded_nccl_one_rank(ctx, comm, prec):
    """abacus_search_sharded through a real NCCL communicator (all-gather +
    finalize kernel) returns exactly abacus_search's decision, in every space;
    the decisions are acceptable to the oracle."""
    ctx.load(ctx.params, prec)
    decs = synth.cfg2_decisions(10) + synth.cfg3_decisions(6)
    for i, (qs, now, infl) in enumerate(decs):
        for space, budget in ((ab.ABACUS_SPACE_GRID, 2**40), (ab.ABACUS_SPACE_CHAIN, 2**40),
                              (ab.ABACUS_SPACE_AUTO, 1 << 20)):
            if i >= 10 and space == ab.ABACUS_SPACE_GRID:
                budget = 2**40  # config-3 GRIDs up to 4e7 candidates: the sharded case of §8(d)
            a = ab.abacus_search(ctx.h, qs, now, infl, space, budget)
            b = ab.abacus_search_sharded(ctx.h, qs, now, infl, space, budget, comm)
            assert _same(a, b), (i, space)
            c = ab.abacus_search_sharded(ctx.h, qs, now, infl, space, budget, None)
            assert _same(a, c), (i, space)
        if i < 10:
            od = oracle.search(ctx.params, qs, now, infl, space=0, eps=EPS[prec])
            d = ab.abacus_search_sharded(ctx.h, qs, now, infl, ab.ABACUS_SPACE_GRID, 2**40, comm)
            if od.status == ab.ABACUS_DECIDE_OK and d.status == ab.ABACUS_DECIDE_OK:
                assert accept_key(d.key, od.maxkey_strict, od.maxkey_loose)


def test_search_grid_nccl_single_rank_carries_y0(ctx, comm):
    """abacus_search_grid with a 1-rank communicator: the same record as the
    local path, including y(0) (the round-1 finalize copied the winner's)."""
    slots = synth.cfg1_grids()[1][1]
    T = oracle.grid_size(slots)
    for prec in PRECS:
        ctx.load(ctx.params, prec)
        for first, count in ((0, T), (17, T - 17), (0, 1), (T - 1, 1), (5, 0)):
            a = ab.abacus_search_grid(ctx.h, ab.make_grid(slots), 12.5, first, count)
            b = ab.abacus_search_grid(ctx.h, ab.make_grid(slots), 12.5, first, count, comm)
            assert _same(a, b), (NAMES[prec], first, count)
            assert (first == 0 and count > 0) == bool(np.isfinite(b.pred_critical_only_ms))
    ctx.load(ctx.params, ab.ABACUS_FP32)


def test_search_sharded_errors(ctx, comm):
    with pytest.raises(ab.AbacusError):
        ab.abacus_search_sharded(ctx.h, [], 0.0, 0.0, ab.ABACUS_SPACE_GRID, 2**40, comm)
    qs = [synth.Query(2, 5, 8, 0, 30.0, 0.0), synth.Query(2, 7, 8, 0, 30.0, 0.0)]
    with pytest.raises(ab.AbacusError) as e:
        ab.abacus_search_sharded(ctx.h, qs, 0.0, 0.0, ab.ABACUS_SPACE_GRID, 2**40, comm)
    assert e.value.code == ab.ABACUS_E_DUP_MODEL
