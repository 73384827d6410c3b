"""NEXT-4: many independent scheduling rounds in one
abacus_search_batch call.  Decision i of a batch must be exactly the
single-round abacus_search of the same inputs (the same per-row arithmetic on
the tensor cores, so bit-identical), and within the oracle's acceptance window
(reading c18) like every other search."""
import numpy as np
import pytest

import oracle
import synth
import paper_conf_sc_cui0czlzsmylg21_b200 as ab
from gpu_util import EPS, Ctx, accept_key
from oracle_helpers import load_fig12, unit0_params

pytestmark = pytest.mark.gpu
TC = [ab.ABACUS_FP16, ab.ABACUS_BF16]
SPACES = [ab.ABACUS_SPACE_GRID, ab.ABACUS_SPACE_CHAIN, ab.ABACUS_SPACE_AUTO]


def _same(a, b):
    fields = ["status", "critical", "key", "index", "evaluated", "total_ops"]
    for f in fields:
        assert getattr(a, f) == getattr(b, f), f
    assert list(a.order) == list(b.order) and list(a.end_op) == list(b.end_op)
    for f in ["headroom_ms", "pred_ms", "pred_critical_only_ms"]:
        x, y = getattr(a, f), getattr(b, f)
        assert (np.isnan(x) and np.isnan(y)) or x == y, f


def _mixed(n, seed=5):
    """cfg2 (3-way) and cfg3 (4-way) rounds, plus k = 1 and k = 2 rounds cut from them."""
    rng = np.random.default_rng(seed)
    d2 = synth.cfg2_decisions(n)
    d3 = synth.cfg3_decisions(n, seed=31)
    out = []
    for i in range(n):
        qs, now, infl = (d2 if i % 2 else d3)[i]
        kk = int(rng.integers(1, len(qs) + 1))
        out.append((qs[:kk], now, infl))
    return out


@pytest.mark.parametrize("prec", TC)
@pytest.mark.parametrize("space", SPACES)
def test_batch_equals_single_rounds(prec, space):
    c = Ctx(params=synth.weights(1), precision=prec)
    try:
        decs = _mixed(96)
        got = ab.abacus_search_batch(c.h, decs, space, 200_000)
        for (qs, now, infl), g in zip(decs, got):
            _same(g, ab.abacus_search(c.h, qs, now, infl, space, 200_000))
    finally:
        c.close()


@pytest.mark.parametrize("prec", TC)
@pytest.mark.parametrize("space", [ab.ABACUS_SPACE_GRID, ab.ABACUS_SPACE_CHAIN])
def test_batch_cfg2_vs_oracle(prec, space):
    c = Ctx(params=synth.weights(1), precision=prec)
    eps = EPS[prec]
    try:
        decs = synth.cfg2_decisions(40)
        got = ab.abacus_search_batch(c.h, decs, space)
        for (qs, now, infl), d in zip(decs, got):
            od = oracle.search(c.params, qs, now, infl, space=space, budget=2**40, eps=eps)
            assert d.critical == od.critical and list(d.order)[:3] == list(od.order)[:3]
            assert d.headroom_ms == np.float32(od.headroom_ms)
            assert d.evaluated == od.evaluated
            assert abs(d.pred_critical_only_ms - od.pred_critical_only_ms) <= eps * abs(od.pred_critical_only_ms)
            if abs(od.pred_critical_only_ms - od.headroom_ms) > eps * abs(od.headroom_ms):
                assert d.status == od.status
            if d.status == ab.ABACUS_DECIDE_OK and od.status == ab.ABACUS_DECIDE_OK:
                assert accept_key(d.key, od.maxkey_strict, od.maxkey_loose)
                assert d.total_ops == (d.key >> 40) - 1
    finally:
        c.close()


@pytest.mark.parametrize("prec", TC)
def test_batch_fig12_among_other_rounds(prec):
    """The Fig. 12 replay at several positions of a batch."""
    f = load_fig12()
    d_feat = f["n_models"] + 16
    p = unit0_params(d_feat, f["unit0"]["bias"], {int(k): v for k, v in f["unit0"]["coef"].items()})
    c = Ctx(ops=f["ops_per_model"], params=p, precision=prec)
    try:
        fig = [synth.Query(q["model_id"], q["next_op"], 1, 0, q["headroom_ms"], 0.0) for q in f["queries"]]
        other = [synth.Query(1, 2, 1, 0, 40.0, 0.0), synth.Query(3, 1, 1, 0, 30.0, 0.0)]
        decs = [(fig, 0.0, 0.0) if i % 3 == 0 else (other[: 1 + i % 2], 0.0, 0.0) for i in range(10)]
        names = [q["name"] for q in f["queries"]]
        for space in (ab.ABACUS_SPACE_GRID, ab.ABACUS_SPACE_CHAIN):
            got = ab.abacus_search_batch(c.h, decs, space)
            for i, d in enumerate(got):
                if i % 3:
                    continue
                assert d.status == ab.ABACUS_DECIDE_OK
                assert names[d.critical] == f["expected"]["critical"]
                assert {names[j]: d.end_op[j] for j in range(3)} == f["expected"]["end_op"]
                assert d.pred_ms == f["expected"]["pred_ms"]
                assert d.index == (f["expected"]["grid_t"] if space == 0 else f["expected"]["chain_u"])
    finally:
        c.close()


def test_batch_large_and_regrow():
    """Batches of growing size (buffers regrow), one decision repeated: every copy identical."""
    c = Ctx(params=synth.weights(1), precision=ab.ABACUS_FP16)
    try:
        qs, now, infl = synth.cfg3_decisions(1, seed=7)[0]
        ref = ab.abacus_search(c.h, qs, now, infl, ab.ABACUS_SPACE_AUTO, 1_000_000)
        for n in (1, 300, 2000):
            got = ab.abacus_search_batch(c.h, [(qs, now, infl)] * n, ab.ABACUS_SPACE_AUTO, 1_000_000)
            for g in got:
                _same(g, ref)
    finally:
        c.close()


def test_batch_fp32_is_per_round():
    c = Ctx(params=synth.weights(1), precision=ab.ABACUS_FP32)
    try:
        decs = synth.cfg2_decisions(12)
        got = ab.abacus_search_batch(c.h, decs, ab.ABACUS_SPACE_GRID)
        for (qs, now, infl), g in zip(decs, got):
            _same(g, ab.abacus_search(c.h, qs, now, infl, ab.ABACUS_SPACE_GRID))
    finally:
        c.close()


@pytest.mark.parametrize("prec", [ab.ABACUS_FP16, ab.ABACUS_BF16, ab.ABACUS_FP32], ids=["fp16", "bf16", "fp32"])
def test_batch_errors_name_the_decision(prec):
    c = Ctx(params=synth.weights(1), precision=prec)
    try:
        decs = synth.cfg2_decisions(5)
        bad = list(decs)
        qs = list(bad[3][0])
        qs[1] = synth.Query(qs[0].model_id, 1, 4, 0, 50.0, 0.0)  # duplicate model
        bad[3] = (qs, bad[3][1], bad[3][2])
        with pytest.raises(ab.AbacusError) as e:
            ab.abacus_search_batch(c.h, bad)
        assert e.value.code == ab.ABACUS_E_DUP_MODEL and "decision 3" in str(e.value)
        with pytest.raises(ab.AbacusError):
            ab.abacus_search_batch(c.h, [])
        # still usable after an error
        assert len(ab.abacus_search_batch(c.h, decs)) == 5
    finally:
        c.close()


def _bad_variants(qs):
    """One invalid version of a round per validation rule of a1 (the device
    planner of a batch checks what abacus_search checks on the host)."""
    m0 = qs[0]
    L0 = synth.L(m0.model_id)
    rep = lambda q, **kw: synth.Query(**{**q.__dict__, **kw})  # noqa: E731
    return [
        ("model_id", [rep(m0, model_id=99)] + list(qs[1:]), ab.ABACUS_E_INVALID),
        ("next_op", [rep(m0, next_op=L0 + 1)] + list(qs[1:]), ab.ABACUS_E_INVALID),
        ("next_op", [rep(m0, next_op=0)] + list(qs[1:]), ab.ABACUS_E_INVALID),
        ("batch", [rep(m0, batch=0)] + list(qs[1:]), ab.ABACUS_E_INVALID),
        ("seqlen", [rep(m0, seqlen=-1)] + list(qs[1:]), ab.ABACUS_E_INVALID),
        ("qos", [rep(m0, qos_ms=float("nan"))] + list(qs[1:]), ab.ABACUS_E_INVALID),
        ("dup", list(qs) + [rep(qs[-1], next_op=1)], ab.ABACUS_E_DUP_MODEL),
    ]


@pytest.mark.parametrize("prec", TC)
def test_batch_validation_matches_single_rounds(prec):
    """Every validation rule, at several positions in a batch: the batch fails
    with the single-round error code, names the first failing decision, and
    leaves the context usable; non-finite now / in-flight times too."""
    c = Ctx(params=synth.weights(1), precision=prec)
    try:
        decs = synth.cfg2_decisions(12)
        for name, bad_qs, code in _bad_variants(decs[0][0]):
            with pytest.raises(ab.AbacusError) as single:
                ab.abacus_search(c.h, bad_qs, decs[0][1], decs[0][2])
            assert single.value.code == code, name
            for pos in (0, 5, 11):
                batch = list(decs)
                batch[pos] = (bad_qs, batch[pos][1], batch[pos][2])
                if pos != 11:  # a second bad round later in the batch: the first one is named
                    batch[11] = (bad_qs, batch[11][1], batch[11][2])
                with pytest.raises(ab.AbacusError) as e:
                    ab.abacus_search_batch(c.h, batch)
                assert e.value.code == code, (name, pos)
                assert ("decision %d:" % pos) in str(e.value), (name, pos, str(e.value))
        for now, infl in ((float("inf"), 0.0), (0.0, float("nan"))):
            batch = list(decs)
            batch[3] = (batch[3][0], now, infl)
            with pytest.raises(ab.AbacusError) as e:
                ab.abacus_search_batch(c.h, batch)
            assert e.value.code == ab.ABACUS_E_INVALID and "decision 3:" in str(e.value)
        got = ab.abacus_search_batch(c.h, decs)
        for (qs, now, infl), d in zip(decs, got):
            _same(d, ab.abacus_search(c.h, qs, now, infl))
    finally:
        c.close()


def test_batch_layout_follows_single_round_bf16():
    """A long critical query (whose slot is fixed) must not push a batch into the
    split layer-1 layout when every single round of it runs unsplit: the batch
    stays bit-identical.  (Both formats split above 1,025 end-op options since
    the bf16 path took the fp16 digit operand; BERT-large from op 1 is the
    registry's longest query.)"""
    c = Ctx(params=synth.weights(1), precision=ab.ABACUS_BF16)
    try:
        decs = []
        for i in range(16):
            # BERT-large (471 ops) from op 1 is critical (tiny headroom); the others
            # have < 257 ops left, so no digit of the round exceeds 257 options
            qs = [synth.Query(8, 1, 4, 128, 5.0 + 0.01 * i, 0.0),
                  synth.Query(2, 241 - 100, 8, 0, 80.0, 0.0),
                  synth.Query(4, 220 - 150, 8, 0, 90.0, 0.0)]
            decs.append((qs, 0.0, 0.0))
        got = ab.abacus_search_batch(c.h, decs)
        for (qs, now, infl), d in zip(decs, got):
            _same(d, ab.abacus_search(c.h, qs, now, infl))
    finally:
        c.close()


@pytest.mark.parametrize("prec", [ab.ABACUS_FP16, ab.ABACUS_BF16], ids=["fp16", "bf16"])
def test_batch_mixed_layer1_layouts(prec):
    """one batch launch runs ONE layer-1 layout, so a round with a
    digit range above 1,025 (a long-model registry) puts the whole batch in the
    split layout.  The wide rounds are then bit-identical to their single
    search (same layout); the narrow ones run the split layout where their
    single search would not, and must still be within the oracle's acceptance
    window (reading c18) -- the ABI promises exactly this."""
    ops = list(synth.OPS_PER_MODEL)
    ops[0] = 3000  # model 1 with 3,000 ops
    params = synth.weights(1)
    c = Ctx(ops=ops, params=params, precision=prec)
    try:
        rng = np.random.default_rng(51)
        decs, wide = [], []
        for i in range(24):
            w = i % 4 == 0
            crit = synth.Query(4, int(rng.integers(1, 200)), 8, 0, 20.0 + rng.uniform(0, 5), 0.0)
            other = synth.Query(1, 1 if w else 2900, 4, 0, 60.0 + rng.uniform(0, 20), 0.0)
            third = synth.Query(7, int(rng.integers(1, 240)), 4, 64, 70.0, 0.0)
            decs.append(([crit, other, third], 0.0, 0.0))
            wide.append(w)
        got = ab.abacus_search_batch(c.h, decs)
        for (qs, now, infl), d, w in zip(decs, got, wide):
            single = ab.abacus_search(c.h, qs, now, infl)
            if w:
                _same(d, single)
            od = oracle.search(params, qs, now, infl, space=0, eps=EPS[prec], ops_per_model=ops)
            if od.status == ab.ABACUS_DECIDE_OK and d.status == ab.ABACUS_DECIDE_OK:
                assert accept_key(d.key, od.maxkey_strict, od.maxkey_loose)
            elif abs(od.pred_critical_only_ms - od.headroom_ms) > EPS[prec] * abs(od.headroom_ms):
                assert d.status == od.status
    finally:
        c.close()
