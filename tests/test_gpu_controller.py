"""NEXT-2 on the GPU: the streamed controller (paper_conf_sc_cui0czlzsmylg21_b200.controller)
driven by abacus_search, with the fp64 oracle deciding the same round beside
it.  Every round's GPU decision must be acceptable to the oracle (reading c18;
the drop decision may differ only when y(critical alone) is within the
tolerance of H), and the closed-form streams of tests/test_controller.py must
replay identically."""
import pytest

import oracle
import synth
import paper_conf_sc_cui0czlzsmylg21_b200 as ab
from paper_conf_sc_cui0czlzsmylg21_b200 import controller as ctl
from gpu_util import EPS, Ctx, accept_key
from oracle_helpers import unit0_params

pytestmark = pytest.mark.gpu


def _qos(params, services):
    """2 x the fp64 prediction of the service alone, whole, at its largest input."""
    out = {}
    for m in services:
        x = oracle.encode(synth.N_MODELS, synth.K_MAX, [(m, 1, synth.L(m), 32, synth.seqlen_for(m, 512))])
        out[m] = 2.0 * oracle.mlp64(params, x)
    return out


@pytest.mark.parametrize("prec", [ab.ABACUS_FP32, ab.ABACUS_FP16])
def test_stream_rounds_match_oracle(prec):
    params = synth.weights(1)
    c = Ctx(params=params, precision=prec)
    eps = EPS[prec]
    services = synth.cfg3_services()
    qos = _qos(params, services)
    arr = synth.cfg3_arrivals(50.0, 600.0, seed=17)
    ops = {m: synth.L(m) for m in services}
    stats = {"rounds": 0, "near": 0}

    def search(qs, now, infl):
        d = ab.abacus_search(c.h, qs, now, infl, ab.ABACUS_SPACE_AUTO, 20_000)
        od = oracle.search(c.params, qs, now, infl, space=ab.ABACUS_SPACE_AUTO, budget=20_000, eps=eps)
        stats["rounds"] += 1
        assert d.critical == od.critical and d.evaluated == od.evaluated
        near = abs(od.pred_critical_only_ms - od.headroom_ms) <= eps * abs(od.headroom_ms)
        stats["near"] += near
        if not near:
            assert d.status == od.status
        if d.status == ab.ABACUS_DECIDE_OK and od.status == ab.ABACUS_DECIDE_OK:
            assert accept_key(d.key, od.maxkey_strict, od.maxkey_loose)
        return d

    try:
        r = ctl.simulate(search, arr, qos, ops)
        assert r.completed + r.dropped == len(arr) and stats["rounds"] == r.rounds > 20
    finally:
        c.close()


def test_closed_form_streams_replay_on_gpu():
    """The linear-predictor stream of tests/test_controller.py, through the GPU search."""
    n, kmax = 2, 4
    d = n + 4 * kmax
    coef = {}
    for p in range(kmax):
        coef[n + 4 * p + 1] = 1.0
        coef[n + 4 * p] = -1.0
    params = unit0_params(d, 1.0, coef)
    ops = {1: 3, 2: 10}
    for prec in (ab.ABACUS_FP32, ab.ABACUS_FP16, ab.ABACUS_BF16):
        c = Ctx(ops=[3, 10], params=params, precision=prec)
        try:
            r = ctl.simulate(lambda qs, now, infl: ab.abacus_search(c.h, qs, now, infl, 0), [(0.0, 1, 1, 0),
                             (0.0, 2, 1, 0)], {1: 5.0, 2: 100.0}, ops, keep_log=True)
            assert r.groups == 2 and r.completed == 2 and sorted(r.latencies_ms) == [5.0, 12.0]
            assert r.log[0][3] == (3, 3) and r.log[1][3] == (10,)
        finally:
            c.close()
