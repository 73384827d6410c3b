"""NEXT-2: the streamed, pipelined controller (host logic), driven by the fp64
oracle's search, pinned by closed forms of hand-built predictors:

* constant predictor y = c (all weights 0, b4 = c): every feasible round takes
  every active query whole; a query's latency is its wait + c;
* linear predictor y = 1 + sum over present queries of (n_i - 1) (hidden unit
  0 of tests/oracle_helpers.unit0_params): the critical query is taken whole
   and the next query gets the largest op prefix that fits.

Eq. 2 / Eq. 3, the drop rule and the
Fig. 13 pipelining each change one number below.
"""
import numpy as np
import pytest

import oracle
from oracle_helpers import offsets, unit0_params, zero_params
from paper_conf_sc_cui0czlzsmylg21_b200 import controller as ctl

N, KMAX = 2, 4
D = N + 4 * KMAX
OPS = {1: 3, 2: 10}


def _search(params, ops=OPS):
    opm = [ops[m] for m in sorted(ops)]
    return lambda qs, now, infl: oracle.search(params, qs, now, infl, space=0, n_models=len(opm), kmax=KMAX,
                                               ops_per_model=opm)


def _const(c):
    p = zero_params(D)
    p[offsets(D)["b4"]] = c
    return p


def _linear():
    # y = 1 + sum_p (ope_p - ops_p): Fig.-8 slot p holds (ops, ope, bs, seqlen) at N + 4p
    coef = {}
    for p in range(KMAX):
        coef[N + 4 * p + 1] = 1.0
        coef[N + 4 * p] = -1.0
    return unit0_params(D, 1.0, coef)


def test_sparse_arrivals_take_exactly_the_prediction():
    arr = [(0.0, 1, 1, 0), (10.0, 2, 1, 0), (20.0, 1, 1, 0)]
    r = ctl.simulate(_search(_const(4.0)), arr, {1: 100.0, 2: 100.0}, OPS)
    assert (r.completed, r.dropped, r.violations, r.groups) == (3, 0, 0, 3)
    assert r.latencies_ms == [4.0, 4.0, 4.0]


def test_simultaneous_arrivals_share_one_group():
    arr = [(0.0, 1, 1, 0), (0.0, 2, 1, 0)]
    r = ctl.simulate(_search(_const(4.0)), arr, {1: 100.0, 2: 100.0}, OPS, keep_log=True)
    assert r.groups == 1 and r.latencies_ms == [4.0, 4.0]
    assert r.log[0][3] == (3, 10)   # both whole: end op = L


@pytest.mark.parametrize("qos_b, completed, dropped, lat_b", [(7.0, 2, 0, 7.0), (6.5, 1, 1, None)])
def test_arrival_during_a_running_group_sees_the_inflight_prediction(qos_b, completed, dropped, lat_b):
    """A runs [0, 4).  B arrives at 1: Eq. 3 subtracts the 3 ms still in flight,
    so B's headroom is qos_b - 0 - 3; c = 4 fits iff qos_b >= 7 (inclusive, c11).
    It then starts when the executor frees up (4) and ends at 8: latency 7."""
    arr = [(0.0, 1, 1, 0), (1.0, 2, 1, 0)]
    r = ctl.simulate(_search(_const(4.0)), arr, {1: 100.0, 2: qos_b}, OPS, keep_log=True)
    assert (r.completed, r.dropped) == (completed, dropped)
    if lat_b is not None:
        assert r.latencies_ms == [4.0, lat_b] and r.violations == 0
    else:
        assert r.violations == 1


def test_qos_below_the_prediction_drops_every_query():
    arr = [(0.0, 1, 1, 0), (0.0, 2, 1, 0), (5.0, 1, 1, 0)]
    r = ctl.simulate(_search(_const(4.0)), arr, {1: 3.0, 2: 3.0}, OPS)
    assert (r.completed, r.dropped, r.violations, r.groups) == (0, 3, 3, 0)


def test_partial_group_then_pipelined_remainder():
    """Round 1 (t = 0): A (headroom 5) is critical and whole (2 more ops than
    one: +2), B (headroom 100) gets the largest prefix with 1 + 2 + (n_B - 1)
    <= 5, i.e. ops 1..3; y = 5.  Round 2 is searched at the START of group 1
    (Fig. 13) with its 5 ms in flight: B alone, whole (7 ops, y = 7), issued
    at 5, done at 12."""
    arr = [(0.0, 1, 1, 0), (0.0, 2, 1, 0)]
    r = ctl.simulate(_search(_linear()), arr, {1: 5.0, 2: 100.0}, OPS, keep_log=True)
    assert r.groups == 2 and r.completed == 2 and r.violations == 0
    assert r.log[0][2] == ((1, 1), (2, 1)) and r.log[0][3] == (3, 3) and r.log[0][4] == 5.0
    assert r.log[1][0] == 0.0 and r.log[1][2] == ((2, 4),) and r.log[1][3] == (10,) and r.log[1][4] == 7.0
    assert sorted(r.latencies_ms) == [5.0, 12.0]


def test_conservation_on_a_random_stream():
    rng = np.random.default_rng(3)
    arr = sorted((float(t), int(m), 1, 0) for t, m in zip(np.cumsum(rng.exponential(2.0, 60)),
                                                          rng.integers(1, 3, 60)))
    r = ctl.simulate(_search(_linear()), arr, {1: 9.0, 2: 14.0}, OPS)
    assert r.completed + r.dropped == len(arr)
    assert all(lat >= 1.0 for lat in r.latencies_ms)
    assert r.violations >= r.dropped
