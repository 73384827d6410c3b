"""GPU parity on the degenerate and boundary cases of the hot path: a single
query (k = 1: GRID and CHAIN are the one candidate t = 0, P:1187-1189 with
reading c14's drop rule), empty ranges (count = 0) of every call, a one-candidate
grid, radix-1 digits in the middle of a grid, and digit ranges above the fp16
tile walker's exact range (v > 1024: the split layer-1 operand) on a registry
with long models. The oracle is the fp64 reference throughout (reading c18
for near-threshold selections).
"""
import numpy as np
import pytest
import torch

import oracle
import synth
import paper_conf_sc_cui0czlzsmylg21_b200 as ab
from gpu_util import EPS, Ctx, accept_key, stream
from test_gpu_parity import _check_sweep

pytestmark = pytest.mark.gpu
PRECS = [ab.ABACUS_FP32, ab.ABACUS_FP16, ab.ABACUS_BF16]


@pytest.mark.parametrize("prec", PRECS)
@pytest.mark.parametrize("space", [ab.ABACUS_SPACE_GRID, ab.ABACUS_SPACE_CHAIN, ab.ABACUS_SPACE_AUTO])
def test_single_query_decisions(prec, space):
    """k = 1: the only candidate is the critical query run to its end (index 0).
    It is issued iff its prediction fits the headroom, else dropped (c14)."""
    c = Ctx(params=synth.weights(1), precision=prec)
    eps = EPS[prec]
    rng = np.random.default_rng(31)
    try:
        for it in range(40):
            m = int(rng.integers(1, 9))
            s = int(rng.integers(1, synth.L(m) + 1))
            q = synth.Query(m, s, int(rng.choice([1, 4, 16, 32])), synth.seqlen_for(m, int(rng.integers(8, 513))),
                            0.0, 0.0)
            # the prediction of the lone candidate, then a headroom on either side of it
            probe = oracle.search(c.params, [synth.Query(m, s, q.batch, q.seqlen, 1e9, 0.0)], 0.0, 0.0,
                                  space=space, eps=eps)
            y = probe.pred_critical_only_ms
            for H in (y * 1.5 + 1.0, y * 0.5):
                qq = synth.Query(m, s, q.batch, q.seqlen, H, 0.0)
                d = ab.abacus_search(c.h, [qq], 0.0, 0.0, space, 1 << 20)
                od = oracle.search(c.params, [qq], 0.0, 0.0, space=space, budget=1 << 20, eps=eps)
                assert d.evaluated == od.evaluated == 1
                assert d.critical == 0 and d.order[0] == 0
                assert d.status == od.status
                assert abs(d.pred_critical_only_ms - y) <= eps * abs(y) + 1e-6
                if d.status == ab.ABACUS_DECIDE_OK:
                    assert d.index == 0 and d.end_op[0] == synth.L(m)
                    assert d.total_ops == synth.L(m) - s + 1
                    assert accept_key(d.key, od.maxkey_strict, od.maxkey_loose)
                else:
                    assert d.status == ab.ABACUS_DECIDE_DROP
    finally:
        c.close()


@pytest.mark.parametrize("prec", PRECS)
def test_search_grid_empty_ranges(prec):
    """count = 0 anywhere in [0, T]: nothing evaluated, nothing selected."""
    c = Ctx(params=synth.weights(1), precision=prec)
    try:
        slots = synth.cfg1_grids()[1][1]
        T = oracle.grid_size(slots)
        for first in (0, 1, T // 2, T - 1, T):
            d = ab.abacus_search_grid(c.h, ab.make_grid(slots), 1e9, first, 0)
            assert d.evaluated == 0 and d.key == 0
            assert d.status == ab.ABACUS_DECIDE_NONE
        # and the context is still usable afterwards
        _check_sweep(c, slots, 1e9, 0, 10)
    finally:
        c.close()


def test_zero_count_calls_are_noops():
    """encode / predict / select with count = 0 leave their outputs untouched
    and launch nothing; NULL buffers are accepted for an empty call."""
    c = Ctx(params=synth.weights(1), precision=ab.ABACUS_FP16)
    try:
        slots = synth.cfg1_grids()[0][1]
        g = ab.make_grid(slots)
        x = torch.full((4, c.D), -7, dtype=torch.int16, device="cuda")
        y = torch.full((4,), 3.5, dtype=torch.float32, device="cuda")
        best = torch.full((1,), 12345, dtype=torch.int64, device="cuda")
        n0 = ab.abacus_kernel_launches(c.h)
        ab.abacus_encode_candidates(c.h, g, 0, 0, x, stream())
        ab.abacus_predict_batch(c.h, x, 0, y, stream())
        ab.abacus_select_group(c.h, g, 0, 0, y, 10.0, best, stream())
        ab.abacus_encode_candidates(c.h, g, 0, 0, None, stream())
        ab.abacus_predict_batch(c.h, None, 0, None, stream())
        torch.cuda.synchronize()
        assert ab.abacus_kernel_launches(c.h) == n0
        assert bool((x == -7).all()) and bool((y == 3.5).all()) and int(best[0]) == 12345
    finally:
        c.close()


@pytest.mark.parametrize("prec", PRECS)
def test_one_candidate_and_radix_one_grids(prec):
    """T = 1 (one slot, one end op, no absent option), and grids whose middle
    slots have radix 1 (a fixed end op): the enumeration skips those digits."""
    c = Ctx(params=synth.weights(1), precision=prec)
    rng = np.random.default_rng(37)
    try:
        one = [synth.GridSlot(3, 10, 8, 0, 200, 200, 0)]
        assert oracle.grid_size(one) == 1
        _, y64, _, _ = oracle.sweep(c.params, one, 0.0, want_y=True)
        for H in (float(np.float32(y64[0] + 1.0)), float(np.float32(y64[0] - 1.0))):
            d = _check_sweep(c, one, H)
            assert d.evaluated == 1
        for it in range(6):
            models = [int(m) for m in rng.choice(np.arange(1, 9), size=4, replace=False)]
            slots = []
            for j, m in enumerate(models):
                Lm = synth.L(m)
                lo = int(rng.integers(1, Lm + 1))
                if j in (1, 2):        # radix 1: one fixed end op, never absent
                    hi, absent = lo, 0
                else:
                    hi, absent = int(min(Lm, lo + rng.integers(20, 200))), int(rng.integers(0, 2))
                slots.append(synth.GridSlot(m, int(rng.integers(1, lo + 1)), int(rng.choice([1, 8, 32])),
                                            synth.seqlen_for(m, 64), lo, hi, absent))
            _, y64, _, _ = oracle.sweep(c.params, slots, 0.0, want_y=True)
            H = float(np.float32(np.quantile(y64, rng.uniform(0.1, 0.9))))
            _check_sweep(c, slots, H)
    finally:
        c.close()


@pytest.mark.parametrize("prec", PRECS)
def test_long_models_split_digits(prec):
    """A registry with 1,500- and 3,000-op models: a slot with more than 1,025
    end-op options has digits above 1,024, which take the tensor kernels' split
    layer-1 operand (256 hi + lo) in fp16 as well as in bf16. Full sweeps and
    shards against the oracle."""
    ops = list(synth.OPS_PER_MODEL)
    ops[0], ops[3] = 3000, 1500
    c = Ctx(ops=ops, params=synth.weights(1), precision=prec)
    rng = np.random.default_rng(43)
    try:
        for it in range(3):
            # the digit of a slot counts its end-op options, so ranges of more than
            # 1,025 values (not large op indices) are what needs the split operand
            s = int(rng.integers(1, 60))
            lo = int(rng.integers(s, 1800))
            slots = [synth.GridSlot(4, 1, 8, 0, int(rng.integers(1400, 1490)), 1500, 1),
                     synth.GridSlot(1, s, 4, 0, lo, lo + int(rng.integers(1030, 1200)), int(rng.integers(0, 2)))]
            T = oracle.grid_size(slots)
            _, y64, _, _ = oracle.sweep(c.params, slots, 0.0, want_y=True)
            H = float(np.float32(np.quantile(y64, rng.uniform(0.1, 0.9))))
            full = _check_sweep(c, slots, H)
            keys = [_check_sweep(c, slots, H, *ab.shard_range(T, r, 3)).key for r in range(3)]
            assert max(keys) == full.key
    finally:
        c.close()


@pytest.mark.parametrize("prec", PRECS)
def test_digit_range_boundary_1025(prec):
    """The largest unsplit digit range: a slot with exactly 1,025 end-op options
    (digits 0..1024, the fp16 operand 1024 + v reaches 2048; the fp16 search
    kernels convert it to the true digit v = 1024 exactly) and one with 1,024,
    each beside a short slot, full sweeps and shards against the oracle; the
    1,026-option range (split operand) beside it."""
    ops = list(synth.OPS_PER_MODEL)
    ops[0] = 1500
    c = Ctx(ops=ops, params=synth.weights(1), precision=prec)
    rng = np.random.default_rng(44)
    try:
        for n_opts in (1024, 1025, 1026):
            lo = int(rng.integers(2, 400))
            slots = [synth.GridSlot(1, 1, 8, 0, lo, lo + n_opts - 1, 0),
                     synth.GridSlot(5, 1, 4, 0, 1, int(rng.integers(20, 40)), 1)]
            T = oracle.grid_size(slots)
            _, y64, _, _ = oracle.sweep(c.params, slots, 0.0, want_y=True)
            for q in (0.2, 0.8):
                H = float(np.float32(np.quantile(y64, q)))
                full = _check_sweep(c, slots, H)
                keys = [_check_sweep(c, slots, H, *ab.shard_range(T, r, 2)).key for r in range(2)]
                assert max(keys) == full.key
    finally:
        c.close()
