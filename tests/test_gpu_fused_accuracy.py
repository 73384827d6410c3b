"""y(t*) returned by the fused search kernels against the fp64 oracle's y at the
same index, over many headroom thresholds on the config-1 grids (one sample per
search: the selected candidate).  The fp16 search kernels accumulate layer 1
in f16 from the true digits; the bars are BASELINE's (1e-4 fp32,
1e-2 for the tensor paths).  tests/fused_y_error.py is the long version
(profiles/r2_fused_y_error.json)."""
import numpy as np
import pytest

import oracle
import synth
import paper_conf_sc_cui0czlzsmylg21_b200 as ab
from gpu_util import Ctx, EPS, NAMES

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("prec", [ab.ABACUS_FP32, ab.ABACUS_FP16, ab.ABACUS_BF16])
def test_selected_y_against_oracle(prec):
    params = synth.weights(1)
    rng = np.random.default_rng(32)
    grids = []
    for _, slots in synth.cfg1_grids():
        _, y64, _, _ = oracle.sweep(params, slots, 0.0, want_y=True)
        grids.append((slots, np.asarray(y64)))
    c = Ctx(params=params, precision=prec)
    try:
        errs = []
        for i in range(300):
            slots, y64 = grids[i % len(grids)]
            H = float(np.float32(np.quantile(y64, rng.uniform(0.02, 0.98))))
            d = ab.abacus_search_grid(c.h, ab.make_grid(slots), H, 0, len(y64))
            assert d.key != 0
            assert d.pred_ms <= H
            errs.append(abs(d.pred_ms - y64[d.index]) / abs(y64[d.index]))
        e = np.array(errs)
        assert e.max() <= EPS[prec], (NAMES[prec], e.max())
        # the tensor paths sit well inside the bar (fp16 6.5e-4, bf16 2.9e-3 max over 3,000 searches)
        if prec != ab.ABACUS_FP32:
            assert e.max() <= 0.5 * EPS[prec], (NAMES[prec], e.max())
    finally:
        c.close()


@pytest.mark.parametrize("prec", [ab.ABACUS_FP32, ab.ABACUS_FP16, ab.ABACUS_BF16])
def test_headroom_boundary_is_inclusive(prec):
    """The fit test is y <= H with H inclusive (reading c11), decided in the tensor
    kernels on the raw output accumulator (y_raw <= T): a search at H = y*, the
    prediction of the group a first search selected, selects the same group, and
    a search at the next float below y* selects a smaller key (that group no
    longer fits)."""
    params = synth.weights(1)
    rng = np.random.default_rng(33)
    c = Ctx(params=params, precision=prec)
    try:
        for b, slots in synth.cfg1_grids():
            _, y64, _, _ = oracle.sweep(params, slots, 0.0, want_y=True)
            g = ab.make_grid(slots)
            T = len(y64)
            for _ in range(8):
                H1 = float(np.float32(np.quantile(y64, rng.uniform(0.05, 0.95))))
                d1 = ab.abacus_search_grid(c.h, g, H1, 0, T)
                assert d1.key != 0
                ystar = float(np.float32(d1.pred_ms))
                d2 = ab.abacus_search_grid(c.h, g, ystar, 0, T)
                assert d2.key == d1.key and d2.pred_ms == d1.pred_ms, (NAMES[prec], H1, ystar)
                below = float(np.nextafter(np.float32(ystar), np.float32(-np.inf)))
                d3 = ab.abacus_search_grid(c.h, g, below, 0, T)
                assert d3.key < d1.key, (NAMES[prec], ystar, below)
                assert d3.key == 0 or d3.pred_ms <= below
    finally:
        c.close()
