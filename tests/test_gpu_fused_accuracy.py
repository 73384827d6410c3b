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
