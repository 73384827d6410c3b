"""Per-candidate accuracy of the fused search kernels (the search returns y(t*)
of the candidate it selects): on config-1 grids (and config-4 windows) with many
headroom thresholds H (quantiles of each grid's fp64 predictions), compare the
kernel's y(t*) with the fp64 oracle's y at the same index.  Samples are the
selected candidates (one per search); every precision.

  python tests/fused_y_error.py [--searches 2000] [--out f.json]
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import synth  # noqa: E402
import paper_conf_sc_cui0czlzsmylg21_b200 as ab  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--searches", type=int, default=2000)
ap.add_argument("--out", default=None)
a = ap.parse_args()
params = synth.weights(1)
rng = np.random.default_rng(31)
grids = []
for b, slots in synth.cfg1_grids():
    _, y64, _, _ = oracle.sweep(params, slots, 0.0, want_y=True)
    grids.append((slots, np.asarray(y64), 0, None))
ctx = ab.abacus_create(0, list(synth.OPS_PER_MODEL))
st = torch.cuda.Stream()
torch.cuda.set_stream(st)
ab.abacus_set_stream(ctx, st)
out = {"samples_per_precision": a.searches, "grids": "config 1 (5 grids, 25,215 candidates), H = uniform quantiles"}
for name, prec in (("fp32", ab.ABACUS_FP32), ("fp16", ab.ABACUS_FP16), ("bf16", ab.ABACUS_BF16)):
    ab.abacus_load_predictor(ctx, params, prec)
    errs = []
    for i in range(a.searches):
        slots, y64, _, _ = grids[i % len(grids)]
        H = float(np.float32(np.quantile(y64, rng.uniform(0.02, 0.98))))
        g = ab.make_grid(slots)
        d = ab.abacus_search_grid(ctx, g, H, 0, len(y64))
        if d.key == 0:
            continue
        yo = y64[d.index]
        errs.append(abs(d.pred_ms - yo) / abs(yo))
    e = np.array(errs)
    out[name] = {"n": int(e.size), "max_rel_err": float(e.max()), "p99_rel_err": float(np.quantile(e, 0.99)),
                 "p50_rel_err": float(np.median(e))}
    print(name, out[name])
ab.abacus_destroy(ctx)
if a.out:
    json.dump(out, open(a.out, "w"), indent=1)
