"""Short launches of the hot kernels for ncu (no timing is taken from here).

  python tools/profile_run.py --precision fp16 --frac 16 --reps 2
runs abacus_search_grid over 1/frac of config 4 (reps times, after 1 warm-up),
plus (with --predict) one predict_batch over 1e6 config-5 rows.
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_sc_cui0czlzsmylg21_b200 as ab  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--precision", default="fp16")
ap.add_argument("--frac", type=int, default=16)
ap.add_argument("--reps", type=int, default=2)
ap.add_argument("--predict", action="store_true")
ap.add_argument("--decisions", type=int, default=0)
a = ap.parse_args()
prec = {"fp32": 0, "bf16": 1, "fp16": 2}[a.precision]
ctx = ab.abacus_create(0, list(synth.OPS_PER_MODEL))
_st = torch.cuda.Stream()
torch.cuda.set_stream(_st)
ab.abacus_set_stream(ctx, _st)
ab.abacus_load_predictor(ctx, synth.weights(1), prec)
slots = synth.cfg4_grid()
T = 1
for s in slots:
    T *= s.allow_absent + s.end_hi - s.end_lo + 1
g = ab.make_grid(slots)
for _ in range(1 + a.reps):
    d = ab.abacus_search_grid(ctx, g, synth.cfg4_headroom(), 0, T // a.frac)
print("key", d.key, "evaluated", d.evaluated)
if a.predict:
    G = [s.slots for s in synth.instance_samples(200_000, seed=15)]
    gr = torch.frombuffer(bytearray(ab.make_groups(G)), dtype=torch.uint8).cuda()
    X = torch.empty((len(G), 24), dtype=torch.int16, device="cuda")
    ab.abacus_encode_groups(ctx, gr, len(G), X)  # the product's encoder builds the input rows
    x = X.repeat(5, 1).contiguous()
    y = torch.empty(x.shape[0], device="cuda")
    for _ in range(2):
        ab.abacus_predict_batch(ctx, x, x.shape[0], y)
    torch.cuda.synchronize()
for qs, now, infl in synth.cfg2_decisions(a.decisions):
    ab.abacus_search(ctx, qs, now, infl, ab.ABACUS_SPACE_GRID)
ab.abacus_destroy(ctx)
