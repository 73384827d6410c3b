"""Per-candidate rate of the batch kernel vs the single-search kernel on the
SAME decisions (config 3, AUTO budget 4,194,304): device time (CUDA events)
summed over single abacus_search calls vs one abacus_search_batch call."""
import os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np
import torch
import synth
import paper_conf_sc_cui0czlzsmylg21_b200 as ab

ctx = ab.abacus_create(0, list(synth.OPS_PER_MODEL))
st = torch.cuda.Stream(); torch.cuda.set_stream(st); ab.abacus_set_stream(ctx, st)
ab.abacus_load_predictor(ctx, synth.weights(1), ab.ABACUS_FP16)
ab.abacus_set_timing(ctx, True)
for cfg, space, budget in (("cfg3", ab.ABACUS_SPACE_AUTO, 4194304), ("cfg3", ab.ABACUS_SPACE_GRID, 2**40),
                           ("cfg2", ab.ABACUS_SPACE_GRID, 2**40)):
    decs = synth.cfg3_decisions(1124)[100:] if cfg == "cfg3" else synth.cfg2_decisions(1124)[100:]
    ab.abacus_search_batch(ctx, decs, space, budget)
    got = ab.abacus_search_batch(ctx, decs, space, budget)
    kb = ab.abacus_last_kernel_ms(ctx)
    ev = sum(d.evaluated for d in got)
    ks, evs = 0.0, 0
    big = [i for i, d in enumerate(got) if d.evaluated >= 1_000_000]
    for i, (qs, now, infl) in enumerate(decs):
        d = ab.abacus_search(ctx, qs, now, infl, space, budget)
        k = ab.abacus_last_kernel_ms(ctx)
        if i in big:
            ks += k; evs += d.evaluated
    kb_big = None
    if big:
        sub = [decs[i] for i in big]
        ab.abacus_search_batch(ctx, sub, space, budget)
        kb_big = ab.abacus_last_kernel_ms(ctx)
    print(cfg, space, "batch all: %.4g cand/s (%.2f ms, %d dec)" % (ev / (kb * 1e-3), kb, len(decs)),
          "| decisions >= 1e6: single %.4g cand/s, batch %.4g cand/s (%d dec)" % (
              evs / (ks * 1e-3) if ks else 0, evs / (kb_big * 1e-3) if kb_big else 0, len(big)), flush=True)
ab.abacus_destroy(ctx)
