"""Batch-kernel rate on the config-4 workload: abacus_search_whatif with 4
BERT-large batch-size variants (4 x 9.19e9 candidates, one launch) vs the
single fused search on the same grid (device time, CUDA events)."""
import os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch
import synth
import paper_conf_sc_cui0czlzsmylg21_b200 as ab
ctx = ab.abacus_create(0, list(synth.OPS_PER_MODEL))
st = torch.cuda.Stream(); torch.cuda.set_stream(st); ab.abacus_set_stream(ctx, st)
ab.abacus_set_timing(ctx, True)
slots = synth.cfg4_grid(); H = synth.cfg4_headroom(); g = ab.make_grid(slots)
T = 9_188_218_208
for prec in (ab.ABACUS_FP16, ab.ABACUS_BF16):
    ab.abacus_load_predictor(ctx, synth.weights(1), prec)
    variants = [([8, 8, 8, b], [0, 0, 128, 512]) for b in (1, 2, 4, 8)]
    ab.abacus_search_whatif(ctx, g, variants, H)
    kw = []
    for _ in range(3):
        ab.abacus_search_whatif(ctx, g, variants, H); kw.append(ab.abacus_last_kernel_ms(ctx))
    ks = []
    for _ in range(3):
        ab.abacus_search_grid(ctx, g, H, 0, T); ks.append(ab.abacus_last_kernel_ms(ctx))
    print(prec, "whatif (batch kernel) %.4g cand/s, single %.4g cand/s, ratio %.3f" % (
        4 * T / (min(kw) * 1e-3), T / (min(ks) * 1e-3), (4 * T / min(kw)) / (T / min(ks))), flush=True)
ab.abacus_destroy(ctx)
