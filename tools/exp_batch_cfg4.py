"""Batch kernel vs single-search kernel per candidate on config-4-sized GRID
decisions (four queries at next_op 1: ResNet-152, Inception-v3, BERT-base
seq 128, BERT-large seq 512 -> ~9.2e9 candidates per decision), device time
(CUDA events): n single abacus_search calls vs one abacus_search_batch of the
same n rounds.  Both sides evaluate the same candidates."""
import os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch
import synth
import paper_conf_sc_cui0czlzsmylg21_b200 as ab

prec = {"fp16": ab.ABACUS_FP16, "bf16": ab.ABACUS_BF16}[sys.argv[1] if len(sys.argv) > 1 else "fp16"]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 4
ctx = ab.abacus_create(0, list(synth.OPS_PER_MODEL))
st = torch.cuda.Stream(); torch.cuda.set_stream(st); ab.abacus_set_stream(ctx, st)
ab.abacus_load_predictor(ctx, synth.weights(1), prec)
ab.abacus_set_timing(ctx, True)
H = synth.cfg4_headroom()
now = 1000.0
rounds = []
for i in range(n):
    h = H * (0.9 + 0.05 * i)
    qs = [synth.Query(3, 1, 8, 0, h + 0.0, now), synth.Query(4, 1, 8, 0, h + 5.0, now),
          synth.Query(7, 1, 8, 128, h + 7.0, now), synth.Query(8, 1, 4, 512, h + 9.0, now)]
    rounds.append((qs, now, 0.0))
S = ab.ABACUS_SPACE_GRID
ab.abacus_search_batch(ctx, rounds, S, 2**40)
for rep in range(3):
    got = ab.abacus_search_batch(ctx, rounds, S, 2**40)
    kb = ab.abacus_last_kernel_ms(ctx)
    ks, evs, same = 0.0, 0, True
    for (qs, nw, infl), g in zip(rounds, got):
        d = ab.abacus_search(ctx, qs, nw, infl, S, 2**40)
        ks += ab.abacus_last_kernel_ms(ctx)
        evs += d.evaluated
        same &= (d.key, list(d.end_op)) == (g.key, list(g.end_op))
    ev = sum(g.evaluated for g in got)
    print("rep %d: %d decisions, %.3g cand each | batch %.4g cand/s (%.1f ms) | single %.4g cand/s (%.1f ms) "
          "| ratio %.3f | identical %s" % (rep, n, ev / n, ev / (kb * 1e-3), kb, evs / (ks * 1e-3), ks,
                                           (ev / kb) / (evs / ks), same), flush=True)
ab.abacus_destroy(ctx)
