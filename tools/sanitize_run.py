"""Small invocations of every kernel family, for compute-sanitizer (memcheck,
synccheck, racecheck, initcheck) runs on the GPU box (SURVEY.md §4 item 4,
§5 "Race detection / sanitizers").  Sizes are tiny so the instrumented run
finishes in minutes; each call still spans several tiles, a ragged tail and
(for the fused kernels) more than one CTA.

Usage: compute-sanitizer --tool memcheck python tools/sanitize_run.py
"""
import argparse
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
import paper_conf_sc_cui0czlzsmylg21_b200 as ab  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--skip", default="", help="comma list of parts to skip")
    a = ap.parse_args()
    skip = set(a.skip.split(",")) if a.skip else set()
    torch.cuda.set_device(0)
    st = torch.cuda.Stream()
    torch.cuda.set_stream(st)
    params = synth.weights(1)
    ctx = ab.abacus_create(0, list(synth.OPS_PER_MODEL))
    ab.abacus_set_stream(ctx, st)
    _, slots = synth.cfg1_grids()[3]
    grid = ab.make_grid(slots)
    T = int(np.prod([s.allow_absent + s.end_hi - s.end_lo + 1 for s in slots]))
    decs = synth.cfg2_decisions(6)
    n = 1000
    for prec in (ab.ABACUS_FP32, ab.ABACUS_FP16, ab.ABACUS_BF16):
        ab.abacus_load_predictor(ctx, params, prec)
        if "fused" not in skip:
            d = ab.abacus_search_grid(ctx, grid, 30.0, 0, T)
            d = ab.abacus_search_grid(ctx, grid, 30.0, 777, T - 1500)
            print("fused", prec, d.key, d.evaluated, flush=True)
        if "search" not in skip:
            for space in (ab.ABACUS_SPACE_GRID, ab.ABACUS_SPACE_CHAIN):
                qs, now, infl = decs[0]
                d = ab.abacus_search(ctx, qs, now, infl, space)
            print("search", prec, d.status, d.key, flush=True)
        if "batch" not in skip:
            got = ab.abacus_search_batch(ctx, decs, ab.ABACUS_SPACE_GRID)
            got = ab.abacus_search_batch(ctx, decs, ab.ABACUS_SPACE_CHAIN)
            print("batch", prec, [g.key for g in got], flush=True)
        if "predict" not in skip:
            # zero-filled first: encode writes its rows with TMA bulk stores, which
            # initcheck does not track (a false "uninitialised read" in predict otherwise)
            x = torch.zeros((n, synth.D), dtype=torch.int16, device="cuda")
            ab.abacus_encode_candidates(ctx, grid, 5, n, x, st)
            y = torch.empty(n, dtype=torch.float32, device="cuda")
            ab.abacus_predict_batch(ctx, x, n, y, st)
            key = torch.zeros(1, dtype=torch.int64, device="cuda")
            ab.abacus_select_group(ctx, grid, 5, n, y, 30.0, key, st)
            torch.cuda.synchronize()
            print("encode/predict/select", prec, float(y[:4].sum()), int(key.item()), flush=True)
    if "peer" not in skip:
        # the in-kernel cross-GPU combine with a one-rank peer communicator
        ab.abacus_load_predictor(ctx, params, ab.ABACUS_FP16)
        pc = ab.abacus_peer_comm_init(ctx, 1, 0, [ab.abacus_peer_export(ctx)])
        d = ab.abacus_search_grid(ctx, grid, 30.0, 100, T - 200, pc)
        qs, now, infl = decs[2]
        d2 = ab.abacus_search_sharded(ctx, qs, now, infl, ab.ABACUS_SPACE_GRID, 2**40, pc)
        ab.abacus_peer_comm_destroy(pc)
        print("peer", d.key, d2.key, flush=True)
    if "groups" not in skip:
        G = synth.instance_samples(300, seed=3)
        raw = ab.make_groups([g.slots for g in G])
        g = torch.frombuffer(bytearray(raw), dtype=torch.uint8).cuda()
        x = torch.empty((len(G), synth.D), dtype=torch.int16, device="cuda")
        bad = torch.zeros(1, dtype=torch.int32, device="cuda")
        ab.abacus_encode_groups(ctx, g, len(G), x, bad, st)
        torch.cuda.synchronize()
        print("encode_groups", int(bad.item()), flush=True)
    if "mway" not in skip:
        ab.abacus_load_predictor(ctx, params, ab.ABACUS_FP32)
        qs, now, infl = decs[1]
        d, r = ab.abacus_search_mway(ctx, qs, now, infl, 4)
        print("mway", d.key, r, flush=True)
    if "train" not in skip:
        G = synth.instance_samples(600, seed=3)
        gr = torch.frombuffer(bytearray(ab.make_groups([g.slots for g in G])), dtype=torch.uint8).cuda()
        X = torch.zeros((len(G), synth.D), dtype=torch.int16, device="cuda")
        ab.abacus_encode_groups(ctx, gr, len(G), X, None, st)
        t = synth.group_latency_ms(G, seed=3).astype(np.float32)
        ab.abacus_train_begin(ctx, synth.raw_weights(1, latency_shaped=False))
        ab.abacus_train_epoch(ctx, X, torch.from_numpy(t).cuda(), len(t), 256, 1e-3, None, st)
        p, loss = ab.abacus_train_params(ctx, synth.n_params())
        print("train", loss, flush=True)
    ab.abacus_destroy(ctx)
    print("sanitize_run done", flush=True)


if __name__ == "__main__":
    main()
