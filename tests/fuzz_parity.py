"""Randomised GPU-vs-oracle parity fuzzing (test infrastructure; not collected
by pytest, run by hand on a GPU box):

    python tests/fuzz_parity.py --minutes 10

Random grids (k, models, start ops, end ranges, absent flags, bs, seqlen,
sub-ranges [first, first+count)) through abacus_search_grid; random
scheduling rounds through abacus_search (GRID / CHAIN / AUTO) and the same
rounds batched through abacus_search_batch (bit-identical to the singles);
random what-if variants.  Every precision.  Acceptance as in the parity tests
(reading c18).  Prints one line per failure and a summary."""
import argparse
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import torch  # noqa: E402

import oracle  # noqa: E402
import synth  # noqa: E402
import paper_conf_sc_cui0czlzsmylg21_b200 as ab  # noqa: E402

EPS = {ab.ABACUS_FP32: 1e-4, ab.ABACUS_BF16: 1e-2, ab.ABACUS_FP16: 1e-2}


def rand_grid(rng):
    k = int(rng.integers(1, 5))
    models = [int(m) for m in rng.choice(np.arange(1, 9), size=k, replace=False)]
    g = []
    for m in models:
        L = synth.L(m)
        s = int(rng.integers(1, L + 1))
        width = int(rng.choice([1, 2, 5, 17, 60, 130, 300]))
        lo = int(rng.integers(s, L + 1))
        hi = min(L, lo + width - 1)
        g.append(synth.GridSlot(m, s, int(rng.integers(1, 33)), synth.seqlen_for(m, int(rng.integers(8, 513))),
                                lo, hi, int(rng.integers(0, 2))))
    return g


def rand_round(rng):
    k = int(rng.integers(1, 5))
    models = [int(m) for m in rng.choice(np.arange(1, 9), size=k, replace=False)]
    now = 100.0
    qs = []
    for m in models:
        ts = float(rng.uniform(0, 80))
        qs.append(synth.Query(m, int(rng.integers(1, synth.L(m) + 1)), int(rng.integers(1, 33)),
                              synth.seqlen_for(m, int(rng.integers(8, 513))),
                              float(rng.uniform(5, 80)) + (now - ts), ts))
    return qs, now, float(rng.uniform(0, 5))


def run(seed, minutes=None, iterations=None):
    """Fuzz until the time or the iteration budget is spent (one iteration =
    one precision: 4 grids, 8 rounds single + batched, one what-if set).
    Returns (counts, failures)."""
    rng = np.random.default_rng(seed)
    params = synth.weights(1)
    ctx = ab.abacus_create(0, list(synth.OPS_PER_MODEL))
    st = torch.cuda.Stream()
    prev = torch.cuda.current_stream()
    torch.cuda.set_stream(st)
    ab.abacus_set_stream(ctx, st)
    t_end = time.time() + (minutes if minutes is not None else 1e9) * 60
    n = {"grid": 0, "round": 0, "batch": 0, "whatif": 0}
    fails = 0
    precs = [ab.ABACUS_FP32, ab.ABACUS_FP16, ab.ABACUS_BF16]
    it = 0
    while time.time() < t_end and (iterations is None or it < iterations):
        prec = precs[it % 3]
        it += 1
        eps = EPS[prec]
        ab.abacus_load_predictor(ctx, params, prec)
        # sweeps
        for _ in range(4):
            g = rand_grid(rng)
            T = oracle.grid_size(g)
            if T > 3_000_000:
                continue
            first = int(rng.integers(0, T))
            count = int(rng.integers(0, T - first + 1))
            _, y, _, _ = oracle.sweep(params, g, 0.0, first=first, count=min(count, 20000), want_y=True)
            H = float(np.float32(np.quantile(y, rng.uniform(0.05, 0.95)))) if len(y) else 10.0
            d = ab.abacus_search_grid(ctx, ab.make_grid(g), H, first, count)
            r, _, _, _ = oracle.sweep(params, g, H, first=first, count=count, eps=eps)
            ok = d.evaluated == count and r.maxkey_strict <= d.key <= r.maxkey_loose
            if ok and d.key:
                _, yt, _, _ = oracle.sweep(params, g, H, first=d.index, count=1, want_y=True)
                ok = abs(d.pred_ms - yt[0]) <= eps * abs(yt[0]) + 1e-6
            if ok and first == 0 and count > 0:
                ok = abs(d.pred_critical_only_ms - r.y0) <= eps * abs(r.y0) + 1e-6
            n["grid"] += 1
            if not ok:
                fails += 1
                print("FAIL grid", prec, g, H, first, count, d.key, r.maxkey_strict, r.maxkey_loose, flush=True)
        # scheduling rounds, single and batched
        rounds = [rand_round(rng) for _ in range(8)]
        space = int(rng.integers(0, 3))
        budget = int(rng.choice([1 << 12, 1 << 16, 1 << 20]))
        singles = []
        for qs, now, infl in rounds:
            d = ab.abacus_search(ctx, qs, now, infl, space, budget)
            singles.append(d)
            od = oracle.search(params, qs, now, infl, space=space, budget=budget, eps=eps)
            near = abs(od.pred_critical_only_ms - od.headroom_ms) <= eps * abs(od.headroom_ms)
            ok = (d.status == od.status) or near
            if ok and d.status == 0 and od.status == 0:
                ok = od.maxkey_strict <= d.key <= od.maxkey_loose
            n["round"] += 1
            if not ok:
                fails += 1
                print("FAIL round", prec, space, budget, qs, now, infl, d.status, od.status, d.key,
                      od.maxkey_strict, od.maxkey_loose, flush=True)
        if prec != ab.ABACUS_FP32:
            got = ab.abacus_search_batch(ctx, rounds, space, budget)
            for dd, d in zip(got, singles):
                n["batch"] += 1
                if (dd.status, dd.key, list(dd.end_op)) != (d.status, d.key, list(d.end_op)):
                    fails += 1
                    print("FAIL batch", prec, dd.status, d.status, dd.key, d.key, flush=True)
        # what-if
        g = rand_grid(rng)
        T = oracle.grid_size(g)
        if T <= 200_000:
            k = len(g)
            variants = [([int(rng.integers(1, 33)) for _ in range(k)],
                         [synth.seqlen_for(s.model_id, int(rng.integers(8, 513))) for s in g])
                        for _ in range(int(rng.integers(1, 5)))]
            H = float(rng.uniform(5, 60))
            per, best, bv = ab.abacus_search_whatif(ctx, ab.make_grid(g), variants, H)
            oper, _, (strict, loose) = oracle.whatif(params, g, variants, H, eps=eps)
            ok = strict <= best.key <= loose and all(
                oper[v].maxkey_strict <= per[v].key <= oper[v].maxkey_loose for v in range(len(variants)))
            n["whatif"] += 1
            if not ok:
                fails += 1
                print("FAIL whatif", prec, g, variants, H, flush=True)
    ab.abacus_destroy(ctx)
    torch.cuda.set_stream(prev)
    return n, fails


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--minutes", type=float, default=5.0)
    ap.add_argument("--seed", type=int, default=1234)
    a = ap.parse_args()
    n, fails = run(a.seed, minutes=a.minutes)
    print("fuzz done:", n, "failures:", fails, flush=True)


if __name__ == "__main__":
    main()
