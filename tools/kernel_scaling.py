"""Fused kernel device time (CUDA events on the ctx stream) vs. launch size,
and the host-side time of the blocking call, to locate fixed costs."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import synth  # noqa: E402
import paper_conf_sc_cui0czlzsmylg21_b200 as ab  # noqa: E402

prec = {"fp32": 0, "bf16": 1, "fp16": 2}[sys.argv[1] if len(sys.argv) > 1 else "fp16"]
ctx = ab.abacus_create(0, list(synth.OPS_PER_MODEL))
ab.abacus_load_predictor(ctx, synth.weights(1), prec)
ab.abacus_set_timing(ctx, True)
g = ab.make_grid(synth.cfg4_grid())
H = synth.cfg4_headroom()
for count in [0, 1, 128, 1280, 12800, 128000, 1280000, 12800000]:
    ks, hs = [], []
    for i in range(60):
        t0 = time.perf_counter()
        ab.abacus_search_grid(ctx, g, H, 10**9, count)
        t1 = time.perf_counter()
        if i >= 10:
            ks.append(ab.abacus_last_kernel_ms(ctx) * 1e3)
            hs.append((t1 - t0) * 1e6)
    print("count %9d  kernel %8.2f us (p50)  host call %8.2f us (p50)" % (count, np.median(ks), np.median(hs)))
ab.abacus_destroy(ctx)
