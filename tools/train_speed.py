import sys, os, json
sys.path.insert(0, '/root/repo')
import numpy as np, torch
import synth, paper_conf_sc_cui0czlzsmylg21_b200 as ab
ctx = ab.abacus_create(0, list(synth.OPS_PER_MODEL))
st = torch.cuda.Stream(); torch.cuda.set_stream(st); ab.abacus_set_stream(ctx, st)
n = 1 << 18
x = torch.randint(0, 30, (n, synth.D), dtype=torch.int16, device="cuda")
y = torch.rand(n, device="cuda") * 20 + 1
ab.abacus_train_begin(ctx, synth.raw_weights(1, latency_shaped=False))
for B in (128, 256, 1024, 4096, 16384, 65536):
    ab.abacus_train_epoch(ctx, x, y, n, B, 1e-4, None, st)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    ab.abacus_train_epoch(ctx, x, y, n, B, 1e-4, None, st)
    e1.record(st); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1); steps = n // B
    print(json.dumps({"batch": B, "us_per_step": ms * 1e3 / steps, "samples_per_s": n / (ms * 1e-3)}))
