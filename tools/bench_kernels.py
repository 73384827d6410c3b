"""Standalone building blocks at HBM scale (inputs >> 126 MB L2), CUDA events
on the launching stream, achieved GB/s vs the measured HBM peak:
  encode_candidates  (48 B written per candidate)
  select_group       (4 B read per candidate)
  predict_batch      (48 B read + 4 B written per row) fp32 / fp16 / bf16
  encode_groups      (84 B read + 48 B written per group)
  python tools/bench_kernels.py [--rows 67108864] [--out profiles/r1_kernels.json]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_sc_cui0czlzsmylg21_b200 as ab  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--rows", type=int, default=1 << 26)
ap.add_argument("--reps", type=int, default=5)
ap.add_argument("--out", default=None)
a = ap.parse_args()
with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
    HBM = json.load(f)["hbm_gbs"]

st = torch.cuda.Stream()
torch.cuda.set_stream(st)
ctx = ab.abacus_create(0, list(synth.OPS_PER_MODEL))
ab.abacus_set_stream(ctx, st)
params = synth.weights(1)
ab.abacus_load_predictor(ctx, params, ab.ABACUS_FP16)
slots = synth.cfg4_grid()
grid = ab.make_grid(slots)
T = 1
for s in slots:
    T *= s.allow_absent + s.end_hi - s.end_lo + 1
n = a.rows
first = T // 3
X = torch.empty((n, synth.D), dtype=torch.int16, device="cuda")
y = torch.empty(n, dtype=torch.float32, device="cuda")
best = torch.zeros(1, dtype=torch.int64, device="cuda")
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")  # 256 MB > L2


def timed(fn):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    fn()
    ms = []
    for _ in range(a.reps):
        flush.zero_()
        e0.record(st)
        fn()
        e1.record(st)
        torch.cuda.synchronize()
        ms.append(e0.elapsed_time(e1))
    return min(ms)


FLOP_PER_ROW = 2 * (synth.D * 32 + 32 * 32 + 32 * 32 + 32)  # 5,696 (D = 24)
res = {"rows": n, "hbm_peak_gbs": HBM, "peak_source": "MEASURED_PEAKS.json hbm_gbs"}
ms = timed(lambda: ab.abacus_encode_candidates(ctx, grid, first, n, X, st))
gb = n * synth.D * 2 / (ms * 1e-3) / 1e9
res["encode_candidates"] = {"ms": ms, "GB_per_s": gb, "frac": gb / HBM, "bytes_per_unit": synth.D * 2,
                            "units_per_s": n / (ms * 1e-3)}
for name, prec in (("predict_fp32", ab.ABACUS_FP32), ("predict_fp16", ab.ABACUS_FP16),
                   ("predict_bf16", ab.ABACUS_BF16)):
    ab.abacus_load_predictor(ctx, params, prec)
    ms = timed(lambda: ab.abacus_predict_batch(ctx, X, n, y, st))
    gb = n * (synth.D * 2 + 4) / (ms * 1e-3) / 1e9
    res[name] = {"ms": ms, "GB_per_s": gb, "frac": gb / HBM, "bytes_per_unit": synth.D * 2 + 4,
                 "units_per_s": n / (ms * 1e-3)}
    if prec == ab.ABACUS_FP32:
        # FP32 SIMT bound: 5,696 algorithmic FLOP per row against 148 SMs x 128 FFMA x 2 x 1965 MHz
        fma_peak = 148 * 128 * 2 * 1965e6 / 1e12
        tf = n * FLOP_PER_ROW / (ms * 1e-3) / 1e12
        res[name].update({"bound": "alu", "TFLOP_per_s": tf, "alu_peak_tflops": fma_peak,
                          "alu_frac": tf / fma_peak, "flop_per_unit": FLOP_PER_ROW})
H = synth.cfg4_headroom()
ms = timed(lambda: ab.abacus_select_group(ctx, grid, first, n, y, H, best, st))
gb = n * 4 / (ms * 1e-3) / 1e9
res["select_group"] = {"ms": ms, "GB_per_s": gb, "frac": gb / HBM, "bytes_per_unit": 4, "units_per_s": n / (ms * 1e-3)}
ng = min(n, 1 << 24)
groups = synth.instance_samples(200_000, seed=15)
raw = ab.make_groups([g.slots for g in groups])
rec = len(raw) // len(groups)
d_groups = torch.frombuffer(bytearray(raw), dtype=torch.uint8).cuda().repeat((ng + len(groups) - 1) // len(groups))
ms = timed(lambda: ab.abacus_encode_groups(ctx, d_groups, ng, X, None, st))
gb = ng * (rec + synth.D * 2) / (ms * 1e-3) / 1e9
res["encode_groups"] = {"ms": ms, "GB_per_s": gb, "frac": gb / HBM, "bytes_per_unit": rec + synth.D * 2,
                        "units": ng, "units_per_s": ng / (ms * 1e-3)}
ab.abacus_destroy(ctx)
print(json.dumps(res, indent=1))
if a.out:
    with open(a.out, "w") as f:
        json.dump(res, f, indent=1)
