"""Config 5: predictor-accuracy replay (BASELINE.json configs[4]).

1e6 instance-based operator-group samples (Fig. 9) are encoded on
the GPU (abacus_encode_groups) and predicted with abacus_predict_batch in the
fp32, fp16 and bf16 paths; the fp64 oracle predicts the same groups.  Reports
per path: max / p99 / p50 relative error, MAPE (Eq. 1, with the
oracle as the 'real' latency), a log-binned error histogram, and (bf16) the
distance to the bf16-emulating oracle (rounding-point check).  Also times the
standalone encode_groups / predict_batch kernels (CUDA events).

  python tests/accuracy_replay.py [--n 1000000] [--out profiles/cfg5_accuracy.json]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402  (test infrastructure: the reference predictions)
import synth  # noqa: E402
import paper_conf_sc_cui0czlzsmylg21_b200 as ab  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--n", type=int, default=1_000_000)
ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "cfg5_accuracy.json"))
a = ap.parse_args()

params = synth.weights(1)
groups = synth.instance_samples(a.n, seed=15)
G = [g.slots for g in groups]
X64 = oracle.encode_groups(8, 4, G)
y64 = oracle.mlp64_batch(params, X64)
y_emu = oracle.mlp64_emu_batch(params, X64, flags=1 | 8)   # bf16 weights + activations (no split)

ctx = ab.abacus_create(0, list(synth.OPS_PER_MODEL))
raw = ab.make_groups(G)
d_groups = torch.frombuffer(bytearray(raw), dtype=torch.uint8).cuda()
X = torch.empty((a.n, synth.D), dtype=torch.int16, device="cuda")
bad = torch.zeros(1, dtype=torch.int32, device="cuda")
st = torch.cuda.Stream()  # explicit stream: the ABI maps NULL to the ctx's own stream
torch.cuda.set_stream(st)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
for _ in range(3):
    ab.abacus_encode_groups(ctx, d_groups, a.n, X, bad, st)
e0.record(st)
ab.abacus_encode_groups(ctx, d_groups, a.n, X, bad, st)
e1.record(st)
torch.cuda.synchronize()
enc_ms = e0.elapsed_time(e1)
assert int(bad.item()) == 0
assert np.array_equal(X.cpu().numpy(), X64), "GPU encoding differs from the oracle"

bins = [0] + [10.0 ** e for e in range(-9, 1)]
report = {"samples": a.n, "oracle_y": {"min": float(y64.min()), "median": float(np.median(y64)),
                                        "max": float(y64.max())},
          "encode_groups": {"ms": enc_ms, "bit_exact": True,
                            "GB_per_s": a.n * (synth.D * 2 + 84) / (enc_ms * 1e-3) / 1e9,
                            "bytes_per_row": "84 in (abacus_group_t) + 48 out"}}
y = torch.empty(a.n, dtype=torch.float32, device="cuda")
for name, prec, eps in (("fp32", ab.ABACUS_FP32, 1e-4), ("fp16", ab.ABACUS_FP16, 1e-2), ("bf16", ab.ABACUS_BF16, 1e-2)):
    ab.abacus_load_predictor(ctx, params, prec)
    for _ in range(3):
        ab.abacus_predict_batch(ctx, X, a.n, y, st)
    e0.record(st)
    ab.abacus_predict_batch(ctx, X, a.n, y, st)
    e1.record(st)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1)
    yg = y.cpu().numpy().astype(np.float64)
    err = np.abs(yg - y64) / np.abs(y64)
    hist, _ = np.histogram(err, bins=bins)
    r = {"max_rel_err": float(err.max()), "p99_rel_err": float(np.quantile(err, 0.99)),
         "p50_rel_err": float(np.median(err)), "mape_vs_oracle": float(np.mean(err)),
         "bar": eps, "within_bar": bool(err.max() <= eps),
         "histogram": {"bin_edges": bins, "counts": [int(v) for v in hist]},
         "predict_ms": ms, "rows_per_s": a.n / (ms * 1e-3),
         "hbm_GB_per_s": a.n * (synth.D * 2 + 4) / (ms * 1e-3) / 1e9}
    if name == "bf16":
        r["max_rel_diff_vs_plain_bf16_emulation"] = float(np.max(np.abs(yg - y_emu) / np.abs(y_emu)))
    report[name] = r
ab.abacus_destroy(ctx)
os.makedirs(os.path.dirname(a.out), exist_ok=True)
with open(a.out, "w") as f:
    json.dump(report, f, indent=1)
print(json.dumps({k: (v if not isinstance(v, dict) else {kk: vv for kk, vv in v.items() if kk != "histogram"})
                  for k, v in report.items()}, indent=1))
