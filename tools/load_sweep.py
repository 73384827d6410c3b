"""NEXT-2 load sweep: the streamed, pipelined controller (config 3 services,
Poisson arrivals, Eq. 3, drop) at loads from light to past saturation, every
round decided by abacus_search on the GPU (AUTO space, 4,194,304 budget).
Per load: QoS-violation rate, throughput, query latency, rounds (= decisions)
and the search's own latency, which must stay hidden behind the group in
flight.  The simulated durations are chosen so the whole sweep
makes >= 1e5 decisions.

  python tools/load_sweep.py [--out profiles/r2_next2_load_sweep.json]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))
import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_sc_cui0czlzsmylg21_b200 as ab  # noqa: E402
import simulate_cfg3 as sim  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--out", default=None)
ap.add_argument("--loads", default="0.5,1,2,3,4,6,10,25")
ap.add_argument("--min-decisions", type=int, default=100_000)
ap.add_argument("--space", default="auto")
a = ap.parse_args()

ctx = ab.abacus_create(0, list(synth.OPS_PER_MODEL))
st = torch.cuda.Stream()
torch.cuda.set_stream(st)
ab.abacus_set_stream(ctx, st)
ab.abacus_load_predictor(ctx, synth.weights(1), ab.ABACUS_FP16)
loads = [float(v) for v in a.loads.split(",")]
rows = []
# first pass at 60 s per load measures the rounds per simulated second; the
# durations are then scaled so the sweep reaches the decision target
probe = {q: sim.simulate(ctx, q, 60.0, sim.SPACE[a.space], 4_194_304) for q in loads}
rate = sum(p["rounds"] / 60.0 for p in probe.values())
seconds = max(60.0, a.min_decisions / rate * 1.05)
total = 0
for q in loads:
    r = sim.simulate(ctx, q, seconds, sim.SPACE[a.space], 4_194_304)
    total += r["rounds"]
    rows.append(r)
    print(json.dumps({k: r[k] for k in ("qps_per_service", "queries", "completed", "qos_violation_rate",
                                        "throughput_qps", "rounds", "search_us_p50", "search_us_p99",
                                        "search_hidden")}), flush=True)
out = {"space": a.space, "budget": 4_194_304, "precision": "fp16", "simulated_s_per_load": seconds,
       "decisions_total": total, "loads": rows}
print(json.dumps({"decisions_total": total, "simulated_s_per_load": seconds}))
if a.out:
    with open(a.out, "w") as f:
        json.dump(out, f, indent=1)
ab.abacus_destroy(ctx)
