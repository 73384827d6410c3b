"""Fig. 23 on B200: per-decision latency of
the paper's multi-way search (abacus_search_mway) against the number of ways,
1..16, through the C ABI (tools/decision_latency.c, host clock around each
call), for config 2 (3-way) and config 3 (4-way) decisions, next to the
exhaustive GRID / CHAIN searches.  The paper (one Xeon core): 0.066 ms at 1
way, 0.088 ms flat from 2 to ~15 ways.

  python tools/fig23.py [--out profiles/r2_fig23_mway.json] [-n 10000]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "tools"))
import decision_latency as dl  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--out", default=None)
ap.add_argument("-n", type=int, default=10_000)
a = ap.parse_args()
keep = ("p50_us", "p90_us", "p99_us", "p999_us", "evaluated_mean", "evaluated_p99", "drops")
res = {"paper": {"1_way_ms": 0.066, "2_to_15_ways_ms": 0.088, "hardware": "Xeon Silver 4210R, 1 core",
                 "cite": "PAPER.md:2514-2527"}, "configs": {}}
for cfg in ("cfg2", "cfg3"):
    rows = {}
    for ways in range(1, 17):
        r = dl.run(cfg, "mway", "fp32", a.n, 100, ways)
        rows[str(ways)] = {k: r[k] for k in keep}
        print(cfg, ways, rows[str(ways)], flush=True)
    ex = {}
    for space in ("grid", "chain"):
        r = dl.run(cfg, space, "fp16", a.n, 100, 0)
        ex[space] = {k: r[k] for k in keep}
    res["configs"][cfg] = {"mway_fp32": rows, "exhaustive_fp16": ex}
print(json.dumps(res))
if a.out:
    with open(a.out, "w") as f:
        json.dump(res, f, indent=1)
