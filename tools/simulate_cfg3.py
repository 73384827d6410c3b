"""Config 3 / NEXT-2: streamed, pipelined headroom-based controller in simulation.

Services: ResNet-101, ResNet-152, VGG-19, BERT-large (the paper's quad with
Bert -> BERT-large).  Per service a FIFO of queries (Poisson arrivals,
P:1504-1506; bs ~ U[1,32], BERT seqlen ~ U{16..512}); the head query is active
with next op s.  QoS per service = 2 x the predicted solo latency at the
maximum input (bs 32, seqlen 512 for Bert).

Controller (Fig. 13 pipelining P:1357-1387): when group G_i is
issued at time t with predicted latency y_i, the next group is searched right
away with Eq. 3 (in-flight prediction y_i subtracted) on the state G_i leaves
behind, and issued at t + y_i.  A DROP removes the critical query (counted as
a QoS violation) and the round searches again.  The simulated executor runs
each group for its predicted latency (the predictor is ground truth here).
Queries whose end op reaches L complete; latency = completion - arrival.

  python tools/simulate_cfg3.py --qps 50 --seconds 20 [--space grid|chain|auto]
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_sc_cui0czlzsmylg21_b200 as ab  # noqa: E402
from paper_conf_sc_cui0czlzsmylg21_b200 import controller as ctl  # noqa: E402

SPACE = {"grid": ab.ABACUS_SPACE_GRID, "chain": ab.ABACUS_SPACE_CHAIN, "auto": ab.ABACUS_SPACE_AUTO}


def solo_latency(ctx, m):
    """Predicted latency of model m alone, ops 1..L, bs 32, seqlen 512 if Bert."""
    g = [[(m, 1, synth.L(m), 32, synth.seqlen_for(m, 512))]]
    raw = ab.make_groups(g)
    d_groups = torch.frombuffer(bytearray(raw), dtype=torch.uint8).cuda()
    x = torch.empty((1, synth.D), dtype=torch.int16, device="cuda")
    y = torch.empty(1, dtype=torch.float32, device="cuda")
    st = torch.cuda.current_stream()
    ab.abacus_encode_groups(ctx, d_groups, 1, x, None, st)
    ab.abacus_predict_batch(ctx, x, 1, y, st)
    torch.cuda.synchronize()
    return float(y.item())


def simulate(ctx, qps, seconds, space, budget, seed=13):
    services = synth.cfg3_services()
    qos = {m: 2.0 * solo_latency(ctx, m) for m in services}
    arrivals = synth.cfg3_arrivals(qps, seconds * 1000.0, seed)
    search_us = []

    def search(qs, now, infl):
        w0 = time.perf_counter()
        d = ab.abacus_search(ctx, qs, now, infl, space, budget)
        search_us.append((time.perf_counter() - w0) * 1e6)
        return d

    r = ctl.simulate(search, arrivals, qos, {m: synth.L(m) for m in services})
    out = {"qps_per_service": qps, "simulated_s": seconds, "space": space, "budget": budget, "qos_ms": qos}
    out.update(ctl.summary(r, seconds))
    sa = np.array(search_us)
    out.update({"search_us_p50": float(np.percentile(sa, 50)), "search_us_p99": float(np.percentile(sa, 99)),
                "search_us_p999": float(np.percentile(sa, 99.9)),
                "search_hidden": bool(r.group_ms) and float(np.max(sa)) / 1000.0 < float(np.min(r.group_ms)),
                "note": "synthetic random-init predictor: its latency landscape is not a real model's, so "
                        "QoS/throughput figures exercise the controller mechanics only"})
    return out


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--qps", type=float, default=50.0)
    ap.add_argument("--seconds", type=float, default=20.0)
    ap.add_argument("--space", default="auto")
    ap.add_argument("--budget", type=int, default=4_194_304)
    ap.add_argument("--precision", default="fp16")
    a = ap.parse_args()
    ctx = ab.abacus_create(0, list(synth.OPS_PER_MODEL))
    st = torch.cuda.Stream()
    torch.cuda.set_stream(st)
    ab.abacus_set_stream(ctx, st)
    ab.abacus_load_predictor(ctx, synth.weights(1), {"fp32": 0, "bf16": 1, "fp16": 2}[a.precision])
    print(json.dumps(simulate(ctx, a.qps, a.seconds, SPACE[a.space], a.budget)))
    ab.abacus_destroy(ctx)
