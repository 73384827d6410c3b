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
from collections import deque

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_sc_cui0czlzsmylg21_b200 as ab  # noqa: E402

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
    fifo = {m: deque() for m in services}
    ai = 0
    t = 0.0
    done_lat, violations, drops, completed = [], 0, 0, 0
    n_groups, search_us, group_ms, evaluated = 0, [], [], 0
    active = {}  # service -> [arrival, bs, seqlen, next_op]

    def admit(until):
        nonlocal ai
        while ai < len(arrivals) and arrivals[ai][0] <= until:
            ta, m, bs, sl = arrivals[ai]
            fifo[m].append((ta, bs, sl))
            ai += 1

    def refill():
        for m in services:
            if m not in active and fifo[m]:
                ta, bs, sl = fifo[m].popleft()
                active[m] = [ta, bs, sl, 1]

    inflight = 0.0  # predicted latency of the group currently executing (Eq. 3)
    horizon = seconds * 1000.0
    while t < horizon or active or any(fifo.values()):
        admit(t)
        refill()
        if not active:
            if ai >= len(arrivals):
                break
            t = max(t, arrivals[ai][0])
            continue
        ms = list(active.keys())
        qs = [synth.Query(m, active[m][3], active[m][1], active[m][2], qos[m], active[m][0]) for m in ms]
        w0 = time.perf_counter()
        d = ab.abacus_search(ctx, qs, t, inflight, space, budget)
        search_us.append((time.perf_counter() - w0) * 1e6)
        evaluated += d.evaluated
        if d.status == ab.ABACUS_DECIDE_DROP:
            m = ms[d.critical]
            del active[m]
            drops += 1
            violations += 1
            continue
        # issue the group: it runs for its predicted latency after the in-flight one
        start = t + inflight
        dur = float(d.pred_ms)
        end = start + dur
        n_groups += 1
        group_ms.append(dur)
        for i, m in enumerate(ms):
            e = d.end_op[i]
            if e == 0:
                continue
            if e >= synth.L(m):
                lat = end - active[m][0]
                done_lat.append(lat)
                completed += 1
                if lat > qos[m]:
                    violations += 1
                del active[m]
            else:
                active[m][3] = e + 1
        # pipelining (Fig. 13): the next search happens now, while this group runs
        t = start
        inflight = dur
    sim_ms = max(t + inflight, horizon)
    lat = np.array(done_lat) if done_lat else np.zeros(1)
    sa = np.array(search_us)
    return {"qps_per_service": qps, "simulated_s": sim_ms / 1000.0, "space": space, "budget": budget,
            "qos_ms": qos, "queries": len(arrivals), "completed": completed, "dropped": drops,
            "qos_violation_rate": violations / max(1, len(arrivals)),
            "throughput_qps": completed / (sim_ms / 1000.0), "latency_p50_ms": float(np.percentile(lat, 50)),
            "latency_p99_ms": float(np.percentile(lat, 99)), "groups": n_groups,
            "group_ms_mean": float(np.mean(group_ms)) if group_ms else 0.0,
            "decisions": len(search_us), "candidates_evaluated": int(evaluated),
            "search_us_p50": float(np.percentile(sa, 50)), "search_us_p99": float(np.percentile(sa, 99)),
            "search_us_p999": float(np.percentile(sa, 99.9)),
            "group_ms_min": float(np.min(group_ms)) if group_ms else 0.0,
            "search_hidden": bool(group_ms) and float(np.max(sa)) / 1000.0 < float(np.min(group_ms)),
            "note": "synthetic random-init predictor: its latency landscape is not a real model's, so QoS/throughput "
                    "figures exercise the controller mechanics only"}


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
