"""NEXT-2: the streamed, pipelined headroom-based query
controller, as a discrete-event simulation around the GPU search.

What it models (P:630-753 steps 1-3, Fig. 13 pipelining P:1357-1387,
drop P:1293-1298, QoS P:1505-1510):

* Each service keeps a FIFO of queries (arrival time, batch, seqlen); its head
  query is active with next op ``s`` (1-based).
* A round: headrooms follow Eq. 2 with t_start = arrival and the service's QoS
  target, minus the prediction still in flight (Eq. 3); ``search`` returns the
  group to issue or DROPs the critical query (counted as a QoS violation; the
  round is searched again).
* The executor runs a group for its predicted latency (the predictor is the
  ground truth here).  A group issued at ``start`` ends at ``start + y``;
  queries whose end op reaches L complete at that time, the others continue
  at ``ope + 1``.
* Pipelining: the next round is searched at the START of the group just
  issued, on the state it leaves behind, with that group's prediction in
  flight (Eq. 3); the next group is issued when the executor frees up.  When
  the controller idles (no active query), the next search happens at the next
  arrival with the remaining in-flight time ``max(0, free - t)``.

``search(queries, now_ms, inflight_ms)`` is injected: the product passes
``abacus_search`` of a context (GPU); tests also drive it with the fp64 oracle.
Host-side logic only: every prediction runs in the search.
"""
from __future__ import annotations

from collections import deque
from dataclasses import dataclass, field
from typing import Callable, Dict, List, Sequence, Tuple

DROP = 1


@dataclass
class Query:
    """ABI abacus_query_t field names (model_id, next_op, batch, seqlen, qos_ms, t_start_ms)."""
    model_id: int
    next_op: int
    batch: int
    seqlen: int
    qos_ms: float
    t_start_ms: float


@dataclass
class SimResult:
    arrivals: int
    completed: int
    dropped: int
    violations: int            # drops + completions later than QoS
    groups: int
    rounds: int                # searches, including the ones that dropped
    latencies_ms: List[float] = field(default_factory=list)
    group_ms: List[float] = field(default_factory=list)
    evaluated: int = 0
    end_ms: float = 0.0
    log: List[Tuple] = field(default_factory=list)   # (t, status, ((model, next_op), ...), end ops, y)


def simulate(search: Callable, arrivals: Sequence[Tuple[float, int, int, int]], qos: Dict[int, float],
             ops: Dict[int, int], keep_log: bool = False) -> SimResult:
    """arrivals: (t_ms, model_id, batch, seqlen) sorted by time; qos[m], ops[m] = L per service.
    Runs until every arrival has completed or been dropped."""
    services = sorted(qos)
    fifo = {m: deque() for m in services}
    active: Dict[int, list] = {}   # service -> [arrival, batch, seqlen, next_op]
    res = SimResult(arrivals=len(arrivals), completed=0, dropped=0, violations=0, groups=0, rounds=0)
    ai = 0
    t = 0.0
    free = 0.0                      # the executor is busy until `free`
    n = len(arrivals)
    while True:
        while ai < n and arrivals[ai][0] <= t:
            ta, m, bs, sl = arrivals[ai]
            fifo[m].append((ta, bs, sl))
            ai += 1
        for m in services:
            if m not in active and fifo[m]:
                ta, bs, sl = fifo[m].popleft()
                active[m] = [ta, bs, sl, 1]
        if not active:
            if ai >= n:
                break
            t = max(t, arrivals[ai][0])   # idle until the next arrival
            continue
        inflight = max(0.0, free - t)      # Eq. 3: prediction of the group still running
        ms = [m for m in services if m in active]
        qs = [Query(m, active[m][3], active[m][1], active[m][2], qos[m], active[m][0]) for m in ms]
        d = search(qs, t, inflight)
        res.rounds += 1
        res.evaluated += int(d.evaluated)
        if d.status == DROP:          # the critical query cannot finish in time
            m = ms[d.critical]
            del active[m]
            res.dropped += 1
            res.violations += 1
            if keep_log:
                res.log.append((t, DROP, tuple((q.model_id, q.next_op) for q in qs), (), float("nan")))
            continue
        start = t + inflight
        y = float(d.pred_ms)
        end = start + y
        res.groups += 1
        res.group_ms.append(y)
        ends = tuple(int(d.end_op[i]) for i in range(len(ms)))
        if keep_log:
            res.log.append((t, 0, tuple((q.model_id, q.next_op) for q in qs), ends, y))
        for m, e in zip(ms, ends):
            if e == 0:
                continue
            if e >= ops[m]:
                lat = end - active[m][0]
                res.latencies_ms.append(lat)
                res.completed += 1
                if lat > qos[m]:
                    res.violations += 1
                del active[m]
            else:
                active[m][3] = e + 1
        free = end
        t = start                    # Fig. 13: search the next group while this one runs
    res.end_ms = max(t, free)
    return res


def summary(res: SimResult, seconds: float) -> dict:
    import numpy as np
    lat = np.array(res.latencies_ms) if res.latencies_ms else np.zeros(1)
    return {"queries": res.arrivals, "completed": res.completed, "dropped": res.dropped,
            "qos_violation_rate": res.violations / max(1, res.arrivals),
            "throughput_qps": res.completed / max(seconds, res.end_ms / 1000.0),
            "latency_p50_ms": float(np.percentile(lat, 50)), "latency_p99_ms": float(np.percentile(lat, 99)),
            "groups": res.groups, "rounds": res.rounds,
            "group_ms_mean": float(np.mean(res.group_ms)) if res.group_ms else 0.0,
            "group_ms_min": float(np.min(res.group_ms)) if res.group_ms else 0.0,
            "candidates_evaluated": res.evaluated}
