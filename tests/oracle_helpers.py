"""Helpers for tests: hand-built predictor weights and closed forms.

Test infrastructure; no CUDA-path code.  The closed forms here are the
independent pins of SURVEY §8(c) (counts, Sigma-n generating function,
linear-predictor knapsack).
"""
from __future__ import annotations

import itertools
import json
import os
from typing import Dict, List, Sequence

import numpy as np

H = 32
GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def zero_params(d: int) -> np.ndarray:
    return np.zeros(H * d + H + H * H + H + H * H + H + H + 1, dtype=np.float32)


def offsets(d: int) -> Dict[str, int]:
    o = {}
    cur = 0
    for name, n in [("W1", H * d), ("b1", H), ("W2", H * H), ("b2", H), ("W3", H * H), ("b3", H),
                    ("w4", H), ("b4", 1)]:
        o[name] = cur
        cur += n
    return o


def unit0_params(d: int, bias: float, coef: Dict[int, float]) -> np.ndarray:
    """MLP whose hidden unit 0 = bias + sum coef[j] x[j] and which passes unit 0
    unchanged to the output (W2[0][0] = W3[0][0] = w4[0] = 1).  ReLU-transparent
    whenever unit 0 > 0 for every input it sees."""
    p = zero_params(d)
    o = offsets(d)
    for j, v in coef.items():
        p[o["W1"] + 0 * d + int(j)] = v
    p[o["b1"] + 0] = bias
    p[o["W2"] + 0] = 1.0
    p[o["W3"] + 0] = 1.0
    p[o["w4"] + 0] = 1.0
    return p


def load_fig12():
    with open(os.path.join(GOLDEN, "fig12.json")) as f:
        return json.load(f)


def load_fig8():
    out = {"slots": []}
    with open(os.path.join(GOLDEN, "fig8.txt")) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            tok = line.split()
            if tok[0] == "slot":
                out["slots"].append(tuple(int(v) for v in tok[1:]))
            elif tok[0] == "expect":
                out["expect"] = [int(v) for v in tok[1:]]
            else:
                out[tok[0]] = int(tok[1])
    return out


def radix(s) -> int:
    return s.allow_absent + s.end_hi - s.end_lo + 1


def sum_n_polynomial(grid) -> np.ndarray:
    """Coefficient c[s] = number of candidates with Sigma n = s:
    prod_j ([absent] x^0 + sum_{e=lo..hi} x^(e - ops + 1))."""
    poly = np.array([1], dtype=object)
    for s in grid:
        f = np.zeros(s.end_hi - s.start_op + 2, dtype=object)
        if s.allow_absent:
            f[0] += 1
        for e in range(s.end_lo, s.end_hi + 1):
            f[e - s.start_op + 1] += 1
        poly = np.convolve(poly, f)
    return poly


# ---------------------------------------------------------------------------
# Linear ReLU-transparent predictor and its knapsack closed form
# ---------------------------------------------------------------------------
class LinearPredictor:
    """y = c0 + sum_{present m} beta[m] + sum_{position p} a[p] (ope_p - ops_p).

    All coefficients are non-negative dyadic numbers, so the hidden unit is
    > 0 (ReLU-transparent), every value is exact in fp64/fp32, and slot i at
    Fig.-8 position p pays a[p] per op beyond its first."""

    def __init__(self, n_models: int, kmax: int, c0: float, beta: Sequence[float], a: Sequence[float]):
        self.n_models, self.kmax = n_models, kmax
        self.c0, self.beta, self.a = float(c0), [float(v) for v in beta], [float(v) for v in a]

    def params(self) -> np.ndarray:
        d = self.n_models + 4 * self.kmax
        coef = {}
        for m in range(self.n_models):
            coef[m] = self.beta[m]
        for p in range(self.kmax):
            coef[self.n_models + 4 * p + 1] = coef.get(self.n_models + 4 * p + 1, 0.0) + self.a[p]
            coef[self.n_models + 4 * p + 0] = coef.get(self.n_models + 4 * p + 0, 0.0) - self.a[p]
        return unit0_params(d, self.c0, coef)

    def predict(self, grid, opes) -> float:
        pres = sorted((s.model_id, e - s.start_op) for s, e in zip(grid, opes) if e != 0)
        y = self.c0
        for p, (m, extra) in enumerate(pres):
            y += self.beta[m - 1] + self.a[p] * extra
        return y

    # -- closed form --------------------------------------------------------
    def _positions(self, grid, pattern):
        ms = sorted(grid[i].model_id for i in range(len(grid)) if pattern[i])
        return {m: p for p, m in enumerate(ms)}

    def best(self, grid, H: float):
        """(max sum_n, t*) of the largest feasible group, or (None, None).

        max sum_n: per presence pattern, budget = H - c0 - sum beta - sum of
        mandatory costs; extra ops bought cheapest position first (unit-value
        knapsack).  t*: greedy over digits in slot order (largest digit that
        still admits a completion with sum_n = max and cost <= H)."""
        k = len(grid)
        radices = [radix(s) for s in grid]

        def digit_choice(j, dg):
            s = grid[j]
            if s.allow_absent:
                return None if dg == 0 else s.end_lo + dg - 1
            return s.end_lo + dg

        def patterns(fixed):
            """Yield (base cost, n_fixed, sorted [(unit cost, cap)]) for every
            presence pattern of the slots after the fixed prefix."""
            j0 = len(fixed)
            opts = [([False, True] if grid[j].allow_absent else [True]) for j in range(j0, k)]
            for pres_rem in itertools.product(*opts):
                pattern = [f is not None for f in fixed] + list(pres_rem)
                pos = self._positions(grid, pattern)
                base, n_fixed, items = self.c0, 0, []
                for j in range(k):
                    if not pattern[j]:
                        continue
                    s = grid[j]
                    p = pos[s.model_id]
                    base += self.beta[s.model_id - 1]
                    if j < j0:
                        base += self.a[p] * (fixed[j] - s.start_op)
                        n_fixed += fixed[j] - s.start_op + 1
                    else:
                        nmin = s.end_lo - s.start_op + 1
                        nmax = s.end_hi - s.start_op + 1
                        base += self.a[p] * (nmin - 1)
                        n_fixed += nmin
                        items.append((self.a[p], nmax - nmin))
                items.sort()
                yield base, n_fixed, items

        def min_cost(fixed, n_target):
            """min predicted latency over completions with sum_n == n_target"""
            best = None
            for base, n_fixed, items in patterns(fixed):
                e = n_target - n_fixed
                if e < 0 or e > sum(c for _, c in items):
                    continue
                cost = base
                for c, cap in items:
                    take = min(cap, e)
                    cost += c * take
                    e -= take
                if best is None or cost < best:
                    best = cost
            return best

        nstar = None
        for base, n_fixed, items in patterns([]):
            if base > H:
                continue
            cost, n = base, n_fixed
            for c, cap in items:
                if c == 0:
                    n += cap
                    continue
                take = min(cap, int((H - cost) // c)) if H >= cost else 0
                while take > 0 and cost + c * take > H:
                    take -= 1
                cost += c * take
                n += take
                if take < cap:
                    break
            nstar = n if nstar is None else max(nstar, n)
        if nstar is None:
            return None, None
        fixed: List = []
        digits = []
        for j in range(k):
            for dg in range(radices[j] - 1, -1, -1):
                trial = fixed + [digit_choice(j, dg)]
                mc = min_cost(trial, nstar)
                if mc is not None and mc <= H:
                    fixed = trial
                    digits.append(dg)
                    break
            else:
                raise AssertionError("closed form lost the optimum")
        t = 0
        for j in range(k):
            t = t * radices[j] + digits[j]
        return nstar, t
