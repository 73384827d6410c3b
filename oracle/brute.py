"""Pure-Python brute force for tiny inputs -- TEST INFRASTRUCTURE ONLY.

A second, deliberately different formulation used to pin the C oracle:
``itertools.product`` over per-slot choice lists (instead of the C oracle's
recursion with a running counter), exact rational MLP arithmetic via
``fractions.Fraction`` (instead of double), and a direct scan for the
largest feasible group.  Same paper passages as abacus_oracle.c.
"""
from __future__ import annotations

import itertools
from fractions import Fraction
from typing import List, Sequence, Tuple


def slot_choices(s) -> List[int]:
    """Choices of ope for one grid slot, in digit order: 0 (absent) first if
    allowed, then end_lo..end_hi ascending (reading c13)."""
    ch = [0] if s.allow_absent else []
    return ch + list(range(s.end_lo, s.end_hi + 1))


def enumerate_grid(grid) -> List[Tuple[int, ...]]:
    """All candidates in index order t = 0,1,..: lexicographic with the last
    slot fastest, i.e. itertools.product order."""
    return list(itertools.product(*[slot_choices(s) for s in grid]))


def chain_candidates(grid) -> List[Tuple[int, ...]]:
    """The paper's chain: critical only; then for each later slot
    j, earlier slots full and slot j growing op by op."""
    k = len(grid)
    out = [tuple([grid[0].end_hi] + [0] * (k - 1))]
    for j in range(1, k):
        for e in range(grid[j].start_op, grid[j].end_hi + 1):
            out.append(tuple([grid[i].end_hi for i in range(j)] + [e] + [0] * (k - j - 1)))
    return out


def encode(n_models: int, kmax: int, present: Sequence[Tuple[int, int, int, int, int]]) -> List[int]:
    """Fig. 8: bitmap by model id, then (ops, ope, bs, seqlen) per
    present model in ascending model id, zero padded."""
    x = [0] * (n_models + 4 * kmax)
    for p, (m, ops, ope, bs, sl) in enumerate(sorted(present)):
        x[m - 1] = 1
        x[n_models + 4 * p: n_models + 4 * p + 4] = [ops, ope, bs, sl]
    return x


def present_of(grid, opes) -> List[Tuple[int, int, int, int, int]]:
    return [(s.model_id, s.start_op, e, s.batch, s.seqlen) for s, e in zip(grid, opes) if e != 0]


def sum_n(grid, opes) -> int:
    return sum(e - s.start_op + 1 for s, e in zip(grid, opes) if e != 0)


def mlp_exact(params, x, d: int) -> Fraction:
    """Exact rational forward pass of D->32->32->32->1 with ReLU hidden layers."""
    p = [Fraction(float(v)) for v in params]
    h = 32
    o = 0
    W1 = p[o:o + h * d]; o += h * d
    b1 = p[o:o + h]; o += h
    W2 = p[o:o + h * h]; o += h * h
    b2 = p[o:o + h]; o += h
    W3 = p[o:o + h * h]; o += h * h
    b3 = p[o:o + h]; o += h
    w4 = p[o:o + h]; o += h
    b4 = p[o]
    relu = lambda v: v if v > 0 else Fraction(0)
    h1 = [relu(sum(W1[i * d + j] * x[j] for j in range(d)) + b1[i]) for i in range(h)]
    h2 = [relu(sum(W2[i * h + j] * h1[j] for j in range(h)) + b2[i]) for i in range(h)]
    h3 = [relu(sum(W3[i * h + j] * h2[j] for j in range(h)) + b3[i]) for i in range(h)]
    return sum(w4[j] * h3[j] for j in range(h)) + b4


def best_by_scan(cands, grid, ys, H) -> Tuple[int, int]:
    """Largest feasible group by direct scan: max (sum_n, t) with y <= H.
    Returns (t*, sum_n*) or (-1, -1) when nothing fits."""
    best = (-1, -1)
    for t, (opes, y) in enumerate(zip(cands, ys)):
        if y <= H:
            s = sum_n(grid, opes)
            if (s, t) > (best[1], best[0]):
                best = (t, s)
    return best
