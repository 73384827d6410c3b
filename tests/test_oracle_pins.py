"""Pins of the fp64 oracle against what the paper and mathematics fix.

Each test names the passage it pins.  None of them re-types the oracle's
formula: they use the paper's printed values (Fig. 8, Fig. 12), hand-computed
dyadic arithmetic, brute force with exact rationals, closed-form counts and a
knapsack closed form.  CPU only.
"""
import itertools
import math
from fractions import Fraction

import numpy as np
import pytest

import oracle
import synth
from oracle import brute
from oracle_helpers import (LinearPredictor, load_fig8, load_fig12, offsets, radix, sum_n_polynomial,
                            unit0_params, zero_params)


# ---------------------------------------------------------------- Fig. 8 ----
def test_fig8_literal_vector():
    """P:859-866 Fig. 8: '0 0 0 1 0 0 1 3 18 4 0 4 12 16 32'."""
    g = load_fig8()
    x = oracle.encode(g["n_models"], g["kmax"], g["slots"])
    assert list(x) == g["expect"]
    # slot packing is by model id, not by caller order (reading c4)
    x2 = oracle.encode(g["n_models"], g["kmax"], list(reversed(g["slots"])))
    assert list(x2) == g["expect"]
    assert brute.encode(g["n_models"], g["kmax"], g["slots"]) == g["expect"]


def test_encode_rejects_duplicate_and_out_of_range():
    """Reading c9: the bitmap cannot encode two queries of one model."""
    with pytest.raises(ValueError):
        oracle.encode(7, 2, [(4, 1, 2, 1, 0), (4, 3, 4, 1, 0)])
    with pytest.raises(ValueError):
        oracle.encode(7, 2, [(8, 1, 2, 1, 0)])
    with pytest.raises(ValueError):
        oracle.encode(7, 2, [(1, 1, 2, 1, 0), (2, 1, 2, 1, 0), (3, 1, 2, 1, 0)])


def test_encode_vs_brute_random_groups():
    groups = synth.instance_samples(300, seed=99)
    X = oracle.encode_groups(8, 4, [g.slots for g in groups])
    for g, x in zip(groups, X):
        assert list(x) == brute.encode(8, 4, g.slots)
        assert sum(x[:8]) == len(g.slots)


# ------------------------------------------------------- dyadic MLP --------
def _dyadic_params():
    """Hand-built weights, every intermediate a small dyadic rational."""
    d = 2
    p = zero_params(d)
    o = offsets(d)
    W1 = {(0, 0): 1.0, (0, 1): 2.0, (1, 0): -1.0, (1, 1): 0.5}
    for (i, j), v in W1.items():
        p[o["W1"] + i * d + j] = v
    p[o["b1"] + 0], p[o["b1"] + 1] = 0.5, 1.0
    for (i, j), v in {(0, 0): 2.0, (1, 0): -1.0, (2, 0): 0.25}.items():
        p[o["W2"] + i * 32 + j] = v
    p[o["W2"] + 0 * 32 + 1] = 4.0
    p[o["b2"] + 0], p[o["b2"] + 1] = -1.0, 0.25
    for (i, j), v in {(0, 0): 0.5, (0, 2): 2.0, (1, 0): -1.0, (5, 2): -2.0}.items():
        p[o["W3"] + i * 32 + j] = v
    p[o["b3"] + 0], p[o["b3"] + 1], p[o["b3"] + 5] = 0.25, 3.0, 3.0
    p[o["w4"] + 0], p[o["w4"] + 1], p[o["w4"] + 5] = 1.5, 7.0, 4.0
    p[o["b4"]] = -2.0
    return p


def test_dyadic_mlp_hand_computed():
    """x = (3, 1).  By hand:
    h1 = relu(1*3 + 2*1 + .5, -1*3 + .5*1 + 1) = (5.5, 0)        [unit 1 clipped]
    h2 = relu(2*5.5 + 4*0 - 1, -5.5 + .25, .25*5.5) = (10, 0, 1.375)
    h3: u0 = .5*10 + 2*1.375 + .25 = 8;  u1 = -10 + 3 -> 0;  u5 = -2*1.375 + 3 = .25
    y = 1.5*8 + 7*0 + 4*.25 - 2 = 11."""
    p = _dyadic_params()
    x = np.array([3, 1], dtype=np.int16)
    assert oracle.mlp64(p, x) == 11.0
    assert brute.mlp_exact(p, [3, 1], 2) == Fraction(11)
    # every value has <= 8 significant bits: the bf16-emulating mode is exact too
    assert oracle.mlp64_emu_batch(p, x.reshape(1, 2), flags=15)[0] == 11.0
    # a transposed W1 or a dropped ReLU would change the result
    assert oracle.mlp64(p, np.array([1, 3], dtype=np.int16)) != 11.0


def test_bf16_rounding_points():
    """RNE to 8 significant bits: ties to even (bf16, c16)."""
    assert oracle.round_bf16(257.0) == 256.0
    assert oracle.round_bf16(259.0) == 260.0
    assert oracle.round_bf16(471.0) == 472.0
    assert oracle.round_bf16(1.0 / 3.0) == 0.333984375
    assert oracle.round_bf16(-3.0) == -3.0


def test_mlp_vs_exact_rationals_random():
    p = synth.weights(1) if _have_shape() else synth.raw_weights(1)
    groups = synth.instance_samples(40, seed=5)
    X = oracle.encode_groups(8, 4, [g.slots for g in groups])
    y = oracle.mlp64_batch(p, X)
    for xi, yi in zip(X, y):
        ex = brute.mlp_exact(p, [int(v) for v in xi], 24)
        assert abs(yi - float(ex)) <= 1e-12 * max(1.0, abs(float(ex)))


def _have_shape():
    try:
        synth.weights(1)
        return True
    except RuntimeError:
        return False


# -------------------------------------------------------- Eq. 2 / 3 ---------
def test_headroom_worked_example():
    """Eq. 2 and Eq. 3: qos 50, start 100, now 120,
    in-flight prediction 5 -> 50 - 20 - 5 = 25 ms."""
    assert oracle.headroom(50.0, 100.0, 120.0, 5.0) == 25.0
    assert oracle.headroom(50.0, 100.0, 120.0, 0.0) == 30.0


def test_order_ascending_ties_by_model():
    """P:630-633 ascending headroom; reading c10 ties by model id."""
    assert oracle.order([45.0, 35.0, 25.0], [3, 2, 1]) == [2, 1, 0]
    assert oracle.order([10.0, 10.0, 5.0], [7, 2, 4]) == [2, 1, 0]


# --------------------------------------------------------------- Fig. 12 ---
def _fig12_setup():
    f = load_fig12()
    d = f["n_models"] + 4 * f["kmax"]
    p = unit0_params(d, f["unit0"]["bias"], {int(k): v for k, v in f["unit0"]["coef"].items()})
    qs = [synth.Query(q["model_id"], q["next_op"], 1, 0, q["headroom_ms"], 0.0) for q in f["queries"]]
    return f, p, qs


@pytest.mark.parametrize("space", [0, 1])
def test_fig12_replay(space):
    """q3 fully, q2 fully, first two ops of q1; headroom 25->15->10->0."""
    f, p, qs = _fig12_setup()
    e = f["expected"]
    dec = oracle.search(p, qs, now=0.0, inflight=0.0, space=space, n_models=f["n_models"],
                        kmax=f["kmax"], ops_per_model=f["ops_per_model"])
    names = [q["name"] for q in f["queries"]]
    assert dec.status == 0
    assert names[dec.critical] == e["critical"]
    assert {names[i]: dec.end_op[i] for i in range(3)} == e["end_op"]
    assert dec.pred_ms == e["pred_ms"]
    assert dec.headroom_ms == 25.0
    assert dec.index == (e["grid_t"] if space == 0 else e["chain_u"])
    if space == 0:
        assert dec.evaluated == e["grid_T"]


def test_fig12_headroom_trace_and_runner_up():
    f, p, qs = _fig12_setup()
    e = f["expected"]
    q3, q2, q1 = (synth.GridSlot(1, 1, 1, 0, 5, 5, 0), synth.GridSlot(2, 2, 1, 0, 2, 5, 1),
                  synth.GridSlot(3, 1, 1, 0, 1, 5, 1))
    grid = [q3, q2, q1]
    r, y, x, ope = oracle.sweep(p, grid, 25.0, n_models=3, kmax=3, want_y=True, want_ope=True)
    # chain probes: critical alone; + q2 full; + q1 ops 1-2
    trace = [25.0 - y[0], 25.0 - y[4 * 6 + 0], 25.0 - y[26]]
    assert [25.0] + trace == e["remaining_headroom_trace_ms"]
    assert y[e["runner_up"]["t"]] == e["runner_up"]["y"]
    assert y[5] == e["grid_t5_y"]
    assert r.best_index == e["grid_t"]


# ------------------------------------------------------ enumeration ---------
def test_enumeration_matches_itertools_product():
    """Brute force on tiny grids (k <= 3, L <= 5): the recursion's order equals
    itertools.product order (last slot fastest); |GRID| = prod radix."""
    grids = synth.tiny_grids(60, seed=3, kmax=3, max_len=5)
    p = synth.raw_weights(2)
    for grid in grids:
        T = oracle.grid_size(grid)
        assert T == math.prod(radix(s) for s in grid)
        r, y, x, ope = oracle.sweep(p, grid, 0.0, want_ope=True, want_x=True)
        cands = brute.enumerate_grid(grid)
        assert len(cands) == T == r.evaluated
        assert [tuple(row) for row in ope] == cands
        for opes, xi in zip(cands, x):
            assert list(xi) == brute.encode(8, 4, brute.present_of(grid, opes))


def test_sum_n_distribution_closed_form():
    """#candidates with Sigma n = s is the x^s coefficient of
    prod_j ([absent] + sum_e x^(e - ops + 1))."""
    for grid in synth.tiny_grids(20, seed=4, kmax=4, max_len=6):
        cands = brute.enumerate_grid(grid)
        hist = np.zeros(200, dtype=object)
        for c in cands:
            hist[brute.sum_n(grid, c)] += 1
        poly = sum_n_polynomial(grid)
        assert list(hist[:len(poly)]) == list(poly)
        assert sum(hist[len(poly):]) == 0


def test_chain_count_closed_form():
    """|CHAIN| = 1 + sum_{j>=2} R_j."""
    rng = np.random.default_rng(0)
    p = synth.raw_weights(2)
    for _ in range(20):
        k = int(rng.integers(1, 5))
        ms = rng.choice(np.arange(1, 9), size=k, replace=False)
        qs = [synth.Query(int(m), int(rng.integers(1, synth.L(int(m)) + 1)), 8, 0, 100.0, 0.0) for m in ms]
        dec = oracle.search(p, qs, 0.0, 0.0, space=1)
        R = [synth.L(q.model_id) - q.next_op + 1 for q in qs]
        crit = dec.critical
        assert dec.evaluated == 1 + sum(R[i] for i in range(k) if i != crit)


# ------------------------------------------------------ selection rule ------
def test_sweep_best_vs_bruteforce_scan():
    """The largest feasible group (max Sigma n, then max t) by direct scan."""
    p = synth.raw_weights(7)
    rng = np.random.default_rng(1)
    for grid in synth.tiny_grids(40, seed=8, kmax=3, max_len=6):
        r, y, _, _ = oracle.sweep(p, grid, 0.0, want_y=True)
        H = float(np.quantile(y, rng.uniform(0.05, 0.95)))
        r, y, _, _ = oracle.sweep(p, grid, H, want_y=True)
        cands = brute.enumerate_grid(grid)
        t, s = brute.best_by_scan(cands, grid, y, H)
        if t < 0:
            assert r.best_key == 0
        else:
            assert r.best_index == t and r.best_sum_n == s
            assert r.best_key == ((s + 1) << 40) | t
            assert r.best_y <= H


def test_range_shards_combine_to_full_sweep():
    """G contiguous shards [floor(rT/G), floor((r+1)T/G)): max key, feasible and
    hash sums equal the unsharded sweep."""
    p = synth.raw_weights(3)
    grid = [synth.GridSlot(1, 3, 4, 0, 3, 40, 1), synth.GridSlot(5, 1, 4, 0, 1, 40, 1),
            synth.GridSlot(7, 10, 2, 64, 12, 30, 0)]
    T = oracle.grid_size(grid)
    full, y, _, _ = oracle.sweep(p, grid, 0.0, want_y=True)
    H = float(np.median(y))
    full, _, _, _ = oracle.sweep(p, grid, H)
    for G in (2, 3, 8):
        parts = [oracle.sweep(p, grid, H, first=(r * T) // G, count=((r + 1) * T) // G - (r * T) // G)[0]
                 for r in range(G)]
        assert max(q.best_key for q in parts) == full.best_key
        assert sum(q.feasible for q in parts) == full.feasible
        assert sum(q.evaluated for q in parts) == T
        assert sum(q.hash for q in parts) % 2**64 == full.hash


def test_shell_sweep_matches_full_sweep_and_counts():
    """orc_sweep_shell (only sum_n >= s_min) against the full sweep: it
    evaluates exactly the sum-n polynomial's tail, and its max keys are the
    full sweep's whenever those lie in the shell, else 0 (nothing above them
    is in the shell)."""
    p = synth.raw_weights(5)
    rng = np.random.default_rng(11)
    for grid in synth.tiny_grids(30, seed=12, kmax=4, max_len=7):
        _, y, _, _ = oracle.sweep(p, grid, 0.0, want_y=True)
        H = float(np.quantile(y, rng.uniform(0.1, 0.9)))
        full, _, _, _ = oracle.sweep(p, grid, H, eps=1e-2)
        poly = sum_n_polynomial(grid)
        for s_min in sorted({0, 1, len(poly) // 2, len(poly) - 1, int(rng.integers(0, len(poly)))}):
            sh = oracle.sweep_shell(p, grid, H, s_min, eps=1e-2)
            assert sh.evaluated == sum(poly[s_min:])
            for name in ("best_key", "maxkey_strict", "maxkey_loose"):
                kf = getattr(full, name)
                want = kf if kf and (kf >> 40) - 1 >= s_min else 0
                assert getattr(sh, name) == want, (name, s_min)


def test_linear_predictor_knapsack_closed_form():
    """Linear ReLU-transparent predictor: the max-Sigma-n feasible group is a
    unit-value knapsack (cheapest slot positions first) and t* the greedy
    lexicographic maximum; the oracle must reach exactly that."""
    rng = np.random.default_rng(11)
    for trial in range(25):
        lp = LinearPredictor(8, 4, c0=2.0, beta=[float(rng.integers(0, 16)) / 4 for _ in range(8)],
                             a=[float(rng.integers(0, 8)) / 8 for _ in range(4)])
        p = lp.params()
        grid = synth.tiny_grids(1, seed=100 + trial, kmax=4, max_len=12)[0]
        r, y, _, ope = oracle.sweep(p, grid, 0.0, want_y=True, want_ope=True)
        for yi, o in zip(y[:50], ope[:50]):
            assert yi == lp.predict(grid, o)
        H = float(np.quantile(y, 0.4))
        r, _, _, _ = oracle.sweep(p, grid, H)
        nstar, tstar = lp.best(grid, H)
        assert r.best_sum_n == nstar and r.best_index == tstar


# --------------------------------------------------------- decisions --------
def test_search_invariants():
    """y(t*) <= H; key_GRID >= key_CHAIN; query order does not matter; AUTO rule;
    DROP iff the critical query alone does not fit."""
    p = synth.raw_weights(5, latency_shaped=True)
    rng = np.random.default_rng(2)
    for _ in range(30):
        k = int(rng.integers(1, 4))
        ms = rng.choice([1, 5, 6], size=k, replace=False)
        qs = [synth.Query(int(m), int(rng.integers(max(1, synth.L(int(m)) - 20), synth.L(int(m)) + 1)),
                          int(rng.choice([1, 8, 32])), 0, float(rng.uniform(0, 60)),
                          float(rng.uniform(0, 10))) for m in ms]
        now, infl = 12.0, float(rng.uniform(0, 3))
        g = oracle.search(p, qs, now, infl, space=0)
        c = oracle.search(p, qs, now, infl, space=1)
        assert g.headroom_ms == c.headroom_ms
        assert g.pred_critical_only_ms == c.pred_critical_only_ms
        assert (g.status == 1) == (not g.pred_critical_only_ms <= g.headroom_ms)
        if g.status == 0:
            assert g.pred_ms <= g.headroom_ms and g.key >= c.key and g.total_ops >= c.total_ops
        perm = list(rng.permutation(k))
        gp = oracle.search(p, [qs[i] for i in perm], now, infl, space=0)
        assert gp.key == g.key and gp.status == g.status
        assert {qs[perm[i]].model_id: gp.end_op[i] for i in range(k)} == \
               {qs[i].model_id: g.end_op[i] for i in range(k)}
        T = g.evaluated
        a1 = oracle.search(p, qs, now, infl, space=2, budget=T)
        a2 = oracle.search(p, qs, now, infl, space=2, budget=T - 1)
        assert a1.space_used == 0 and a2.space_used == 1


def test_fit_is_against_the_fp32_headroom():
    """Reading c11: the fit test compares y with the fp32 headroom both sides
    use, H = (float)h_c.  Constant predictor y = 1 exactly (unit 0 = bias 1,
    passed through): h_c = 1 - 2^-30 rounds to H = 1.0 in fp32, so the
    critical query fits (y <= H, inclusive); h_c = 1 - 2^-23 is an fp32 value
    below 1, so it is dropped."""
    d = 8 + 4 * 4
    p = unit0_params(d, 1.0, {})
    q = synth.Query(5, 1, 1, 0, 1.0 - 2.0 ** -30, 0.0)
    r = oracle.search(p, [q], 0.0, 0.0, space=0)
    assert r.h[0] == 1.0 - 2.0 ** -30 and r.headroom_ms == 1.0
    assert r.pred_critical_only_ms == 1.0 and r.status == 0 and r.pred_ms == 1.0
    q = synth.Query(5, 1, 1, 0, 1.0 - 2.0 ** -23, 0.0)
    r = oracle.search(p, [q], 0.0, 0.0, space=0)
    assert r.headroom_ms == 1.0 - 2.0 ** -23 and r.status == 1


def test_acceptance_window_is_relative():
    """Reading c18: the acceptance window is y <= H -/+ eps |H| (relative).
    Constant predictor y = 16 exactly: with H = 16 (1 + eps/2) every candidate
    fits but none fits the strict window, so maxkey_strict = 0 and
    maxkey_loose = best_key = the brute-force maximum key; with
    H = 16 (1 - eps/2) nothing fits, only the loose window holds every
    candidate."""
    d = 8 + 4 * 4
    p = unit0_params(d, 16.0, {})
    eps = 1e-2
    for grid in synth.tiny_grids(6, seed=91, max_len=5):
        top = max(((brute.sum_n(grid, o) + 1) << 40) | t for t, o in enumerate(brute.enumerate_grid(grid)))
        r, _, _, _ = oracle.sweep(p, grid, 16.0 * (1 + eps / 2), eps=eps)
        assert r.best_key == top and r.maxkey_loose == top and r.maxkey_strict == 0
        r, _, _, _ = oracle.sweep(p, grid, 16.0 * (1 - eps / 2), eps=eps)
        assert r.best_key == 0 and r.maxkey_strict == 0 and r.maxkey_loose == top


# ------------------------------------------------------- multi-way search ---
def test_fig12_multiway_two_predictions():
    """3-way search -- first between queries, then among q1's ops;
    'After two predictions, the query controller completes the exploration'."""
    f, p, qs = _fig12_setup()
    m = oracle.search_mway(p, qs, 0.0, 0.0, ways=3, n_models=3, kmax=3, ops_per_model=f["ops_per_model"])
    names = [q["name"] for q in f["queries"]]
    assert m.status == 0 and m.rounds == 2
    assert m.u == f["expected"]["chain_u"] and m.pred_ms == 25.0
    assert {names[i]: m.end_op[i] for i in range(3)} == f["expected"]["end_op"]


def test_multiway_equals_exhaustive_chain_under_monotone_predictor():
    """With a predictor monotone along the chain (non-negative linear, ReLU-
    transparent), the m-way search finds the exhaustive CHAIN optimum for every
    m, in about log_{m+1} steps."""
    rng = np.random.default_rng(21)
    for trial in range(40):
        lp = LinearPredictor(8, 4, c0=2.0, beta=[float(rng.integers(0, 16)) / 4 for _ in range(8)],
                             a=[float(rng.integers(1, 8)) / 8 for _ in range(4)])
        p = lp.params()
        k = int(rng.integers(1, 5))
        ms = rng.choice(np.arange(1, 9), size=k, replace=False)
        qs = [synth.Query(int(m), int(rng.integers(1, synth.L(int(m)) + 1)), 8, 0,
                          float(rng.uniform(5, 200)), 0.0) for m in ms]
        ex = oracle.search(p, qs, 0.0, 0.0, space=1)
        for ways in (1, 2, 3, 4, 8, 15):
            mw = oracle.search_mway(p, qs, 0.0, 0.0, ways)
            assert mw.status == ex.status
            if ex.status == 0:
                assert mw.u == ex.index and list(mw.end_op)[:k] == list(ex.end_op)[:k]
                R = max(1, ex.evaluated)
                assert mw.rounds <= 2 + int(np.ceil(np.log(R) / np.log(ways + 1)))


# ------------------------------------------------- hash primitives ----
def test_splitmix64_known_answers():
    """SplitMix64 (Steele, Lea, Flood 2014; Vigna's reference generator) seeded
    at 0: the state advances by the golden gamma 0x9E3779B97F4A7C15 and the
    first three outputs are the published 0xE220A8397B1DCDAF,
    0x6E789E6AA1B965F4, 0x06C45D188009454F.  orc_splitmix64(z) is one output
    from state z (the gamma is added inside)."""
    g = 0x9E3779B97F4A7C15
    assert oracle.splitmix64(0) == 0xE220A8397B1DCDAF
    assert oracle.splitmix64(g) == 0x6E789E6AA1B965F4
    assert oracle.splitmix64((2 * g) % 2**64) == 0x06C45D188009454F


def test_fnv1a64_known_answers():
    """FNV-1a 64 (Fowler/Noll/Vo): the empty input gives the offset basis
    0xcbf29ce484222325 and "foobar" the published 0x85944171f73967e8.  The
    oracle hashes int16 feature values as little-endian bytes, so "foobar" is
    the three int16 words 'fo' 'ob' 'ar'."""
    assert oracle.fnv1a64(np.array([], dtype=np.int16)) == 0xCBF29CE484222325
    words = np.frombuffer(b"foobar", dtype="<i2")
    assert oracle.fnv1a64(words) == 0x85944171F73967E8
    # byte order matters: the big-endian reading is a different string
    assert oracle.fnv1a64(np.frombuffer(b"offbra", dtype="<i2")) != 0x85944171F73967E8


def test_sweep_hash_is_the_sum_over_brute_force_rows():
    """The sweep's determinism hash = sum_t splitmix64(t xor fnv1a64(x(t))) mod
    2^64 over brute-force enumerated Fig.-8 rows (both primitives pinned above)."""
    p = synth.raw_weights(2)
    grid = [synth.GridSlot(2, 3, 4, 0, 3, 9, 1), synth.GridSlot(7, 1, 8, 64, 2, 6, 0)]
    r, _, x, _ = oracle.sweep(p, grid, 0.0, want_x=True)
    cands = brute.enumerate_grid(grid)
    assert len(cands) == len(x)
    h = 0
    for t in range(len(x)):
        h = (h + oracle.splitmix64(t ^ oracle.fnv1a64(x[t]))) % 2**64
    assert r.hash == h


# ------------------------------------------------ reading r2: why fp16, not plain bf16 ----
def test_reading_r2_plain_bf16_misses_the_bar_on_config5():
    """DESIGN.md reading r2: with plain bf16 (weights and post-ReLU activations
    rounded RNE to bf16, fp64 accumulation: flags 1 | 8 of the emulation; the
    integer features < 256 are exact and the larger ones round too with flag
    4) the config-5 predictions miss the north star's 1e-2 relative bar
    against the fp64 oracle (max 1.06e-2 / 1.08e-2 here), which is why the
    tensor path uses fp16 operands (or split bf16 weights).  5e4
    instance-based samples (Fig. 9)."""
    params = synth.weights(1)
    G = synth.instance_samples(50_000, seed=15)
    X = oracle.encode_groups(8, 4, [g.slots for g in G])
    y64 = oracle.mlp64_batch(params, X)
    for flags in (1 | 8, 15):
        ye = oracle.mlp64_emu_batch(params, X, flags=flags)
        err = np.abs(ye - y64) / np.abs(y64)
        assert err.max() > 1e-2, (flags, err.max())
    # the weights alone (flags 1 | 2) already cost more than half the bar
    ye = oracle.mlp64_emu_batch(params, X, flags=3)
    assert (np.abs(ye - y64) / np.abs(y64)).max() > 5e-3


def test_bf16_emulation_against_torch_rounding():
    """orc_mlp64_emu pinned beyond single rounding points: flags 1 (weights),
    2 (biases), 1|2 and 4 (features) equal the plain fp64 MLP evaluated on operands
    pre-rounded by torch's own fp32 -> bf16 conversion (RNE), bit for bit; with
    flag 8 (activations) a float64 numpy forward that rounds each post-ReLU
    activation through torch bf16 agrees to fp64 rounding noise."""
    torch = pytest.importorskip("torch")
    params = synth.weights(1)
    G = synth.instance_samples(3000, seed=5)
    X = oracle.encode_groups(8, 4, [g.slots for g in G])
    pr = torch.from_numpy(params.astype(np.float32)).to(torch.bfloat16).float().numpy()
    assert np.array_equal(oracle.mlp64_emu_batch(params, X, flags=3), oracle.mlp64_batch(pr, X))
    # flag 1 rounds the weights only, flag 2 the biases only
    o = offsets(24)
    bias = np.zeros(params.size, dtype=bool)
    for name, n in (("b1", 32), ("b2", 32), ("b3", 32), ("b4", 1)):
        bias[o[name]:o[name] + n] = True
    pw = np.where(bias, params, pr).astype(np.float32)
    pb = np.where(bias, pr, params).astype(np.float32)
    assert not np.array_equal(pw, params) and not np.array_equal(pb, params)
    assert np.array_equal(oracle.mlp64_emu_batch(params, X, flags=1), oracle.mlp64_batch(pw, X))
    assert np.array_equal(oracle.mlp64_emu_batch(params, X, flags=2), oracle.mlp64_batch(pb, X))
    Xr = torch.from_numpy(X.astype(np.float32)).to(torch.bfloat16).float().numpy().astype(np.int16)
    assert not np.array_equal(Xr, X)  # some features (>= 256) do round
    assert np.array_equal(oracle.mlp64_emu_batch(params, X, flags=4), oracle.mlp64_batch(params, Xr))
    W1, b1, W2, b2, W3, b3, w4, b4 = [a.astype(np.float64) for a in synth.split_params(params)]

    def rb(a):  # fp64 -> bf16 via torch (the fp32 step is exact for these magnitudes up to 2^-24 rel)
        return torch.from_numpy(a).to(torch.float32).to(torch.bfloat16).to(torch.float64).numpy()
    h = rb(np.maximum(X.astype(np.float64) @ W1.T + b1, 0))
    h = rb(np.maximum(h @ W2.T + b2, 0))
    h = rb(np.maximum(h @ W3.T + b3, 0))
    y = h @ w4 + b4[0]
    ye = oracle.mlp64_emu_batch(params, X, flags=8)
    d = np.abs(ye - y) / np.abs(y)
    assert np.quantile(d, 0.99) <= 1e-12   # same roundings
    assert d.max() <= 2 ** -7              # a rare tie flipped by fp64 summation order moves one activation by 1 ulp


# ------------------------------------------ NEXT-4: bs / seqlen as swept dims ----
def test_whatif_vs_bruteforce_exact():
    """The what-if sweep (bs and seqlen per slot as an outer variant digit,
    P:513-520) against brute force: itertools over (variant, end ops), the
    brute Fig.-8 encoder with the variant's bs / seqlen, exact rational MLP,
    direct scan for max (sum_n, v T + t) under H."""
    rng = np.random.default_rng(41)
    p = synth.raw_weights(4)
    for trial in range(6):
        grid = synth.tiny_grids(1, seed=300 + trial, max_len=4)[0]
        k = len(grid)
        nv = int(rng.integers(1, 4))
        variants = [([int(rng.integers(1, 33)) for _ in range(k)],
                     [int(rng.choice([0, 16, 128, 512])) for _ in range(k)]) for _ in range(nv)]
        T = oracle.grid_size(grid)
        cands = brute.enumerate_grid(grid)
        ys, meta = [], []
        for v, (bss, sls) in enumerate(variants):
            for t, opes in enumerate(cands):
                pres = [(s.model_id, s.start_op, e, bss[j], sls[j]) for j, (s, e) in enumerate(zip(grid, opes)) if e]
                ys.append(brute.mlp_exact(p, brute.encode(8, 4, pres), synth.D))
                meta.append((v, t, brute.sum_n(grid, opes)))
        sy = sorted(ys)
        m = len(sy) // 2
        H = Fraction(float((sy[m] + (sy[m + 1] if m + 1 < len(sy) else sy[m] + 1)) / 2))  # between values: no tie
        best = (-1, -1, -1)
        for (v, t, sn), y in zip(meta, ys):
            if y <= H and (sn, v * T + t) > (best[2], best[0] * T + best[1] if best[0] >= 0 else -1):
                best = (v, t, sn)
        per, (key, bv, bt), _ = oracle.whatif(p, grid, variants, float(H))
        assert (bv, bt) == best[:2], (trial, (bv, bt), best)
        assert key == ((best[2] + 1) << 40) | (best[0] * T + best[1])
        for v in range(nv):  # per variant: the plain grid scan of that variant
            yv = ys[v * T:(v + 1) * T]
            tv, sv = brute.best_by_scan(cands, grid, yv, H)
            assert (per[v].best_index if per[v].best_key else -1) == tv


def test_whatif_larger_batch_never_fits_more_under_monotone_predictor():
    """With a predictor increasing in every slot's bs (linear, non-negative
    coefficients, ReLU-transparent), the largest fitting group of a variant can
    only shrink as the batch sizes grow."""
    lp = LinearPredictor(8, 4, c0=2.0, beta=[0.5] * 8, a=[0.25, 0.125, 0.5, 0.75])
    p = lp.params()
    o = offsets(synth.D)
    for q in range(4):  # bs coefficient of slot position q
        p[o["W1"] + 0 * synth.D + 8 + 4 * q + 2] = 0.0625
    grid = [synth.GridSlot(1, 1, 1, 0, 1, 60, 1), synth.GridSlot(5, 1, 1, 0, 1, 40, 1)]
    variants = [([b, b], [0, 0]) for b in (1, 2, 4, 8, 16, 32)]
    per, _, _ = oracle.whatif(p, grid, variants, 20.0)
    sns = [(r.best_key >> 40) if r.best_key else 0 for r in per]
    assert all(a >= b for a, b in zip(sns, sns[1:])) and sns[0] > sns[-1], sns
