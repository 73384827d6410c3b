"""Pins of the NEXT-3 training oracle (oracle/train.py) against things other
than itself: the C oracle's forward pass (pinned in test_oracle_pins.py),
central finite differences of the loss (the gradient), and the closed form of
Adam under a constant gradient (Kingma & Ba bias correction)."""
import numpy as np

import oracle
import synth
from oracle import train as T

D = synth.D


def _samples(n, seed=3):
    G = synth.instance_samples(n, seed=seed)
    X = oracle.encode_groups(synth.N_MODELS, synth.K_MAX, [g.slots for g in G])
    return X, synth.group_latency_ms(G, seed=seed)


def test_forward_matches_c_oracle():
    X, _ = _samples(64)
    p = synth.raw_weights(2, latency_shaped=False)
    y, _ = T.forward(p, X, D)
    ref = oracle.mlp64_batch(p, X)
    assert np.allclose(y, ref, rtol=1e-12, atol=1e-12)


def test_gradient_matches_central_differences():
    X, t = _samples(6, seed=4)
    p = synth.raw_weights(3, latency_shaped=False).astype(np.float64)
    p[-1] += 40.0  # positive outputs, well away from y = 0
    _, (_, z1, _, z2, _, z3, _) = T.forward(p, X, D)
    assert min(np.abs(z).min() for z in (z1, z2, z3)) > 1e-4  # no ReLU kink within the step
    L0, G = T.grad(p, X, t, D)
    assert np.isclose(L0, T.loss(p, X, t, D), rtol=1e-14)
    h = 1e-6
    fd = np.zeros_like(p)
    for i in range(p.size):
        q = p.copy()
        q[i] += h
        lp = T.loss(q, X, t, D)
        q[i] -= 2 * h
        lm = T.loss(q, X, t, D)
        fd[i] = (lp - lm) / (2 * h)
    scale = np.abs(G).max()
    assert np.abs(fd - G).max() <= 1e-6 * scale
    # every block of the layout is exercised (W1, b1, ..., b4)
    assert np.count_nonzero(G) > 0.5 * G.size


def test_adam_constant_gradient_closed_form():
    """m_t = (1 - b1^t) g and v_t = (1 - b2^t) g^2, so every bias-corrected
    step is lr * g / (|g| + eps): p_T = p_0 - T lr g / (|g| + eps)."""
    rng = np.random.default_rng(1)
    p0 = rng.normal(size=50)
    g = rng.normal(size=50)
    g[:5] = 0.0  # zero gradient: the parameter never moves
    opt = T.Adam(50)
    p = p0.copy()
    for _ in range(7):
        p = opt.update(p, g, 1e-3)
    want = p0 - 7 * 1e-3 * g / (np.abs(g) + 1e-8)
    assert np.allclose(p, want, rtol=0, atol=1e-13)
    assert np.array_equal(p[:5], p0[:5])


def test_training_reduces_the_loss_and_beats_linear_regression():
    X, t = _samples(3000, seed=5)
    Xtr, ttr, Xte, tte = X[:2400], t[:2400], X[2400:], t[2400:]
    p0 = synth.raw_weights(1, latency_shaped=False)
    p, losses = T.train(p0, Xtr, ttr, D, batch=128, epochs=25, lr=3e-3)
    assert np.mean(losses[-10:]) < 0.5 * np.mean(losses[:10])
    A = np.hstack([Xtr, np.ones((len(Xtr), 1))])
    coef, *_ = np.linalg.lstsq(A, ttr, rcond=None)
    lr_mape = T.mape(np.hstack([Xte, np.ones((len(Xte), 1))]) @ coef, tte)
    mlp_mape = T.mape(T.forward(p, Xte, D)[0], tte)
    assert mlp_mape < 0.6 * lr_mape


def test_mape_eq1_hand_values():
    """Eq. 1: error = |predicted - real| / real, averaged.
    Hand values: (2 vs 1) -> 1, (3 vs 4) -> 1/4, (5 vs 5) -> 0; mean 5/12."""
    assert T.mape([2.0], [1.0]) == 1.0
    assert T.mape([3.0], [4.0]) == 0.25
    assert abs(T.mape([2.0, 3.0, 5.0], [1.0, 4.0, 5.0]) - 5.0 / 12.0) < 1e-15
