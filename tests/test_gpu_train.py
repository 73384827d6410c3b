"""NEXT-3 on the GPU: abacus_train_* against the fp64 training oracle
(oracle/train.py, pinned in tests/test_oracle_train.py).

Bars: the minibatch gradient within 1e-4 of the gradient's scale (fp32
accumulation over the batch vs fp64), the Adam update exact to fp32 rounding
given the same gradient, a 30-step trajectory's losses within 1e-3."""
import numpy as np
import pytest
import torch

import oracle
import synth
from oracle import train as T
import paper_conf_sc_cui0czlzsmylg21_b200 as ab
from gpu_util import Ctx, stream

pytestmark = pytest.mark.gpu
D = synth.D
NP = synth.n_params()


def _data(n, seed):
    G = synth.instance_samples(n, seed=seed)
    X = oracle.encode_groups(synth.N_MODELS, synth.K_MAX, [g.slots for g in G])
    return X, synth.group_latency_ms(G, seed=seed)


def _dev(X, t):
    return (torch.from_numpy(np.ascontiguousarray(X, dtype=np.int16)).cuda(),
            torch.from_numpy(np.ascontiguousarray(t, dtype=np.float32)).cuda())


@pytest.mark.parametrize("n", [1, 77, 300, 4096])
def test_gradient_and_loss_match_oracle(n):
    X, t = _data(n, seed=40 + n)
    t32 = t.astype(np.float32).astype(np.float64)
    p0 = synth.raw_weights(1, latency_shaped=False)
    c = Ctx()
    try:
        ab.abacus_train_begin(c.h, p0)
        dx, dt = _dev(X, t)
        g = torch.zeros(NP, dtype=torch.float32, device="cuda")
        ab.abacus_train_step(c.h, dx, dt, n, 0.0, g, stream())
        p1, loss = ab.abacus_train_params(c.h, NP)
        L64, G64 = T.grad(p0, X, t32, D)
        G = g.cpu().numpy().astype(np.float64)
        assert np.array_equal(p1, p0.astype(np.float32))          # lr = 0: unchanged
        assert abs(loss - L64) <= 1e-5 * abs(L64)
        assert np.abs(G - G64).max() <= 1e-4 * np.abs(G64).max()
        assert np.array_equal(G == 0, G64 == 0)                    # same dead units / absent features
    finally:
        c.close()


def test_adam_step_matches_oracle_given_the_same_gradient():
    X, t = _data(512, seed=7)
    p0 = synth.raw_weights(2, latency_shaped=False)
    c = Ctx()
    try:
        ab.abacus_train_begin(c.h, p0, 0.9, 0.999, 1e-8)
        dx, dt = _dev(X, t)
        opt = T.Adam(NP)
        p_ref = p0.astype(np.float64)
        g = torch.zeros(NP, dtype=torch.float32, device="cuda")
        for step, lr in enumerate([1e-3, 3e-3, 2e-3]):
            # feed the oracle optimiser the GPU's own gradient: isolates Adam
            ab.abacus_train_step(c.h, dx, dt, 512, lr, g, stream())
            torch.cuda.synchronize()
            p_ref = opt.update(p_ref, g.cpu().numpy().astype(np.float64), lr)
            p_gpu, _ = ab.abacus_train_params(c.h, NP)
            assert np.abs(p_gpu - p_ref).max() <= 2e-6, step
            p_ref = p_gpu.astype(np.float64)  # continue from the fp32 state both sides hold
    finally:
        c.close()


def test_thirty_step_trajectory_tracks_oracle():
    X, t = _data(30 * 256, seed=9)
    t32 = t.astype(np.float32).astype(np.float64)
    p0 = synth.raw_weights(1, latency_shaped=False)
    c = Ctx()
    try:
        ab.abacus_train_begin(c.h, p0)
        dx, dt = _dev(X, t)
        losses = torch.zeros(30, dtype=torch.float32, device="cuda")
        ab.abacus_train_epoch(c.h, dx, dt, len(t), 256, 3e-3, losses, stream())
        p_gpu, last = ab.abacus_train_params(c.h, NP)
        p_ref, l_ref = T.train(p0, X, t32, D, batch=256, epochs=1, lr=3e-3)
        lg = losses.cpu().numpy().astype(np.float64)
        assert last == lg[-1]
        assert np.max(np.abs(lg - l_ref) / np.array(l_ref)) <= 1e-3
        assert np.linalg.norm(p_gpu - p_ref) <= 1e-3 * np.linalg.norm(p_ref)
    finally:
        c.close()


def test_trained_predictor_beats_linear_regression_and_serves_the_search():
    X, t = _data(24_000, seed=11)
    Xtr, ttr, Xte, tte = X[:20_000], t[:20_000], X[20_000:], t[20_000:]
    c = Ctx()
    try:
        ab.abacus_train_begin(c.h, synth.raw_weights(1, latency_shaped=False))
        dx, dt = _dev(Xtr, ttr)
        epochs = 40
        for ep in range(epochs):
            lr = 3e-3 * 0.5 * (1 + np.cos(np.pi * ep / epochs))
            ab.abacus_train_epoch(c.h, dx, dt, len(ttr), 256, lr, None, stream())
        p, _ = ab.abacus_train_params(c.h, NP)
        A = np.hstack([Xtr, np.ones((len(Xtr), 1))])
        coef, *_ = np.linalg.lstsq(A, ttr, rcond=None)
        lr_mape = T.mape(np.hstack([Xte, np.ones((len(Xte), 1))]) @ coef, tte)
        # the trained weights, loaded into the search's predictor (fp32 and fp16 paths)
        for prec in (ab.ABACUS_FP32, ab.ABACUS_FP16):
            c.load(p, prec)
            mape = T.mape(c.predict(Xte), tte)
            assert mape < 0.5 * lr_mape and mape < 0.25, (prec, mape, lr_mape)
    finally:
        c.close()


def test_train_errors():
    c = Ctx()
    try:
        with pytest.raises(ab.AbacusError) as e:
            ab.abacus_train_step(c.h, 16, 16, 1, 1e-3)
        assert e.value.code == ab.ABACUS_E_NOT_LOADED
        with pytest.raises(ab.AbacusError):
            ab.abacus_train_begin(c.h, np.zeros(5, dtype=np.float32))
        ab.abacus_train_begin(c.h, synth.raw_weights(1))
        with pytest.raises(ab.AbacusError):
            ab.abacus_train_step(c.h, 16, 16, 0, 1e-3)
        with pytest.raises(ab.AbacusError):
            ab.abacus_train_step(c.h, 16, 16, 1 << 20, 1e-3)
    finally:
        c.close()
