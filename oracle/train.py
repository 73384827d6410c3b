"""Oracle for NEXT-3 (training the latency predictor on the GPU).  TEST
INFRASTRUCTURE: only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / reference legs may import this module.

The paper fixes the network (D -> 32 -> 32 -> 32 -> 1), the data
(instance-based samples, Fig. 9) and the error metric (MAPE,
Eq. 1) but not the training procedure.  Readings (DESIGN.md
t1-t3):
  t1  loss = mean over the batch of (y_pred / y_true - 1)^2, the smooth
      square of Eq. 1's per-sample error;
  t2  optimiser = Adam (beta1 0.9, beta2 0.999, eps 1e-8, bias-corrected),
      one update per minibatch, learning rate given per step;
  t3  initialisation = PyTorch nn.Linear default (synth.raw_weights).
Everything here is plain fp64 numpy, written from the definitions: forward
pass, the chain rule layer by layer, the Adam recurrences.
"""
from __future__ import annotations

import numpy as np

H = 32


def unpack(p, d):
    """params (W1[32][d] b1 W2[32][32] b2 W3[32][32] b3 w4[32] b4) -> arrays (views, fp64)."""
    p = np.asarray(p, dtype=np.float64)
    o = 0
    out = []
    for shape in [(H, d), (H,), (H, H), (H,), (H, H), (H,), (H,), (1,)]:
        n = int(np.prod(shape))
        out.append(p[o:o + n].reshape(shape))
        o += n
    return out


def forward(p, X, d):
    """P:976-980 with reading c1: ReLU on the three hidden layers, linear output."""
    W1, b1, W2, b2, W3, b3, w4, b4 = unpack(p, d)
    X = np.asarray(X, dtype=np.float64)
    z1 = X @ W1.T + b1
    a1 = np.maximum(z1, 0.0)
    z2 = a1 @ W2.T + b2
    a2 = np.maximum(z2, 0.0)
    z3 = a2 @ W3.T + b3
    a3 = np.maximum(z3, 0.0)
    y = a3 @ w4 + b4[0]
    return y, (X, z1, a1, z2, a2, z3, a3)


def loss(p, X, t, d):
    """Reading t1: mean((y / t - 1)^2)."""
    y, _ = forward(p, X, d)
    r = y / np.asarray(t, dtype=np.float64) - 1.0
    return float(np.mean(r * r))


def grad(p, X, t, d):
    """(loss, dloss/dparams) by the chain rule, in the params layout."""
    W1, b1, W2, b2, W3, b3, w4, b4 = unpack(p, d)
    y, (X, z1, a1, z2, a2, z3, a3) = forward(p, X, d)
    t = np.asarray(t, dtype=np.float64)
    B = len(t)
    r = y / t - 1.0
    g = 2.0 * r / t / B                    # dL/dy per sample
    gw4 = a3.T @ g
    gb4 = np.array([g.sum()])
    d3 = np.outer(g, w4) * (z3 > 0)        # dL/dz3
    gW3 = d3.T @ a2
    gb3 = d3.sum(axis=0)
    d2 = (d3 @ W3) * (z2 > 0)              # dL/dz2
    gW2 = d2.T @ a1
    gb2 = d2.sum(axis=0)
    d1 = (d2 @ W2) * (z1 > 0)              # dL/dz1
    gW1 = d1.T @ X
    gb1 = d1.sum(axis=0)
    G = np.concatenate([gW1.ravel(), gb1, gW2.ravel(), gb2, gW3.ravel(), gb3, gw4, gb4])
    return float(np.mean(r * r)), G


class Adam:
    """Reading t2 (Kingma & Ba): m <- b1 m + (1 - b1) g; v <- b2 v + (1 - b2) g^2;
    p <- p - lr * (m / (1 - b1^t)) / (sqrt(v / (1 - b2^t)) + eps)."""

    def __init__(self, n, beta1=0.9, beta2=0.999, eps=1e-8):
        self.m = np.zeros(n)
        self.v = np.zeros(n)
        self.t = 0
        self.b1, self.b2, self.eps = beta1, beta2, eps

    def update(self, p, g, lr):
        self.t += 1
        self.m = self.b1 * self.m + (1.0 - self.b1) * g
        self.v = self.b2 * self.v + (1.0 - self.b2) * g * g
        mh = self.m / (1.0 - self.b1 ** self.t)
        vh = self.v / (1.0 - self.b2 ** self.t)
        return np.asarray(p, dtype=np.float64) - lr * mh / (np.sqrt(vh) + self.eps)


def train(p, X, t, d, batch, epochs, lr, opt=None):
    """Minibatches in the given order; lr(epoch) or a constant.  Returns (params, per-step losses)."""
    p = np.asarray(p, dtype=np.float64).copy()
    opt = opt or Adam(p.size)
    losses = []
    for ep in range(epochs):
        lre = lr(ep) if callable(lr) else lr
        for s in range(0, len(t), batch):
            L, G = grad(p, X[s:s + batch], t[s:s + batch], d)
            p = opt.update(p, G, lre)
            losses.append(L)
    return p, losses


def mape(y_pred, y_true):
    """Eq. 1, averaged."""
    y_pred = np.asarray(y_pred, dtype=np.float64)
    y_true = np.asarray(y_true, dtype=np.float64)
    return float(np.mean(np.abs(y_pred - y_true) / y_true))
