"""ORACLE (test infrastructure only): fp64 MLP forward / backward / SGD.

Follows PAPER.md §III:
  * Eq. (1) [L43]: L^{l+1} = F_l(W^l L^l); F = sigmoid on hidden layers and
    softmax on the output layer [L258 "The sigmoid function is used as
    activation in the hidden layers. Softmax activation is applied to the
    output layer in order to compute the cross-entropy loss."].
  * Eq. (2) [L49]: gradient by the chain rule from the loss back to W^1.
  * Eq. (3) [L53]: W^l <- W^l - eta * g^l.
  * Mini-batch [L55–L56]: the gradient of a batch of B examples; the loss is
    the batch MEAN of the per-example cross-entropy (reading R10).
  * Bias terms b_l are included (reading R9).

Notation: params = [(W_1, b_1), ..., (W_L, b_L)], W_l has shape
[n_l, n_{l-1}] (the paper's W^l in R^{d_{l+1} x d_l}, [L41]), X is [b, n_0],
labels y are integers in [0, C).  Everything is float64.
"""
from __future__ import annotations

import numpy as np


def sigmoid(z):
    """sigma(z) = 1 / (1 + exp(-z)), evaluated without overflow in fp64."""
    z = np.asarray(z, dtype=np.float64)
    out = np.empty_like(z)
    pos = z >= 0
    out[pos] = 1.0 / (1.0 + np.exp(-z[pos]))
    ez = np.exp(z[~pos])
    out[~pos] = ez / (1.0 + ez)
    return out


def forward(params, X):
    """Eq. (1): returns (Z, H) with Z[l] the pre-activation of layer l+1 and
    H[l] its input (H[0] = X); Z[-1] are the output logits."""
    H = [np.asarray(X, dtype=np.float64)]
    Z = []
    L = len(params)
    for l, (W, b) in enumerate(params):
        z = H[-1] @ np.asarray(W, np.float64).T + np.asarray(b, np.float64)
        Z.append(z)
        if l < L - 1:
            H.append(sigmoid(z))
    return Z, H


def log_softmax(logits):
    """Row-wise log softmax: z - logsumexp(z) (max-shifted)."""
    m = logits.max(axis=1, keepdims=True)
    lse = m + np.log(np.exp(logits - m).sum(axis=1, keepdims=True))
    return logits - lse


def xent_rows(logits, y):
    """Per-example cross-entropy  -log softmax(z_i)[y_i]  [L258]."""
    y = np.asarray(y)
    return -log_softmax(logits)[np.arange(len(y)), y]


def loss(params, X, y):
    """Batch-mean cross-entropy of the MLP on (X, y)."""
    Z, _ = forward(params, X)
    return float(xent_rows(Z[-1], y).mean())


def grads(params, X, y):
    """Eq. (2): gradients of the batch-mean loss.

    Returns (dW, db, loss) with dW[l] shaped like W_l.  Written out:
      dZ_L = (softmax(Z_L) - onehot(y)) / b
      dW_l = dZ_l^T H_{l-1},  db_l = 1^T dZ_l
      dZ_{l-1} = (dZ_l W_l) * sigma'(Z_{l-1}),  sigma' = sigma (1 - sigma)
    """
    y = np.asarray(y)
    Z, H = forward(params, X)
    b = len(y)
    P = np.exp(log_softmax(Z[-1]))
    Y1 = np.zeros_like(P)
    Y1[np.arange(b), y] = 1.0
    dZ = (P - Y1) / b
    L = len(params)
    dW = [None] * L
    db = [None] * L
    for l in range(L - 1, -1, -1):
        dW[l] = dZ.T @ H[l]
        db[l] = dZ.sum(axis=0)
        if l > 0:
            Hl = H[l]
            dZ = (dZ @ np.asarray(params[l][0], np.float64)) * Hl * (1.0 - Hl)
    return dW, db, float(xent_rows(Z[-1], y).mean())


def sgd_step(params, X, y, lr):
    """Eq. (3) applied to every layer with the batch gradient; returns
    (new_params, batch_loss_before_update)."""
    dW, db, ls = grads(params, X, y)
    new = [(np.asarray(W, np.float64) - lr * dW[l], np.asarray(b, np.float64) - lr * db[l])
           for l, (W, b) in enumerate(params)]
    return new, ls


def full_loss(params, X, y, chunk: int = 65536):
    """Mean cross-entropy over the whole dataset (epoch-end loss, [L273])."""
    tot = 0.0
    n = len(y)
    for s in range(0, n, chunk):
        Z, _ = forward(params, X[s:s + chunk])
        tot += xent_rows(Z[-1], y[s:s + chunk]).sum()
    return tot / n


def flops_per_sample(dims) -> int:
    """Algorithmic FLOPs per example of one SGD step:
    forward 2P, dX 2(P - n0 n1) (no input gradient for layer 1), dW 2P."""
    P = sum(dims[l] * dims[l - 1] for l in range(1, len(dims)))
    return 6 * P - 2 * dims[0] * dims[1]
