"""Pins for oracle/mlp64.py against things other than itself (CPU only).

Each test names the paper passage it checks and what independent fact pins it:
library routines (scipy, sklearn), closed forms, central finite differences,
brute force, and the hand-derived worked step in tests/golden/d1_step.json.
"""
import json
import os

import numpy as np
import pytest
from scipy.special import expit, softmax
from sklearn.metrics import log_loss

from oracle import mlp64

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _rand_params(dims, rng, scale=1.0):
    return [(rng.standard_normal((dims[l], dims[l - 1])) * scale / np.sqrt(dims[l - 1]),
             rng.standard_normal(dims[l]) * 0.1) for l in range(1, len(dims))]


def test_sigmoid_matches_scipy_expit():
    # hidden activation F_l = sigmoid [L258]
    z = np.concatenate([np.linspace(-800, 800, 4001), [-1e-300, 0.0, 1e-300]])
    np.testing.assert_allclose(mlp64.sigmoid(z), expit(z), rtol=1e-15, atol=1e-300)


def test_single_layer_loss_is_sklearn_log_loss():
    # L = 1 reduces to multinomial logistic regression; the loss is the mean
    # cross-entropy of the softmax output [L258] = sklearn's log_loss.
    rng = np.random.default_rng(11)
    X = rng.standard_normal((37, 9))
    y = rng.integers(0, 5, 37)
    params = _rand_params([9, 5], rng, scale=2.0)
    W, b = params[0]
    P = softmax(X @ W.T + b, axis=1)
    assert abs(mlp64.loss(params, X, y) - log_loss(y, P, labels=range(5))) < 1e-12


def test_single_layer_gradient_textbook():
    # multinomial logistic regression gradient (textbook): X^T (P - Y) / b
    rng = np.random.default_rng(12)
    X = rng.standard_normal((23, 6))
    y = rng.integers(0, 4, 23)
    params = _rand_params([6, 4], rng)
    W, b = params[0]
    P = softmax(X @ W.T + b, axis=1)
    Y = np.eye(4)[y]
    dW, db, _ = mlp64.grads(params, X, y)
    np.testing.assert_allclose(dW[0], (P - Y).T @ X / 23, rtol=1e-12, atol=1e-15)
    np.testing.assert_allclose(db[0], (P - Y).sum(0) / 23, rtol=1e-12, atol=1e-15)


def test_zero_weight_closed_form():
    # All weights and biases 0: logits 0 -> loss = ln C; dZ_L = (1/C - onehot)/b;
    # hidden H = 1/2 so dW_L[c,:] = (1/C - n_c/b)/2 and db_L[c] = 1/C - n_c/b;
    # dZ_{L-1} = dZ_L W_L = 0, so every lower-layer gradient is exactly 0.
    dims = [5, 4, 3, 3]
    params = [(np.zeros((dims[l], dims[l - 1])), np.zeros(dims[l])) for l in range(1, 4)]
    X = np.random.default_rng(0).standard_normal((6, 5))
    y = np.array([0, 1, 1, 2, 2, 2])
    dW, db, ls = mlp64.grads(params, X, y)
    assert abs(ls - np.log(3)) < 1e-15
    n = np.bincount(y, minlength=3)
    np.testing.assert_allclose(db[2], 1 / 3 - n / 6, atol=1e-16)
    np.testing.assert_allclose(dW[2], np.repeat(((1 / 3 - n / 6) / 2)[:, None], 3, 1), atol=1e-16)
    for l in (0, 1):
        assert np.all(dW[l] == 0) and np.all(db[l] == 0)


@pytest.mark.parametrize("dims,b", [([5, 4, 3, 3], 4), ([7, 6, 5, 4, 3], 3), ([3, 2], 2),
                                    ([54, 8, 8, 7], 4)])
def test_gradients_match_central_finite_differences(dims, b):
    # Eq. (2) [L49]: back-propagation must equal the derivative of the loss.
    rng = np.random.default_rng(sum(dims) + b)
    params = _rand_params(dims, rng, scale=1.5)
    X = rng.standard_normal((b, dims[0]))
    y = rng.integers(0, dims[-1], b)
    dW, db, _ = mlp64.grads(params, X, y)
    h = 1e-6
    worst = 0.0
    for l in range(len(params)):
        W, bb = params[l]
        # sample at most 40 weight entries per layer (all of them on tiny nets)
        idx = [(i, j) for i in range(W.shape[0]) for j in range(W.shape[1])]
        if len(idx) > 40:
            idx = [idx[k] for k in rng.choice(len(idx), 40, replace=False)]
        for (i, j) in idx:
            def f(delta):
                P = [(w.copy(), c.copy()) for w, c in params]
                P[l][0][i, j] += delta
                return mlp64.loss(P, X, y)
            fd = (f(h) - f(-h)) / (2 * h)
            worst = max(worst, abs(fd - dW[l][i, j]) / max(1e-8, abs(fd) + abs(dW[l][i, j])))
        for i in range(len(bb)):
            def g(delta):
                P = [(w.copy(), c.copy()) for w, c in params]
                P[l][1][i] += delta
                return mlp64.loss(P, X, y)
            fd = (g(h) - g(-h)) / (2 * h)
            worst = max(worst, abs(fd - db[l][i]) / max(1e-8, abs(fd) + abs(db[l][i])))
    assert worst < 1e-6, worst


def test_batch_gradient_is_mean_of_per_example_gradients():
    # mini-batch SGD [L55–L56]: the batch gradient is the mean over its examples
    rng = np.random.default_rng(5)
    dims = [6, 5, 4, 3]
    params = _rand_params(dims, rng)
    X = rng.standard_normal((9, 6))
    y = rng.integers(0, 3, 9)
    dW, db, ls = mlp64.grads(params, X, y)
    acc_W = [np.zeros_like(w) for w, _ in params]
    acc_b = [np.zeros_like(c) for _, c in params]
    acc_l = 0.0
    for i in range(9):
        gW, gb, li = mlp64.grads(params, X[i:i + 1], y[i:i + 1])
        for l in range(3):
            acc_W[l] += gW[l] / 9
            acc_b[l] += gb[l] / 9
        acc_l += li / 9
    for l in range(3):
        np.testing.assert_allclose(dW[l], acc_W[l], rtol=1e-12, atol=1e-16)
        np.testing.assert_allclose(db[l], acc_b[l], rtol=1e-12, atol=1e-16)
    assert abs(ls - acc_l) < 1e-14


def test_hand_derived_2_2_2_step():
    # SURVEY.md Appendix D1, hand-derived from Eq. (1)-(3) [L43, L49, L53]
    g = json.load(open(os.path.join(GOLD, "d1_step.json")))
    params = [(np.array(g["W1"]), np.array(g["b1"])), (np.array(g["W2"]), np.array(g["b2"]))]
    X = np.array([g["x"]])
    y = np.array([g["y"]])
    Z, H = mlp64.forward(params, X)
    np.testing.assert_allclose(Z[0][0], g["z1"], atol=1e-12)
    np.testing.assert_allclose(H[1][0], g["h"], atol=1e-12)
    np.testing.assert_allclose(Z[1][0], g["z2"], atol=1e-12)
    np.testing.assert_allclose(np.exp(mlp64.log_softmax(Z[1]))[0], g["p"], atol=1e-12)
    dW, db, ls = mlp64.grads(params, X, y)
    assert abs(ls - g["loss"]) < 1e-12
    np.testing.assert_allclose(db[1], g["db2"], atol=1e-12)
    np.testing.assert_allclose(dW[1], g["dW2"], atol=1e-12)
    np.testing.assert_allclose(db[0], g["db1"], atol=1e-12)
    np.testing.assert_allclose(dW[0], g["dW1"], atol=1e-12)
    new, ls2 = mlp64.sgd_step(params, X, y, g["lr"])
    assert ls2 == ls
    np.testing.assert_allclose(new[0][0], g["W1_after"], atol=1e-12)
    np.testing.assert_allclose(new[1][0], g["W2_after"], atol=1e-12)


def test_softmax_gradient_rows_sum_to_zero_and_probabilities_sum_to_one():
    rng = np.random.default_rng(3)
    dims = [4, 7]
    params = _rand_params(dims, rng, scale=3)
    X = rng.standard_normal((11, 4))
    y = rng.integers(0, 7, 11)
    dW, db, _ = mlp64.grads(params, X, y)
    # db = 1^T dZ and each row of dZ sums to 0 -> sum(db) == 0
    assert abs(db[0].sum()) < 1e-15
    Z, _ = mlp64.forward(params, X)
    np.testing.assert_allclose(np.exp(mlp64.log_softmax(Z[-1])).sum(1), 1.0, atol=1e-15)


def test_loss_is_stable_for_huge_logits():
    # max-shifted log-sum-exp: no overflow at |z| ~ 1e4
    params = [(np.array([[1e4], [-1e4], [0.0]]), np.zeros(3))]
    X = np.array([[1.0], [-1.0]])
    y = np.array([0, 0])
    Z, _ = mlp64.forward(params, X)
    rows = mlp64.xent_rows(Z[-1], y)
    assert rows[0] == 0.0 and abs(rows[1] - 2e4) < 1e-9


def test_full_loss_equals_batch_loss():
    rng = np.random.default_rng(8)
    params = _rand_params([5, 6, 3], rng)
    X = rng.standard_normal((100, 5))
    y = rng.integers(0, 3, 100)
    assert abs(mlp64.full_loss(params, X, y, chunk=7) - mlp64.loss(params, X, y)) < 1e-14


@pytest.mark.parametrize("dims", [[54, 64, 64, 7], [54, 512, 512, 512, 512, 7],
                                  [300, 1024, 1024, 1024, 2], [20958] + [4096] * 4 + [2]])
def test_flops_per_sample_brute_force(dims):
    # count multiply-adds layer by layer: forward GEMM, input-gradient GEMM (not for
    # layer 1) and weight-gradient GEMM, 2 flops each
    f = 0
    for l in range(1, len(dims)):
        mac = dims[l] * dims[l - 1]
        f += 2 * mac              # forward
        f += 2 * mac              # dW
        if l > 1:
            f += 2 * mac          # dX
    assert mlp64.flops_per_sample(dims) == f


def test_c2_trajectory_golden_is_the_oracle_s():
    # tests/golden/c2_trajectory.json (scripts/make_goldens.py) pinned to the oracle: the first
    # two steps of the stored 100-step C2 trajectory are recomputed here
    import json
    import os
    import sys
    sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "scripts"))
    import make_goldens
    gold = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "c2_trajectory.json")))
    assert len(gold["losses"]) == gold["steps"] == 100
    got = make_goldens.c2_trajectory(steps=2)
    np.testing.assert_allclose(got, gold["losses"][:2], rtol=1e-12)
