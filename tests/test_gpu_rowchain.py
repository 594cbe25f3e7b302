"""GPU parity of the fused row-block step (rowchain.cuh) against the fp64 oracle.

The fused kernel computes the forward chain, the softmax cross-entropy head and the whole dX
chain of every 128-row block in one launch (1 or 2 CTAs per block), followed by the dW GEMMs.
These cases are chosen to be eligible (uniform hidden width <= 512, n_0 <= 512, C <= 16) and to
span: one and two CTAs per block, ragged 64-column chunks (n = 40, 200, 300), X wider than
one chunk (n_0 = 300), ragged row blocks, one hidden layer (L = 2), the paper's deep 8-hidden-
layer w8a net, C = 16, and the full C2 batch (b = 8192, 64 row blocks).
Tolerance: BASELINE.json north_star, normwise relative error <= 1e-2 per tensor (bf16).
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import paper_conf_ipps_marws21_b200 as hb  # noqa: E402
from oracle import mlp64  # noqa: E402
from tests.helpers import dataset, grad_errors, init_params, params_to_flat, rel_err, split_flat, to_device  # noqa: E402

TOL = 1e-2


def _need_gpu():
    if not torch.cuda.is_available() or not hb.device_ok(0):
        pytest.fail("no sm_100 GPU visible: the -m gpu tests must run on a B200")


CASES = [
    # dims, dataset kind, batch, expected CTAs per row block (widest of 1/2/4/8 with >= 64
    # columns per CTA whose clusters still fill the 148 SMs in one wave)
    ([54, 64, 64, 7], "covtype", 32, 1),
    ([54, 64, 64, 7], "covtype", 1, 1),
    ([24, 40, 3], "gauss", 77, 1),
    ([54, 128, 128, 7], "covtype", 4096, 2),
    ([54, 512, 512, 7], "covtype", 1000, 8),
    ([54, 200, 200, 200, 7], "covtype", 129, 4),
    ([300, 300, 300, 2], "w8a", 333, 2),
    ([54, 512, 7], "covtype", 256, 8),
    ([300] + [512] * 8 + [2], "w8a", 200, 8),
    ([64, 256, 256, 16], "gauss", 500, 4),
    ([54, 512, 512, 512, 512, 7], "covtype", 4096, 4),
    ([54, 512, 512, 512, 512, 7], "covtype", 8192, 2),
]


@pytest.mark.parametrize("dims,kind,b,cs", CASES)
def test_fused_gradients_match_oracle(dims, kind, b, cs):
    _need_gpu()
    X, y = dataset(kind, b, d=dims[0], seed=11)
    y = (y % dims[-1]).astype(np.int32)
    if dims[-1] > 2:
        y = np.random.default_rng(5).integers(0, dims[-1], b).astype(np.int32)
    m = hb.MLP(dims, precision="bf16", seed=0)
    m.set_fused_min_batch(1)  # exercise the fused kernel at every batch size
    assert m.fused_path(b) == cs
    params = init_params(dims, seed=2)
    m.set_params(params_to_flat(params))
    w = hb.Worker(m, b)
    tX, ty = to_device(X, y)
    g, loss = w.step_grads(tX, ty, b)
    dW, db, l_ref = mlp64.grads(params, X.astype(np.float64), y)
    got = split_flat(g, dims)
    errs = [(l, rel_err(got[l][0], dW[l]), rel_err(got[l][1], db[l])) for l in range(len(dims) - 1)]
    assert max(max(e[1], e[2]) for e in errs) <= TOL, errs
    assert abs(loss - l_ref) / l_ref <= TOL


def test_fused_steps_track_oracle_trajectory():
    # 30 in-place SGD steps on consecutive batches (each step reads the model the previous one
    # wrote): batch losses and the final parameters against the oracle's serial SGD
    _need_gpu()
    dims, b, steps, lr = [54, 512, 512, 7], 512, 30, 0.5
    X, y = dataset("covtype", b * steps, seed=4)
    m = hb.MLP(dims, precision="bf16", seed=0)
    m.set_fused_min_batch(1)
    assert m.fused_path(b) == 8
    params = init_params(dims, seed=2)
    m.set_params(params_to_flat(params))
    w = hb.Worker(m, b)
    tX, ty = to_device(X, y)
    ref = [(W.copy(), c.copy()) for W, c in params]
    for k in range(steps):
        sl = slice(k * b, (k + 1) * b)
        loss = w.step(tX[sl], ty[sl], b, lr, want_loss=True)
        ref, l_ref = mlp64.sgd_step(ref, X[sl].astype(np.float64), y[sl], lr)
        assert abs(loss - l_ref) / l_ref <= TOL, (k, loss, l_ref)
    got = split_flat(m.get_params(), dims)
    for l in range(len(dims) - 1):
        dref = ref[l][0] - params[l][0]
        assert np.linalg.norm(got[l][0] - ref[l][0]) <= TOL * np.linalg.norm(dref) + 1e-6 * np.linalg.norm(ref[l][0])


def test_fused_saturated_init():
    # sigma' near saturation (init x4): S is stashed from fp32 z inside the fused epilogue
    _need_gpu()
    dims, b = [54, 512, 512, 512, 512, 7], 384
    X, y = dataset("covtype", b, seed=8)
    m = hb.MLP(dims, precision="bf16", seed=0)
    m.set_fused_min_batch(1)
    assert m.fused_path(b) > 0
    params = init_params(dims, seed=2, scale=4.0)
    m.set_params(params_to_flat(params))
    w = hb.Worker(m, b)
    tX, ty = to_device(X, y)
    g, _ = w.step_grads(tX, ty, b)
    dW, db, _ = mlp64.grads(params, X.astype(np.float64), y)
    got = split_flat(g, dims)
    for l in range(len(dims) - 1):
        assert rel_err(got[l][0], dW[l]) <= TOL, l
        assert rel_err(got[l][1], db[l]) <= TOL, l


@pytest.mark.parametrize("cs", [1, 2, 4, 8])
def test_every_cluster_size_matches_oracle(cs):
    # the same 256-wide net at every cluster size (HB_OPT_RC_CLUSTER); at CS = 8 the last four CTAs
    # of every cluster own no valid column (n = 256 < 8 x 64 chunks)
    _need_gpu()
    dims, b = [54, 256, 256, 7], 300
    X, y = dataset("covtype", b, seed=13)
    m = hb.MLP(dims, precision="bf16", seed=0)
    m.set_fused_min_batch(1)
    m.set_option("rc_cluster", cs)
    params = init_params(dims, seed=2)
    m.set_params(params_to_flat(params))
    w = hb.Worker(m, b)
    tX, ty = to_device(X, y)
    g, loss = w.step_grads(tX, ty, b)
    dW, db, l_ref = mlp64.grads(params, X.astype(np.float64), y)
    assert m.fused_path(b) == cs
    norm, elem = grad_errors(g, dims, dW, db)
    assert max(norm) <= TOL and max(elem) <= TOL, (norm, elem)
    assert abs(loss - l_ref) / l_ref <= TOL


def test_unfused_shapes_report_layer_chain():
    _need_gpu()
    m = hb.MLP([54, 512, 512, 7])
    assert m.fused_path(8192) == 2 and m.fused_path(4096) == 4   # default crossover b = 4096
    assert m.fused_path(2048) == 0
    m.set_fused_min_batch(0)
    assert m.fused_path(8192) == 0
    assert hb.MLP([54, 1024, 1024, 7]).fused_path() == 0     # n > 512
    assert hb.MLP([54, 128, 64, 7]).fused_path() == 0        # non-uniform hidden widths
    assert hb.MLP([64, 96, 40]).fused_path() == 0            # C > 16
    assert hb.MLP([54, 7]).fused_path() == 0                 # no hidden layer
    assert hb.MLP([54, 64, 7], precision="fp32").fused_path() == 0
