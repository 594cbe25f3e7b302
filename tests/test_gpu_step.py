"""GPU parity: the CUDA path (through the C ABI) against the fp64 oracle.

Tolerances (BASELINE.json north_star, R13): per tensor, the normwise relative error
||g - g_ref|| / ||g_ref|| AND the element-wise error max|g - g_ref| / max|g_ref| are <= 1e-2 for
the bf16 tensor-core path and <= 1e-5 for the fp32 CUDA-core check mode; every row's
cross-entropy is within tol * max(1, max_c |z_ic|) of the oracle's (a dropped or duplicated ragged row
fails the row check and, through its ~1/sqrt(b) share of some dW elements, the element-wise one).
The oracle sees exactly the GPU's inputs: bf16-exact X and fp32-exact parameters, in fp64.
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import paper_conf_ipps_marws21_b200 as hb  # noqa: E402
from oracle import mlp64  # noqa: E402
from tests.helpers import (dataset, grad_errors, init_params, params_to_flat, rel_err, split_flat,  # noqa: E402
                           to_device)

TOL = {"bf16": 1e-2, "fp32": 1e-5}


def _need_gpu():
    if not torch.cuda.is_available() or not hb.device_ok(0):
        pytest.fail("no sm_100 GPU visible: the -m gpu tests must run on a B200")


def make(dims, prec, max_batch, seed=2, scale=1.0):
    _need_gpu()
    m = hb.MLP(dims, precision=prec, seed=0)
    params = init_params(dims, seed=seed, scale=scale)
    m.set_params(params_to_flat(params))
    w = hb.Worker(m, max_batch)
    return m, w, params


def grads_case(dims, kind, b, prec, scale=1.0, d=None, opts=None, elem_tol=None):
    X, y = dataset(kind, b, d=d or dims[0], seed=7)
    y = (y % dims[-1]).astype(np.int32)
    m, w, params = make(dims, prec, b, scale=scale)
    for k, v in (opts or {}).items():
        m.set_option(k, v)
    tX, ty = to_device(X, y, "bf16" if prec == "bf16" else "f32")
    g, loss = w.step_grads(tX, ty, b)
    rows = w.row_losses(b)
    dW, db, l_ref = mlp64.grads(params, X.astype(np.float64), y)
    norm, elem = grad_errors(g, dims, dW, db)
    Z, _ = mlp64.forward(params, X.astype(np.float64))
    ref_rows = mlp64.xent_rows(Z[-1], y)
    # a row's loss is a function of its logits: bound its error relative to the logit scale
    scale = np.maximum(1.0, np.abs(Z[-1]).max(axis=1))
    row_err = float((np.abs(rows - ref_rows) / scale).max())
    assert row_err <= TOL[prec], ("per-row loss", row_err)
    assert max(elem) <= (elem_tol or TOL[prec]), ("element-wise", elem)
    return max(norm), abs(loss - l_ref) / l_ref, norm


CASES = [
    # (dims, dataset kind, batch) — tiny C1, ragged batches/widths, paper-shaped heads
    ([54, 64, 64, 7], "covtype", 32),
    ([54, 64, 64, 7], "covtype", 1),
    ([54, 512, 512, 7], "covtype", 300),
    ([54, 200, 136, 7], "covtype", 129),
    ([300, 1024, 1024, 2], "w8a", 1000),
    ([2000, 256, 2], "realsim", 200),
    ([24, 40, 3], "gauss", 77),
]


@pytest.mark.parametrize("dims,kind,b", CASES)
def test_gradients_bf16_tensor_cores(dims, kind, b):
    e, le, errs = grads_case(dims, kind, b, "bf16")
    assert e <= TOL["bf16"], errs
    assert le <= TOL["bf16"]


@pytest.mark.parametrize("dims,kind,b", CASES)
def test_gradients_fp32_check_mode(dims, kind, b):
    e, le, errs = grads_case(dims, kind, b, "fp32")
    assert e <= TOL["fp32"], errs
    assert le <= 1e-6


def test_gradients_saturated_init_bf16():
    # hard part: sigma' near saturation; S = sigma'(z) is stashed from fp32, not from bf16 H
    e, _, errs = grads_case([54, 512, 512, 512, 512, 7], "covtype", 256, "bf16", scale=4.0)
    assert e <= TOL["bf16"], errs


@pytest.mark.parametrize("prec", ["bf16", "fp32"])
def test_one_sgd_step_updates_model_in_place(prec):
    dims = [54, 128, 64, 7]
    X, y = dataset("covtype", 256, seed=3)
    m, w, params = make(dims, prec, 256)
    tX, ty = to_device(X, y, "bf16" if prec == "bf16" else "f32")
    lr = 0.5
    loss = w.step(tX, ty, 256, lr, want_loss=True)
    new, l_ref = mlp64.sgd_step(params, X.astype(np.float64), y, lr)
    got = split_flat(m.get_params(), dims)
    for l in range(3):
        for j in (0, 1):
            # the update lr*dW must match to the path's tolerance; the fp32 master adds at most
            # one rounding of W_new (<= 2^-24 |W_new| per element)
            err = np.linalg.norm(got[l][j] - new[l][j])
            allowed = TOL[prec] * np.linalg.norm(new[l][j] - params[l][j]) + 2.0 ** -23 * np.linalg.norm(new[l][j])
            assert err <= allowed, (l, j, err, allowed)
    assert abs(loss - l_ref) / l_ref <= TOL[prec]


@pytest.mark.parametrize("prec", ["bf16", "fp32"])
def test_mlp_loss_full_data(prec):
    dims = [54, 96, 7]
    X, y = dataset("covtype", 20000, seed=1)
    m, w, params = make(dims, prec, 64)
    tX, ty = to_device(X, y, "bf16" if prec == "bf16" else "f32")
    got = m.loss(tX, ty)
    ref = mlp64.full_loss(params, X.astype(np.float64), y)
    assert abs(got - ref) / ref <= (1e-3 if prec == "bf16" else 1e-6)


def test_step_argument_errors():
    dims = [54, 64, 7]
    X, y = dataset("covtype", 64, seed=1)
    m, w, _ = make(dims, "bf16", 32)
    tX, ty = to_device(X, y)
    with pytest.raises(hb.HogbatchError):
        w.step(tX, ty, 33, 0.1)          # batch > max_batch
    with pytest.raises(hb.HogbatchError):
        w.step(tX, ty, 0, 0.1)           # empty batch
    with pytest.raises(hb.HogbatchError):
        w.step(tX.float(), ty, 8, 0.1)   # bf16 model needs bf16 X


@pytest.mark.parametrize("prec", ["bf16", "fp32"])
def test_single_layer_logistic_regression(prec):
    # L = 1: the output layer reads X directly; its dW GEMM takes X as an MN-major operand
    e, le, errs = grads_case([54, 7], "covtype", 300, prec)
    assert e <= TOL[prec], errs


@pytest.mark.parametrize("prec", ["bf16", "fp32"])
def test_many_classes_uses_warp_shuffle_softmax(prec):
    # C > 16 takes the standalone warp-per-row softmax-xent kernel (delicious-like heads)
    dims = [64, 96, 40]
    X, y = dataset("gauss", 257, d=64, seed=3)
    y = np.random.default_rng(0).integers(0, 40, 257).astype(np.int32)
    m, w, params = make(dims, prec, 257)
    tX, ty = to_device(X, y, "bf16" if prec == "bf16" else "f32")
    g, loss = w.step_grads(tX, ty, 257)
    dW, db, l_ref = mlp64.grads(params, X.astype(np.float64), y)
    got = split_flat(g, dims)
    for l in range(2):
        assert rel_err(got[l][0], dW[l]) <= TOL[prec]
        assert rel_err(got[l][1], db[l]) <= TOL[prec]
    assert abs(loss - l_ref) / l_ref <= TOL[prec]


@pytest.mark.parametrize("prec", ["bf16", "fp32"])
def test_delicious_shaped_983_class_head(prec):
    # the paper's delicious shape (983 labels) as a single-label softmax head:
    # logits GEMM + the standalone warp-per-row softmax-xent kernel (C > 16), ragged batch
    e, le, errs = grads_case([500, 256, 983], "delicious", 300, prec)
    assert e <= TOL[prec], errs
    assert le <= TOL[prec]


@pytest.mark.parametrize("b", [32, 256, 1000, 2048])
def test_persistent_step_kernel_matches_oracle_and_per_layer_path(b):
    # small batches of narrow nets run as ONE persistent launch (step_kernel.cuh): the same GEMMs,
    # operands and epilogues as the per-layer launches, as stages between grid barriers
    dims = [54, 512, 512, 512, 512, 7]
    X, y = dataset("covtype", b, seed=21)
    params = init_params(dims, seed=2)
    tX, ty = to_device(X, y)
    out = {}
    for mode in ("persistent", "per_layer"):
        m = hb.MLP(dims)
        m.set_params(params_to_flat(params))
        m.set_option("step_kernel_max_b", 2048 if mode == "persistent" else 0)
        w = hb.Worker(m, b)
        l0 = hb.kernel_launches()
        g, loss = w.step_grads(tX, ty, b)
        out[mode] = (g, loss, hb.kernel_launches() - l0)
    # per-layer: 4 hidden forward, the output-layer kernel + its update (head.cuh), 4 dX, 5 dW GEMMs;
    # + the batch-loss reduction
    assert out["persistent"][2] == 2 and out["per_layer"][2] == 14
    dW, db, l_ref = mlp64.grads(params, X.astype(np.float64), y)
    norm, elem = grad_errors(out["persistent"][0], dims, dW, db)
    assert max(norm) <= TOL["bf16"] and max(elem) <= TOL["bf16"], (norm, elem)
    assert abs(out["persistent"][1] - l_ref) / l_ref <= TOL["bf16"]
    assert rel_err(out["persistent"][0], out["per_layer"][0]) <= 1e-3
    # and one in-place SGD step through it
    m = hb.MLP(dims)
    m.set_params(params_to_flat(params))
    m.set_option("step_kernel_max_b", 2048)
    w = hb.Worker(m, b)
    w.step(tX, ty, b, 0.5)
    new, _ = mlp64.sgd_step(params, X.astype(np.float64), y, 0.5)
    got = split_flat(m.get_params(), dims)
    for l in range(len(dims) - 1):
        assert rel_err(got[l][0] - params[l][0], new[l][0] - params[l][0]) <= TOL["bf16"], l


def test_batch_equal_to_max_batch_and_ragged_tiles():
    # b = max_batch with a ragged last row tile (b % 128 != 0) and ragged widths
    e, le, errs = grads_case([100, 136, 72, 3], "gauss", 1000, "bf16", d=100)
    assert e <= TOL["bf16"], errs


@pytest.mark.parametrize("dims,kind,b,elem_tol", [
    ([300, 1024, 1024, 1024, 2], "w8a", 5000, None),   # forward + dX pairs
    # forward + unsplit dW pairs; a 4096-wide sigmoid layer on unit-norm realsim rows is in its
    # near-linear regime, where bf16 rounding gives element-wise errors ~1.5e-2 (R25,
    # the C4 bound 2.5e-2; normwise stays <= 1e-2)
    ([4000, 4096, 2], "realsim", 2200, 2.5e-2)])
def test_cta_pair_gemms(dims, kind, b, elem_tol):
    # HB_OPT_GEMM_PAIR (default on): forward / dX / unsplit dW GEMMs run as persistent CTA pairs
    # (cta_group::2, 256 x 256 tiles over two SMs, ragged last pair tile).  Same k order per output
    # element as the one-CTA tiles, so the gradients must agree bitwise with the one-CTA path, and
    # with the oracle
    e, le, errs = grads_case(dims, kind, b, "bf16", opts={"gemm_pair": 1, "rowchain": 0}, elem_tol=elem_tol)
    assert e <= TOL["bf16"], errs
    assert le <= TOL["bf16"]
    X, y = dataset(kind, b, d=dims[0], seed=7)
    y = (y % dims[-1]).astype(np.int32)
    tX, ty = to_device(X, y, "bf16")
    out = []
    for pair in (0, 1):
        m, w, _ = make(dims, "bf16", b)
        m.set_option("rowchain", 0)
        m.set_option("gemm_pair", pair)
        g, loss = w.step_grads(tX, ty, b)
        out.append((np.array(g, copy=True), loss))
    assert np.array_equal(out[0][0], out[1][0])
    assert out[0][1] == out[1][1]


def test_mlp_create_argument_errors():
    _need_gpu()
    with pytest.raises(hb.HogbatchError):
        hb.MLP([54])                  # needs n_dims >= 2
    with pytest.raises(hb.HogbatchError):
        hb.MLP([54, 0, 7])            # zero width
    with pytest.raises(hb.HogbatchError):
        hb.MLP([54, 64, 1])           # one class
    m = hb.MLP([5, 4, 3])
    with pytest.raises(hb.HogbatchError):
        m.set_params(np.zeros(3, np.float32))   # wrong parameter count
