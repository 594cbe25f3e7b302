"""Seeded input generators (synth/): determinism, shapes, bf16 exactness, priors."""
import numpy as np

from synth import bf16_round, covtype_like, flat_to_params, init_params, params_to_flat, sparse_like
from synth.data import COVTYPE_PRIORS, csr_to_dense


def test_bf16_round_exact_and_rne():
    x = np.array([1.0, 1.0 + 2 ** -8, 1.0 + 3 * 2 ** -9, -2.5, 0.0], dtype=np.float32)
    r = bf16_round(x)
    assert r[0] == 1.0 and r[1] == 1.0          # tie -> even
    assert r[2] == 1.0 + 2 ** -7                 # 1.01100.. rounds up
    assert r[3] == -2.5 and r[4] == 0.0
    assert np.array_equal(bf16_round(r), r)


def test_covtype_like_is_deterministic_and_calibrated():
    X1, y1 = covtype_like(20000)
    X2, y2 = covtype_like(20000)
    assert np.array_equal(X1, X2) and np.array_equal(y1, y2)
    assert X1.shape == (20000, 54) and y1.dtype == np.int32
    assert np.array_equal(bf16_round(X1), X1)
    assert np.all(X1[:, 10:14].sum(1) == 1) and np.all(X1[:, 14:].sum(1) == 1)
    freq = np.bincount(y1, minlength=7) / len(y1)
    assert np.abs(freq - COVTYPE_PRIORS).max() < 0.02


def test_sparse_like_rows():
    csr, y = sparse_like(500, 300, 11.6, 0.03, True)
    X = csr_to_dense(csr, 300, 304)
    assert X.shape == (500, 304) and np.all(X[:, 300:] == 0)
    assert set(np.unique(X)) <= {0.0, 1.0}
    csr, y = sparse_like(300, 2000, 20, 0.3, False)
    X = csr_to_dense(csr, 2000)
    np.testing.assert_allclose(np.linalg.norm(X, axis=1), 1.0, atol=2e-2)


def test_param_flat_roundtrip():
    dims = [5, 4, 3]
    p = init_params(dims)
    q = flat_to_params(params_to_flat(p), dims)
    for (a, b), (c, d) in zip(p, q):
        assert np.array_equal(a, c) and np.array_equal(b, d)


def test_delicious_like_single_label_zipf_priors():
    from synth import delicious_like
    csr, y = delicious_like(3000)
    csr2, y2 = delicious_like(3000)
    assert np.array_equal(y, y2) and np.array_equal(csr[1], csr2[1])
    X = csr_to_dense(csr, 500)
    assert X.shape == (3000, 500) and set(np.unique(X)) <= {0.0, 1.0}
    assert y.dtype == np.int32 and y.min() >= 0 and y.max() < 983
    # Zipf-like priors: the head classes dominate, frequencies decrease on average
    f = np.bincount(y, minlength=983) / len(y)
    assert f[:10].sum() > f[500:510].sum() * 5
