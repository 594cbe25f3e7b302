"""Seeded synthetic datasets shaped like the paper's (§VII.A).

Table II of the paper (dataset sizes) is missing from the extracted text
[PAPER.md L255]; shapes and class counts come from BASELINE.json.configs and
SURVEY.md §8(d) (covtype 581,012 x 54 / 7 classes, w8a 64,700 x 300 / 2,
real-sim 72,309 x 20,958 / 2).  Everything here is data preparation only:

* features are generated from numpy PCG64 streams and rounded to bf16-exact
  values (the GPU path stores the dataset in bf16, the oracle reads the very
  same values in fp64);
* labels come from a fixed random *tanh* teacher with Gumbel-max sampling
  whose per-class offsets are calibrated so class frequencies match the
  target priors.  The teacher deliberately uses different arithmetic from the
  method (tanh, Gumbel argmax) so this module shares no computation with the
  MLP being trained;
* initial parameters: W ~ N(0, 1/fan_in), b = 0 (reading R11 of the
  paper's "std equal to the number of units" [PAPER.md L258]).

Seeds: data = 0, teacher = 1, init = 2, schedule = 3.
"""
from __future__ import annotations

import numpy as np

# ---------------------------------------------------------------------------
# small helpers
# ---------------------------------------------------------------------------


def _rng(seed: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(seed))


def bf16_round(a) -> np.ndarray:
    """Round float values to the nearest bf16 (ties to even); returns float32."""
    x = np.ascontiguousarray(np.asarray(a, dtype=np.float32))
    u = x.view(np.uint32).astype(np.uint64)
    u = (u + 0x7FFF + ((u >> 16) & 1)) & 0xFFFF0000
    return u.astype(np.uint32).view(np.float32).reshape(x.shape)


def pad_cols(X: np.ndarray, ld: int) -> np.ndarray:
    """Zero-pad the columns of a 2-D array to width ``ld``."""
    n, d = X.shape
    if ld < d:
        raise ValueError("ld < d")
    out = np.zeros((n, ld), dtype=X.dtype)
    out[:, :d] = X
    return out


def _gumbel_labels(scores: np.ndarray, priors: np.ndarray, g: np.ndarray,
                   iters: int = 40) -> np.ndarray:
    """y = argmax(scores + o + g), with offsets o calibrated (fixed point on
    the empirical class frequencies) so that freq(y) ~= priors."""
    C = scores.shape[1]
    o = np.log(priors).astype(np.float64)
    for _ in range(iters):
        y = np.argmax(scores + o + g, axis=1)
        freq = np.bincount(y, minlength=C) / len(y)
        o += 0.8 * np.log(priors / np.maximum(freq, 0.5 / len(y)))
    return np.argmax(scores + o + g, axis=1).astype(np.int32)


# ---------------------------------------------------------------------------
# covtype-shaped: 10 continuous + one-hot(4) + one-hot(40) = 54 features, 7 classes
# ---------------------------------------------------------------------------

COVTYPE_PRIORS = np.array([211840, 283301, 35754, 2747, 9493, 17367, 20510],
                          dtype=np.float64) / 581012.0


def covtype_like(N: int, seed: int = 0, teacher_seed: int = 1):
    """Dense covtype-shaped dataset: X float32 [N, 54] (bf16-exact), y int32 [N]."""
    rng = _rng(seed)
    X = np.zeros((N, 54), dtype=np.float32)
    X[:, :10] = bf16_round(rng.standard_normal((N, 10)))
    rows = np.arange(N)
    X[rows, 10 + rng.integers(0, 4, N)] = 1.0
    X[rows, 14 + rng.integers(0, 40, N)] = 1.0
    t = _rng(teacher_seed)
    A = t.standard_normal((54, 32)) * (3.0 / np.sqrt(54.0))
    Cm = t.standard_normal((32, 7)) * 2.0
    scores = np.tanh(X.astype(np.float64) @ A) @ Cm / 0.5
    g = -np.log(-np.log(rng.uniform(1e-12, 1.0, size=(N, 7))))
    y = _gumbel_labels(scores, COVTYPE_PRIORS, g)
    return X, y


# ---------------------------------------------------------------------------
# sparse-shaped (w8a / real-sim): CSR generator + densification
# ---------------------------------------------------------------------------


def sparse_like(N: int, d: int, nnz_mean: float, pos_frac: float, binary: bool,
                seed: int = 0, teacher_seed: int = 1):
    """CSR (indptr, indices, values float32 bf16-exact) and labels y int32 in {0,1}.

    Column popularity is Zipf-like (p_j ~ 1/(rank+10)); row lengths are
    1 + Poisson(nnz_mean - 1).  binary=True gives 0/1 values (w8a-shaped);
    otherwise tf-idf-like positive values with unit-L2 rows (real-sim-shaped).
    """
    rng = _rng(seed)
    lens = 1 + rng.poisson(max(nnz_mean - 1.0, 0.0), size=N)
    lens = np.minimum(lens, d)
    indptr = np.zeros(N + 1, dtype=np.int64)
    np.cumsum(lens, out=indptr[1:])
    nnz = int(indptr[-1])
    perm = rng.permutation(d)
    p = 1.0 / (np.arange(d) + 10.0)
    p /= p.sum()
    cols = perm[rng.choice(d, size=nnz, p=p)]
    # de-duplicate within rows (sort, drop repeats by re-drawing uniformly)
    indices = np.empty(nnz, dtype=np.int64)
    for i in range(N):
        a, b = indptr[i], indptr[i + 1]
        c = np.unique(cols[a:b])
        while len(c) < b - a:
            c = np.unique(np.concatenate([c, rng.integers(0, d, b - a - len(c))]))
        indices[a:b] = c[: b - a]
    if binary:
        vals = np.ones(nnz, dtype=np.float64)
    else:
        vals = np.abs(rng.standard_normal(nnz)) + 0.1
        sq = np.add.reduceat(vals * vals, indptr[:-1])
        vals = vals / np.sqrt(np.repeat(sq, lens))
    vals = bf16_round(vals)
    t = _rng(teacher_seed)
    A = t.standard_normal((d, 32)) * (3.0 / np.sqrt(nnz_mean))
    Cm = t.standard_normal((32, 2)) * 2.0
    # x @ A for CSR rows
    XA = np.zeros((N, 32))
    rows = np.repeat(np.arange(N), lens)
    np.add.at(XA, rows, vals.astype(np.float64)[:, None] * A[indices])
    scores = np.tanh(XA) @ Cm / 0.5
    g = -np.log(-np.log(rng.uniform(1e-12, 1.0, size=(N, 2))))
    y = _gumbel_labels(scores, np.array([1.0 - pos_frac, pos_frac]), g)
    return (indptr, indices.astype(np.int32), vals), y


def delicious_like(N: int, seed: int = 0, teacher_seed: int = 1, C: int = 983, d: int = 500,
                   nnz_mean: float = 18.2):
    """delicious-shaped CSR (500 binary features, ~18 nonzeros/row) with ONE label per row out
    of C = 983 classes (the paper's multi-label task is out of scope; a
    single-label head of this width exercises the warp-per-row softmax kernel).  Class priors
    are Zipf-like (p_c ~ 1/(c + 5)); labels from a C-class tanh teacher with Gumbel-max sampling
    and calibrated offsets, as for the other shapes."""
    csr, _ = sparse_like(N, d, nnz_mean, 0.5, True, seed=seed, teacher_seed=teacher_seed)
    indptr, indices, vals = csr
    rng = _rng(seed + 1000)
    t = _rng(teacher_seed + 1000)
    A = t.standard_normal((d, 32)) * (3.0 / np.sqrt(nnz_mean))
    Cm = t.standard_normal((32, C)) * 2.0
    lens = np.diff(indptr)
    XA = np.zeros((N, 32))
    rows = np.repeat(np.arange(N), lens)
    np.add.at(XA, rows, vals.astype(np.float64)[:, None] * A[indices])
    scores = np.tanh(XA) @ Cm / 0.5
    g = -np.log(-np.log(rng.uniform(1e-12, 1.0, size=(N, C))))
    pri = 1.0 / (np.arange(C) + 5.0)
    y = _gumbel_labels(scores, pri / pri.sum(), g)
    return csr, y


def csr_to_dense(csr, d: int, ld: int | None = None) -> np.ndarray:
    indptr, indices, vals = csr
    N = len(indptr) - 1
    ld = d if ld is None else ld
    X = np.zeros((N, ld), dtype=np.float32)
    rows = np.repeat(np.arange(N), np.diff(indptr))
    X[rows, indices] = vals
    return X


# name -> (features, classes, default N, hidden widths of the BASELINE config)
DATASETS = {
    "covtype": dict(d=54, C=7, N=581012, hidden=[512] * 4),
    "w8a": dict(d=300, C=2, N=64700, hidden=[1024] * 3),
    "realsim": dict(d=20958, C=2, N=72309, hidden=[4096] * 4),
    "tiny": dict(d=54, C=7, N=10000, hidden=[64, 64]),
    "delicious": dict(d=500, C=983, N=16105, hidden=[512] * 8),
}


def make_dataset(name: str, N: int | None = None, seed: int = 0, dense: bool = True):
    """Return (X or CSR, y, d, C).  X is float32 [N, d] bf16-exact when dense."""
    spec = DATASETS[name]
    N = spec["N"] if N is None else N
    if name in ("covtype", "tiny"):
        X, y = covtype_like(N, seed=seed)
        return X, y, spec["d"], spec["C"]
    if name == "w8a":
        csr, y = sparse_like(N, 300, 11.6, 0.03, True, seed=seed)
    elif name == "delicious":
        csr, y = delicious_like(N, seed=seed)
    else:
        csr, y = sparse_like(N, 20958, 51.5, 0.31, False, seed=seed)
    X = csr_to_dense(csr, spec["d"]) if dense else csr
    return X, y, spec["d"], spec["C"]


# ---------------------------------------------------------------------------
# parameters
# ---------------------------------------------------------------------------


def init_params(dims, seed: int = 2, scale: float = 1.0):
    """[(W_l [n_l x n_{l-1}], b_l [n_l])] with W ~ N(0, (scale/sqrt(fan_in))^2), b = 0.

    Values are float32-exact (returned as float64 arrays) so the GPU fp32
    master and the fp64 oracle start from identical numbers.
    """
    rng = _rng(seed)
    params = []
    for l in range(1, len(dims)):
        W = rng.standard_normal((dims[l], dims[l - 1])) * (scale / np.sqrt(dims[l - 1]))
        params.append((W.astype(np.float32).astype(np.float64),
                       np.zeros(dims[l], dtype=np.float64)))
    return params


def params_to_flat(params) -> np.ndarray:
    """Flat float32 [W1 (row-major, unpadded), b1, W2, b2, ...] (mlp_get/set_params)."""
    return np.concatenate([np.concatenate([W.ravel(), b.ravel()]) for W, b in params]
                          ).astype(np.float32)


def flat_to_params(flat, dims):
    out, o = [], 0
    flat = np.asarray(flat, dtype=np.float64)
    for l in range(1, len(dims)):
        n, k = dims[l], dims[l - 1]
        W = flat[o:o + n * k].reshape(n, k)
        o += n * k
        b = flat[o:o + n]
        o += n
        out.append((W.copy(), b.copy()))
    return out
