"""Shared test helpers: device copies of the seeded synthetic inputs (synth/) and
normwise comparison.  No method arithmetic here."""
from __future__ import annotations

import numpy as np

from synth import bf16_round, covtype_like, init_params, pad_cols, params_to_flat, sparse_like
from synth.data import csr_to_dense


def rel_err(a, b) -> float:
    a = np.asarray(a, np.float64)
    b = np.asarray(b, np.float64)
    nb = np.linalg.norm(b)
    return float(np.linalg.norm(a - b) / (nb if nb > 0 else 1.0))


def grad_errors(flat, dims, dW, db):
    """Per tensor (W_1, b_1, W_2, ...): normwise error ||g - g_ref||_F / ||g_ref||_F and
    element-wise error max_i |g_i - g_ref_i| / max_i |g_ref_i| (R13)."""
    got = split_flat(flat, dims)
    norm, elem = [], []
    for l in range(len(dims) - 1):
        for a, r in ((got[l][0], dW[l]), (got[l][1], db[l])):
            r = np.asarray(r, np.float64)
            norm.append(rel_err(a, r))
            mx = np.abs(r).max()
            elem.append(float(np.abs(np.asarray(a, np.float64) - r).max() / (mx if mx > 0 else 1.0)))
    return norm, elem


def split_flat(flat, dims):
    out, o = [], 0
    for l in range(1, len(dims)):
        n, k = dims[l], dims[l - 1]
        W = np.asarray(flat[o:o + n * k], np.float64).reshape(n, k)
        o += n * k
        b = np.asarray(flat[o:o + n], np.float64)
        o += n
        out.append((W, b))
    return out


def dataset(kind: str, N: int, d: int | None = None, seed: int = 0):
    """(X float32 bf16-exact [N, d], y int32)"""
    if kind == "covtype":
        return covtype_like(N, seed=seed)
    if kind == "w8a":
        csr, y = sparse_like(N, 300, 11.6, 0.03, True, seed=seed)
        return csr_to_dense(csr, 300), y
    if kind == "realsim":
        csr, y = sparse_like(N, d or 20958, 51.5, 0.31, False, seed=seed)
        return csr_to_dense(csr, d or 20958), y
    if kind == "delicious":  # 500 binary features, one of 983 Zipf-distributed labels
        from synth import delicious_like
        csr, y = delicious_like(N, seed=seed)
        return csr_to_dense(csr, 500), y
    if kind == "gauss":  # generic dense inputs for odd shapes
        rng = np.random.default_rng(seed)
        X = bf16_round(rng.standard_normal((N, d)))
        return X, rng.integers(0, 2, N).astype(np.int32)
    raise ValueError(kind)


def to_device(X, y, dtype="bf16", device="cuda:0"):
    """Device copies: X padded to a multiple of 8 columns (bf16 or fp32), y int32."""
    import torch
    ld = (X.shape[1] + 7) // 8 * 8
    Xp = pad_cols(np.asarray(X, np.float32), ld)
    tX = torch.from_numpy(Xp).to(device)
    tX = tX.to(torch.bfloat16) if dtype == "bf16" else tX
    ty = torch.from_numpy(np.asarray(y, np.int32)).to(device)
    torch.cuda.synchronize()  # the library's streams do not order after torch's stream
    return tX, ty


__all__ = ["grad_errors", "rel_err", "split_flat", "dataset", "to_device", "init_params", "params_to_flat"]
