"""bf16 emulation of the tensor-core step's rounding sites (NOT the oracle; test tooling).

Emulates, in NumPy fp32 with explicit bf16 round-to-nearest-even at each storage site, the
arithmetic of the bf16 tensor-core SGD step (DESIGN.md §4/§5):
  * operands of every GEMM are bf16 (X, the bf16 shadow of W, H_l, dZ_l), accumulation fp32;
  * H_l = bf16(sigma(z)), S_l = bf16(sigma'(z)) from the fp32 z (R22);
  * dZ_L = bf16((softmax(z_L) - onehot) / b) for the dX GEMM; the head's dW GEMM reads the
    split-precision pair hi + lo (R24; site "dZLw"), dZ_{l-1} = bf16(fp32(dZ_l W_l) * S_{l-1});
  * dW fp32 from the bf16 operands; W_master -= lr dW in fp32; shadow = bf16(W_master).
Each site can be switched off (kept fp32) to attribute the trajectory drift against the fp64
oracle.  Usage:  python scripts/bf16_emulation.py --case c1|c2|adaptive --eta0 E [--sites]
(profiles/r02_bf16_emulation.txt holds the runs quoted in DESIGN.md R24/R25.)
"""
from __future__ import annotations

import argparse
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from synth import bf16_round, covtype_like, init_params  # noqa: E402


def _r(a, on):
    return bf16_round(a) if on else np.asarray(a, np.float32)


def _sig(z):
    return (1.0 / (1.0 + np.exp(-z.astype(np.float64)))).astype(np.float32)


def step(params, X, y, lr, sites):
    """One emulated SGD step; params = [(W fp32 master, b fp32)].  Returns (new params, loss)."""
    L = len(params)
    bsz = len(y)
    A = _r(X, True)
    Hs, Ss = [A], []
    for l, (W, b) in enumerate(params):
        Wb = _r(W, sites["W"])
        z = (A @ Wb.T).astype(np.float32) + b
        if l < L - 1:
            s = _sig(z)
            Ss.append(_r(s * (1 - s), sites["S"]))
            A = _r(s, sites["H"])
            Hs.append(A)
    m = z.max(axis=1, keepdims=True)
    e = np.exp((z - m).astype(np.float64))
    p = e / e.sum(axis=1, keepdims=True)
    loss = float(np.mean(np.log(e.sum(axis=1)) + m[:, 0] - z[np.arange(bsz), y]))
    p[np.arange(bsz), y] -= 1.0
    d32 = (p / bsz).astype(np.float32)
    dZ = _r(d32, sites["dZ"])
    if sites.get("dZLw", "bf16") == "hilo":  # R24: hi + lo planes, ~2^-17 relative
        dZw = dZ + bf16_round(d32 - dZ)
    elif sites.get("dZLw", "bf16") == "fp32":
        dZw = d32
    else:
        dZw = dZ
    new = [None] * L
    for l in range(L - 1, -1, -1):
        W, b = params[l]
        dW = ((dZw if l == L - 1 else dZ).T @ Hs[l]).astype(np.float32)
        db = (d32 if l == L - 1 else dZ).astype(np.float32).sum(axis=0)  # head bias from fp32 dz
        if l > 0:
            dZ = _r((dZ @ _r(W, sites["W"])).astype(np.float32) * Ss[l - 1], sites["dZ"])
        new[l] = ((W - np.float32(lr) * dW).astype(np.float32), (b - np.float32(lr) * db).astype(np.float32))
    return new, loss


def _oracle_traj(params, X, y, batches):
    from oracle import mlp64  # the fp64 reference trajectory (tooling only)
    out, P = [], params
    for s, b, lr in batches:
        P, ls = mlp64.sgd_step(P, X[s:s + b].astype(np.float64), y[s:s + b], lr)
        out.append(ls)
    return np.array(out)


def _emu_traj(params, X, y, batches, sites):
    P = [(W.astype(np.float32), bb.astype(np.float32)) for W, bb in params]
    out = []
    for s, b, lr in batches:
        P, ls = step(P, X[s:s + b], y[s:s + b], lr, sites)
        out.append(ls)
    return np.array(out)


def case_batches(case, eta0):
    """(dims, X, y, [(offset, b, lr)]) of the GPU parity tests' trajectories."""
    if case == "c1":  # test_deterministic_minibatch_trajectory_100_steps: C1, b = 32, 100 steps
        dims = [54, 64, 64, 7]
        X, y = covtype_like(10000, seed=0)
        return dims, X, y, [(k * 32, 32, eta0 * 32 / 32) for k in range(100)]
    if case == "c2":  # test_c2_fused_trajectory_100_steps: C2, b = 8192 (fused chain), 100 steps
        dims = [54, 512, 512, 512, 512, 7]
        X, y = covtype_like(581012, seed=0)
        nb = 581012 // 8192
        return dims, X, y, [((k % nb) * 8192, 8192, eta0 * 8192 / 32) for k in range(100)]
    if case == "adaptive":  # test_deterministic_adaptive_serial_matches_oracle (Alg. 2 trace)
        from oracle import coord as oc
        dims = [54, 96, 7]
        X, y = covtype_like(4096, seed=0)
        specs = [oc.WorkerSpec(16, 128, 16, 1.0, 0.0, 1.0), oc.WorkerSpec(64, 512, 512, 1.0, 20.0, 0.05)]
        recs = oc.run(oc.Policy(kind=oc.ADAPTIVE, alpha=2, eta0=eta0, b0=32, workers=specs), 4096, 2)
        return dims, X, y, [(r.offset, r.b_after, r.lr) for r in recs if r.served]
    raise ValueError(case)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--case", default="c1", choices=["c1", "c2", "adaptive"])
    ap.add_argument("--eta0", type=float, default=1.0)
    ap.add_argument("--sites", action="store_true", help="attribute the drift to each rounding site")
    args = ap.parse_args()
    dims, X, y, batches = case_batches(args.case, args.eta0)
    y = (y % dims[-1]).astype(np.int32)
    params = init_params(dims, seed=2)
    ref = _oracle_traj(params, X, y, batches)
    allon = dict(W=True, H=True, S=True, dZ=True)
    cases = {"round-1 kernels (bf16 dZ_L)": allon}
    if args.sites:
        cases["fp32 everywhere"] = {k: False for k in allon}
        for k in allon:
            cases[f"only {k} bf16"] = {kk: kk == k for kk in allon}
            cases[f"all but {k}"] = {kk: kk != k for kk in allon}
        cases["head dW from fp32 dZ_L"] = dict(allon, dZLw="fp32")
    cases["R24 hi/lo head dZ_L (current)"] = dict(allon, dZLw="hilo")
    print(f"case {args.case}, eta0 {args.eta0}, {len(batches)} steps; oracle batch loss: first "
          f"{np.round(ref[:4], 3).tolist()} max {ref.max():.3f} last {ref[-1]:.3f}")
    for name, sites in cases.items():
        got = _emu_traj(params, X, y, batches, sites)
        rel = np.abs(got - ref) / ref
        print(f"  {name:32s} max rel {rel.max():.2e} at step {rel.argmax():3d}")


if __name__ == "__main__":
    main()
