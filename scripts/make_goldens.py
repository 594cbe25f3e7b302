"""Write the oracle-computed goldens under tests/golden/ (calls ONLY oracle/ and synth/).

    python scripts/make_goldens.py

c2_trajectory.json — SURVEY §8(c) "Loss trajectory: deterministic SERIAL mode vs oracle, 100
steps ... then C2 truncated to 100 steps": the fp64 oracle's per-step batch loss of MINIBATCH
SGD on the covtype-shaped C2 net 54-512x4-7 at b = 8192 (the fused row-block chain's batch size),
eta0 = 0.001 at b0 = 32 (lr = eta0 * b / b0 = 0.256; the smallest rate of the
paper's powers-of-10 grid, L258), contiguous batches in dataset order [L141], 100 steps over the
581,012-row dataset (the tail of each epoch dropped, R7).  The oracle takes ~100 s
for this, so the GPU test reads the stored losses; tests/test_oracle_mlp.py re-derives the first
steps from the oracle to pin the file.
"""
from __future__ import annotations

import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from oracle import mlp64  # noqa: E402
from synth import covtype_like, init_params  # noqa: E402

C2 = dict(dims=[54, 512, 512, 512, 512, 7], N=581012, b=8192, eta0=0.001, b0=32, steps=100,
          data_seed=0, init_seed=2)


def c2_batches(spec=C2):
    nb = spec["N"] // spec["b"]
    lr = spec["eta0"] * spec["b"] / spec["b0"]
    return [((k % nb) * spec["b"], spec["b"], lr) for k in range(spec["steps"])]


def c2_trajectory(spec=C2, steps=None):
    X, y = covtype_like(spec["N"], seed=spec["data_seed"])
    P = init_params(spec["dims"], seed=spec["init_seed"])
    out = []
    for s, b, lr in c2_batches(spec)[:steps]:
        P, ls = mlp64.sgd_step(P, X[s:s + b].astype(np.float64), y[s:s + b], lr)
        out.append(ls)
    return out


def main():
    losses = c2_trajectory()
    doc = dict(_source="fp64 oracle (oracle/mlp64.sgd_step) written by scripts/make_goldens.py; see its "
                       "docstring.  Not produced by the CUDA path.", **C2, losses=losses)
    path = os.path.join(ROOT, "tests", "golden", "c2_trajectory.json")
    with open(path, "w") as f:
        json.dump(doc, f, indent=1)
    print("wrote", path, losses[:3], losses[-1])


if __name__ == "__main__":
    main()
