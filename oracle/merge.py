"""ORACLE (test infrastructure only): replica merge.

PAPER.md §VI.B [L174–L175]: the GPU worker computes on a deep replica and,
"once the replica is updated, we push it to the global model"; §V.B [L141]:
"If the update is applied to the deep replica, this has to be subsequently
integrated in the global model".  With several replicas that started from the
same base W_base, each push integrates that replica's delta:

    W <- W_base + gamma * sum_E (W_E - W_base)

gamma = 1 keeps every replica's update (delta sum, R18, the default);
gamma = 1/n averages the replicas.
"""
from __future__ import annotations

import numpy as np


def merge(base, replicas, gamma: float = 1.0):
    """base, replicas[E]: lists of (W, b); returns the merged list of (W, b)."""
    out = []
    for l, (Wb, bb) in enumerate(base):
        dW = sum(np.asarray(r[l][0], np.float64) - Wb for r in replicas)
        db = sum(np.asarray(r[l][1], np.float64) - bb for r in replicas)
        out.append((Wb + gamma * dW, bb + gamma * db))
    return out
