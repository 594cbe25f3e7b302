"""ORACLE (test infrastructure only): deterministic SERIAL execution of a
coordinator trace.

PAPER.md §V.A [L125–L128]: "the default policy is synchronous model updates—
the replicas are applied to the global model one after another, in the order
in which they are received".  Each served record of ``oracle.coord.run``
(in ``seq`` order) becomes one SGD step (Eq. (3), [L53]) on the rows
[offset, offset + b) with the record's learning rate.
"""
from __future__ import annotations

from . import mlp64


def run_trace(params, X, y, records, max_steps: int | None = None):
    """Returns (final_params, list of per-step batch losses)."""
    losses = []
    for r in records:
        if not r.served:
            continue
        if max_steps is not None and len(losses) >= max_steps:
            break
        s, b = r.offset, r.b_after
        params, ls = mlp64.sgd_step(params, X[s:s + b], y[s:s + b], r.lr)
        losses.append(ls)
    return params, losses
