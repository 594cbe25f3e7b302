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


def split_sizes(b: int, t: int):
    """Alg. 2 CPU worker line 1 [L229] "split B into t sub-batches of size B/t"; reading R6:
    when t does not divide b the first (b mod t) sub-batches get ceil(b/t) rows."""
    return [b // t + (1 if i < b % t else 0) for i in range(t)]


def run_trace_nested(params, X, y, records, t_of_worker, max_steps: int | None = None):
    """SERIAL execution of a trace where worker E splits each batch into t_of_worker[E]
    sub-batches [L229–L233], applied one after another (lr scaled to the sub-batch size,
    [L179]).  Returns (final_params, per-batch mean loss)."""
    losses = []
    for r in records:
        if not r.served:
            continue
        if max_steps is not None and len(losses) >= max_steps:
            break
        tot, off = 0.0, r.offset
        for sz in split_sizes(r.b_after, t_of_worker[r.worker]):
            if sz == 0:
                continue
            params, ls = mlp64.sgd_step(params, X[off:off + sz], y[off:off + sz], r.lr * sz / r.b_after)
            tot += ls * sz
            off += sz
        losses.append(tot / r.b_after)
    return params, losses
