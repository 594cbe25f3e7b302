"""ORACLE — test infrastructure only.

A plain, slow, obviously-correct fp64 NumPy implementation of what the
Adaptive Hogbatch hot path computes (Ma, Rusu, Wu, Sim, IPDPSW/MARWS 2021,
/root/reference/PAPER.md).  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import it.
The CUDA product path (``paper_conf_ipps_marws21_b200``) never imports,
calls or links anything under ``oracle/``, and this package never imports
the product path.  The two share only the seeded input generators in
``synth/`` (which hold none of the method's arithmetic).

Modules
  mlp64   — Eq. (1) forward, Eq. (2) back-propagation, Eq. (3) SGD update,
            softmax cross-entropy loss (§III, §VII.A).
  coord   — Algorithm 1 (Hogbatch) and Algorithm 2 (Adaptive Hogbatch)
            coordinator on a deterministic virtual clock (§VI
            L147–L238), producing the schedule trace (O5).
  merge   — replica merge W <- W_base + gamma * sum_E (W_E - W_base)
            (§VI.B, §V.B).
  serial  — deterministic SERIAL execution of a schedule trace ("replicas are
            applied to the global model one after another, in the order in
            which they are received", §V.A).

Parity status: every function here is pinned by ``tests/test_oracle_*.py``
against closed forms, finite differences, library routines, brute force or
the golden fixtures in ``tests/golden/``.  The coordinator's golden trace
pins OUR reconstruction of the garbled Algorithm 2 (R1–R4), not a
value printed in the paper.
"""
