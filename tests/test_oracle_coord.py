"""Pins for oracle/coord.py, oracle/merge.py and oracle/serial.py (CPU only).

Pins: Algorithm 1's contiguous-batch semantics [PAPER.md L149–L158, L170],
hand-derived Algorithm 2 traces (derivations in the comments), the golden
trace of SURVEY.md Appendix D2, invariants of Algorithm 2 [L236] under
random configurations, reductions between policies, and the paper's
qualitative claims [L271, L273].
"""
import os

import numpy as np
from hypothesis import given, settings, strategies as st

from oracle import coord, merge, mlp64, serial
from oracle.coord import ADAPTIVE, HOGBATCH, MINIBATCH, STATIC, Policy, WorkerSpec

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def tup(recs):
    return [r.astuple() for r in recs]


def test_minibatch_contiguous_ranges_and_dropped_tail():
    # Alg. 1: extract the next batch while B != {} [L153–L156]; epoch restarts on
    # the full dataset [L170]; a tail smaller than b is not served (R7).
    p = Policy(kind=MINIBATCH, eta0=0.5, b0=4, workers=[WorkerSpec(4, 4, 4, 1.0, 0.0)])
    recs = coord.run(p, N=18, epochs=2)
    served = [r for r in recs if r.served]
    assert [r.offset for r in served] == [0, 4, 8, 12] * 2
    assert all(r.lr == 0.5 and r.b_after == 4 for r in served)
    assert [r.epoch for r in recs if not r.served] == [0, 1]


def test_hogbatch_equal_batches_disjoint_cover():
    # Alg. 1 with 3 workers of different speeds: same b for all [L170]
    p = Policy(kind=HOGBATCH, eta0=0.1, b0=8,
               workers=[WorkerSpec(8, 8, 8, 0, c) for c in (1.0, 0.3, 2.5)])
    recs = coord.run(p, N=100, epochs=3)
    for e in range(3):
        offs = sorted(r.offset for r in recs if r.served and r.epoch == e)
        assert offs == list(range(0, 96, 8))
    assert all(r.action == "none" and r.b_after == 8 for r in recs)


def test_hand_derived_adaptive_trace_reading_A_dispatch_credit():
    # N=10, 1 epoch, alpha=2, eta0=1, b0=1; W0: [1,4] init 1, T=b; W1: [2,8] init 8, T=1+b/2.
    # t=0 E0: u=(0,0) none, serve 1@0, u0=1, done t=1
    # t=0 E1: u1=0 < 1 -> halve 8->4, serve 4@1, u1=1, done t=3
    # t=1 E0: u0=1 = 1 none, serve 1@5, u0=2, done t=2
    # t=2 E0: u0=2 > 1 -> double 1->2, u0 <- 1, serve 2@6, u0=2, done t=4
    # t=3 E1: u1=1 < 2 -> halve 4->2 (= floor), serve 2@8, cursor 10, done t=5
    # t=4 E0: u0=2 = 2 none, 0 rows left -> idle;  t=5 E1: none, idle -> epoch ends
    p = Policy(kind=ADAPTIVE, alpha=2, eta0=1.0, b0=1,
               workers=[WorkerSpec(1, 4, 1, 0.0, 1.0), WorkerSpec(2, 8, 8, 1.0, 0.5)])
    exp = [(0, 0, 0, 0, 0, 1, "none", 1, 0, 1, 0, 1),
           (1, 0, 1, 0, 0, 8, "halve", 4, 0, 1, 1, 4),
           (2, 0, 0, 1, 1, 1, "none", 1, 1, 1, 5, 1),
           (3, 0, 0, 2, 2, 1, "double", 2, 1, 1, 6, 2),
           (4, 0, 1, 3, 1, 4, "halve", 2, 1, 1, 8, 2),
           (5, 0, 0, 4, 2, 2, "none", 2, 2, 0, -1, 0),
           (6, 0, 1, 5, 2, 2, "none", 2, 2, 0, -1, 0)]
    assert tup(coord.run(p, N=10, epochs=1)) == exp


def test_hand_derived_adaptive_trace_reading_C_completion_credit():
    # Same workers, credit at the worker's next ScheduleWork, no u reset (reading C), 2 epochs.
    # ep0: t=0 E0 none serve 1@0 (done 1); t=0 E1 none serve 8@1 (done 5), cursor 9
    #      t=1 E0: u0=1 > 0 -> double 2, 1 row left -> idle; t=5 E1: u1=1 = 1 none, idle
    # ep1 starts at t=5: E0 u=(1,1) none serve 2@0 (done 7); E1 none serve 8@2 (done 10)
    #      t=7 E0: u0=2 > 1 -> double 4, idle; t=10 E1: u1=2 = 2 none, idle
    p = Policy(kind=ADAPTIVE, alpha=2, eta0=1.0, b0=1, reset="none", credit="completion",
               workers=[WorkerSpec(1, 4, 1, 0.0, 1.0), WorkerSpec(2, 8, 8, 1.0, 0.5)])
    exp = [(0, 0, 0, 0, 0, 1, "none", 1, 0, 1, 0, 1),
           (1, 0, 1, 0, 0, 8, "none", 8, 0, 1, 1, 8),
           (2, 0, 0, 1, 1, 1, "double", 2, 1, 0, -1, 0),
           (3, 0, 1, 5, 1, 8, "none", 8, 1, 0, -1, 0),
           (4, 1, 0, 5, 1, 2, "none", 2, 1, 1, 0, 2),
           (5, 1, 1, 5, 1, 8, "none", 8, 1, 1, 2, 8),
           (6, 1, 0, 7, 2, 2, "double", 4, 2, 0, -1, 0),
           (7, 1, 1, 10, 2, 8, "none", 8, 2, 0, -1, 0)]
    assert tup(coord.run(p, N=10, epochs=2)) == exp


def load_d2():
    rows = []
    for line in open(os.path.join(GOLD, "d2_trace.txt")):
        if line.startswith("#") or not line.strip():
            continue
        f = line.split()
        rows.append((int(f[0]), int(f[1]), int(f[2]), float(f[3]), float(f[4]), int(f[5]), f[6],
                     int(f[7]), float(f[8]), int(f[9]), int(f[10]), float(f[11])))
    return rows


D2_POLICY = dict(kind=ADAPTIVE, alpha=2, eta0=0.1, b0=8)
D2_WORKERS = [WorkerSpec(2, 8, 2, 0.0, 1.0), WorkerSpec(4, 16, 16, 2.0, 0.25)]


def test_golden_trace_d2():
    p = Policy(workers=D2_WORKERS, **D2_POLICY)
    got = tup(coord.run(p, N=40, epochs=2))
    exp = load_d2()
    assert len(got) == len(exp)
    for g, e in zip(got, exp):
        assert g[:3] == e[:3] and g[5:8] == e[5:8] and g[9:11] == e[9:11], (g, e)
        assert abs(g[3] - e[3]) < 1e-12 and g[4] == e[4] and g[8] == e[8]
        assert abs(g[11] - e[11]) < 1e-12


@settings(max_examples=60, deadline=None)
@given(nw=st.integers(1, 4), N=st.integers(1, 400), epochs=st.integers(1, 3),
       seed=st.integers(0, 10**6), reset=st.sampled_from(["fastest", "none"]),
       credit=st.sampled_from(["dispatch", "completion"]))
def test_adaptive_invariants(nw, N, epochs, seed, reset, credit):
    rng = np.random.default_rng(seed)
    specs = []
    for _ in range(nw):
        lo = int(2 ** rng.integers(0, 4))
        hi = lo * int(2 ** rng.integers(0, 4))
        init = int(rng.choice([lo, hi]))
        specs.append(WorkerSpec(lo, hi, init, float(rng.uniform(0, 3)), float(rng.uniform(0.05, 2)),
                                float(rng.choice([1.0, 4.0]))))
    p = Policy(kind=ADAPTIVE, alpha=2, eta0=0.1, b0=4, reset=reset, credit=credit, workers=specs)
    recs = coord.run(p, N=N, epochs=epochs, max_records=5000)
    cursor = {}
    for r in recs:
        s = specs[r.worker]
        # thresholds are never crossed [L236]
        assert s.minb <= r.b_after <= s.maxb
        # b changes only by x alpha / floor(/ alpha), clamped [L211, L213, L236]
        if r.action == "halve":
            assert r.b_after == max(r.b_before // 2, s.minb) and r.b_after < r.b_before
        elif r.action == "double":
            assert r.b_after == min(r.b_before * 2, s.maxb) and r.b_after > r.b_before
        else:
            assert r.b_after == r.b_before
        if r.served:
            # contiguous ranges handed out in order within an epoch [L141]
            assert r.offset == cursor.get(r.epoch, 0)
            cursor[r.epoch] = r.offset + r.b_after
            assert cursor[r.epoch] <= N
            assert r.lr == 0.1 * r.b_after / 4
    if nw == 1:
        assert all(r.action == "none" for r in recs)


def test_adaptive_with_fixed_thresholds_is_static_and_one_worker_is_minibatch():
    specs = [WorkerSpec(4, 4, 4, 0, 1.0), WorkerSpec(16, 16, 16, 1.0, 0.1)]
    a = coord.run(Policy(kind=ADAPTIVE, workers=specs), N=203, epochs=2)
    s = coord.run(Policy(kind=STATIC, workers=specs), N=203, epochs=2)
    assert [(r.worker, r.offset, r.b_after) for r in a] == [(r.worker, r.offset, r.b_after) for r in s]
    one = [WorkerSpec(2, 64, 8, 0, 1.0)]
    a1 = coord.run(Policy(kind=ADAPTIVE, workers=one), N=99, epochs=2)
    m1 = coord.run(Policy(kind=MINIBATCH, workers=[WorkerSpec(8, 8, 8, 0, 1.0)]), N=99, epochs=2)
    assert [(r.offset, r.b_after) for r in a1] == [(r.offset, r.b_after) for r in m1]


def test_paper_like_heterogeneous_run_balances_updates():
    # [L264]/[L253]: CPU worker t=56 threads, beta=1 (credits 56 updates per batch, Alg. 2
    # line 6), ~270x slower per example than the GPU; GPU b in [512, 8192] with ~50%
    # utilisation at the lower threshold [L258]; CPU b in [56, 3584] (1–64/thread, [L255]).
    # Paper: each of CPU and GPU performs approximately half of the updates [L271], and
    # the GPU batch decreases to the lower threshold [L273].
    cpu = WorkerSpec(56, 3584, 56, 0.0, 270 / 8192, 56.0)
    gpu = WorkerSpec(512, 8192, 8192, 512 / 8704, 1 / 8704, 1.0)
    recs = coord.run(Policy(kind=ADAPTIVE, workers=[cpu, gpu]), N=581012, epochs=3)
    upd = [sum(cpu.incr for r in recs if r.served and r.worker == 0),
           sum(gpu.incr for r in recs if r.served and r.worker == 1)]
    share = upd[0] / sum(upd)
    assert 0.4 < share < 0.65, share
    gb = [r.b_after for r in recs if r.served and r.worker == 1]
    assert np.median(gb) == 512


def test_merge_delta_sum_and_average():
    # [L141], [L175]: W <- W_base + gamma * sum_E (W_E - W_base)
    rng = np.random.default_rng(0)
    base = [(rng.standard_normal((3, 2)), rng.standard_normal(3))]
    deltas = [[(rng.standard_normal((3, 2)), rng.standard_normal(3))] for _ in range(4)]
    reps = [[(base[0][0] + d[0][0], base[0][1] + d[0][1])] for d in deltas]
    m = merge.merge(base, reps, 1.0)
    np.testing.assert_allclose(m[0][0], base[0][0] + sum(d[0][0] for d in deltas), atol=1e-14)
    a = merge.merge(base, reps, 0.25)
    np.testing.assert_allclose(a[0][0], sum(r[0][0] for r in reps) / 4, atol=1e-14)
    one = merge.merge(base, reps[:1], 1.0)
    np.testing.assert_allclose(one[0][1], reps[0][0][1], atol=1e-15)


def test_serial_run_equals_manual_sgd_loop():
    rng = np.random.default_rng(1)
    dims = [5, 4, 3]
    params = [(rng.standard_normal((dims[l], dims[l - 1])), np.zeros(dims[l])) for l in (1, 2)]
    X = rng.standard_normal((30, 5))
    y = rng.integers(0, 3, 30)
    recs = coord.run(Policy(kind=MINIBATCH, eta0=0.3, b0=4, workers=[WorkerSpec(4, 4, 4)]), 30, 1)
    got, losses = serial.run_trace(params, X, y, recs)
    P = params
    exp_l = []
    for s in range(0, 28, 4):
        P, ls = mlp64.sgd_step(P, X[s:s + 4], y[s:s + 4], 0.3)
        exp_l.append(ls)
    assert losses == exp_l
    for (a, b), (c, d) in zip(got, P):
        assert np.array_equal(a, c) and np.array_equal(b, d)


def test_nested_split_sizes_and_t1_reduces_to_serial():
    # R6 reading of Alg. 2 line 1 [L229]
    assert serial.split_sizes(10, 4) == [3, 3, 2, 2]
    assert serial.split_sizes(8, 4) == [2, 2, 2, 2]
    assert sum(serial.split_sizes(1000, 56)) == 1000
    rng = np.random.default_rng(2)
    dims = [5, 4, 3]
    params = [(rng.standard_normal((dims[l], dims[l - 1])), np.zeros(dims[l])) for l in (1, 2)]
    X = rng.standard_normal((64, 5))
    y = rng.integers(0, 3, 64)
    recs = coord.run(Policy(kind=MINIBATCH, eta0=0.2, b0=8, workers=[WorkerSpec(16, 16, 16)]), 64, 1)
    a, la = serial.run_trace(params, X, y, recs)
    b, lb = serial.run_trace_nested(params, X, y, recs, [1])
    assert la == lb and all(np.array_equal(p[0], q[0]) for p, q in zip(a, b))
    # t = 2: each batch = two half-size SGD steps with half the learning rate
    c, lc = serial.run_trace_nested(params, X, y, recs, [2])
    P = params
    for s in range(0, 64, 16):
        P, _ = mlp64.sgd_step(P, X[s:s + 8], y[s:s + 8], 0.2 * 16 / 8 * 0.5)
        P, _ = mlp64.sgd_step(P, X[s + 8:s + 16], y[s + 8:s + 16], 0.2 * 16 / 8 * 0.5)
    np.testing.assert_allclose(c[0][0], P[0][0], atol=1e-14)
