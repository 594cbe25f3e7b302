"""C-ABI boundary checks that need no GPU: the library loads, exports every symbol
include/hogbatch.h declares, and its coordinator (hb_schedule_trace) reproduces the
oracle's Algorithm 1/2 traces exactly."""
import os
import re

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

import paper_conf_ipps_marws21_b200 as hb
from oracle import coord as ocoord

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_functions():
    src = open(os.path.join(ROOT, "include", "hogbatch.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"^\s*(?:const\s+char\*|void\*|int64_t|int)\s+(\w+)\s*\(", src, flags=re.M)))


def test_library_exports_every_declared_symbol():
    names = header_functions()
    assert len(names) >= 20
    for n in names:
        assert hasattr(hb.lib, n), n
    assert set(names) == set(hb._lib.EXPORTS)
    assert hb.lib.hb_abi_version() == 2


def test_no_device_is_reported_for_bad_ordinal():
    assert hb.lib.hb_device_ok(4096) == 0


def to_c_policy(p: ocoord.Policy, kind_override=None):
    return hb.Policy(kind=p.kind if kind_override is None else kind_override, alpha=p.alpha,
                     eta0=p.eta0, b0=p.b0,
                     reset=hb.HB_RESET_FASTEST if p.reset == "fastest" else hb.HB_RESET_NONE,
                     credit=hb.HB_CREDIT_DISPATCH if p.credit == "dispatch" else hb.HB_CREDIT_COMPLETION,
                     workers=[hb.WorkerSpec(w.minb, w.maxb, w.initb, w.incr, w.c0, w.c1) for w in p.workers])


def same(a, b):
    assert len(a) == len(b)
    for x, y in zip(a, b):
        assert x[0] == y[0] and x[1] == y[1] and x[2] == y[2], (x, y)
        assert x[3] == y[3] and x[4] == y[4] and x[5] == y[5] and x[6] == y[6], (x, y)
        assert x[7] == y[7] and x[8] == y[8] and x[9] == y[9] and x[10] == y[10], (x, y)
        assert x[11] == y[11], (x, y)


def test_cpp_coordinator_matches_golden_d2():
    p = ocoord.Policy(kind=ocoord.ADAPTIVE, alpha=2, eta0=0.1, b0=8,
                      workers=[ocoord.WorkerSpec(2, 8, 2, 0.0, 1.0), ocoord.WorkerSpec(4, 16, 16, 2.0, 0.25)])
    got = hb.schedule_trace(to_c_policy(p), 40, 2)
    same(got, [r.astuple() for r in ocoord.run(p, 40, 2)])
    assert len(got) == 28


@settings(max_examples=80, deadline=None)
@given(nw=st.integers(1, 4), N=st.integers(1, 500), epochs=st.integers(1, 3),
       seed=st.integers(0, 10**6), kind=st.sampled_from([ocoord.HOGBATCH, ocoord.STATIC, ocoord.ADAPTIVE]),
       reset=st.sampled_from(["fastest", "none"]), credit=st.sampled_from(["dispatch", "completion"]))
def test_cpp_coordinator_matches_oracle_random(nw, N, epochs, seed, kind, reset, credit):
    rng = np.random.default_rng(seed)
    ws = []
    for _ in range(nw):
        lo = int(2 ** rng.integers(0, 4))
        hi = lo * int(2 ** rng.integers(0, 4))
        init = int(rng.choice([lo, hi]))
        ws.append(ocoord.WorkerSpec(lo, hi, init, float(rng.integers(0, 4)), float(rng.integers(1, 8)) / 4,
                                    float(rng.choice([1.0, 4.0]))))
    if kind == ocoord.HOGBATCH:
        ws = [ocoord.WorkerSpec(w.minb, w.maxb, ws[0].initb if w.minb <= ws[0].initb <= w.maxb else w.initb,
                                w.c0, w.c1, w.incr) for w in ws]
        if len({w.initb for w in ws}) != 1:
            ws = [ocoord.WorkerSpec(4, 4, 4, w.c0, w.c1, w.incr) for w in ws]
    p = ocoord.Policy(kind=kind, alpha=2, eta0=0.25, b0=4, reset=reset, credit=credit, workers=ws)
    exp = [r.astuple() for r in ocoord.run(p, N, epochs, max_records=4000)]
    got = hb.schedule_trace(to_c_policy(p), N, epochs, cap=4000)
    same(got, exp)


def test_minibatch_trace_and_validation_errors():
    p = hb.Policy(kind=hb.HB_MINIBATCH, eta0=1.0, b0=32, workers=[hb.WorkerSpec(32, 32, 32)])
    tr = hb.schedule_trace(p, 100, 1)
    assert [r[10] for r in tr if r[9]] == [0, 32, 64]
    with pytest.raises(hb.HogbatchError) as e:
        hb.schedule_trace(hb.Policy(kind=hb.HB_MINIBATCH, workers=[hb.WorkerSpec(1, 1, 1)] * 2), 10, 1)
    assert e.value.code == hb._lib.HB_EINVAL
    with pytest.raises(hb.HogbatchError):
        hb.schedule_trace(hb.Policy(workers=[hb.WorkerSpec(4, 2, 3)]), 10, 1)
    with pytest.raises(hb.HogbatchError):
        hb.schedule_trace(hb.Policy(kind=hb.HB_HOGBATCH, workers=[hb.WorkerSpec(2, 2, 2), hb.WorkerSpec(4, 4, 4)]), 10, 1)


def test_model_creation_without_sm100_device_fails_loudly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(hb.HogbatchError) as e:
        hb.MLP([54, 64, 7])
    assert e.value.code in (hb._lib.HB_ECUDA, hb._lib.HB_EUNSUPPORTED)


def test_cpp_coordinator_matches_oracle_exhaustive_two_workers():
    # exhaustive small space (SURVEY §8(c) "brute-force enumeration" pin): every pair of worker
    # specs from a grid of thresholds / initial batches / virtual-clock costs, two data-set sizes,
    # both u-reset readings (R3) and both credit points (R21), two epochs — exact trace equality
    specs = []
    for lo, hi, init in [(1, 4, 1), (1, 4, 4), (2, 2, 2), (1, 2, 2), (2, 8, 8)]:
        for c0 in (0.0, 1.0):
            for c1 in (0.5, 2.0):
                specs.append((lo, hi, init, c0, c1))
    n = 0
    for a in specs:
        for b in specs:
            ws = [ocoord.WorkerSpec(a[0], a[1], a[2], a[3], a[4]), ocoord.WorkerSpec(b[0], b[1], b[2], b[3], b[4])]
            for N in (7, 23):
                for reset in ("fastest", "none"):
                    for credit in ("dispatch", "completion"):
                        p = ocoord.Policy(kind=ocoord.ADAPTIVE, alpha=2, eta0=0.5, b0=2, reset=reset, credit=credit,
                                          workers=ws)
                        exp = [r.astuple() for r in ocoord.run(p, N, 2, max_records=2000)]
                        same(hb.schedule_trace(to_c_policy(p), N, 2, cap=2000), exp)
                        n += 1
    assert n == 3200
