"""Fused row-block step: per-step device time vs batch size, and per-step phase stamps of one launch.

    python scripts/rc_probe.py [dims comma-separated] [batches comma-separated]
"""
import ctypes as C, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_ipps_marws21_b200 as hb
from tests.helpers import dataset, init_params, params_to_flat, to_device

dims = [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "54,512,512,512,512,7").split(",")]
batches = [int(x) for x in (sys.argv[2] if len(sys.argv) > 2 else "32,256,2048,8192").split(",")]
m = hb.MLP(dims, precision="bf16")
if os.environ.get("HB_ROWCHAIN", "1") != "0":
    m.set_fused_min_batch(int(os.environ.get("HB_RC_MIN_B", "1")))
m.set_params(params_to_flat(init_params(dims)))
B = max(batches)
w = hb.Worker(m, B)
X, y = dataset("covtype", B, seed=1)
tX, ty = to_device(X, y)
st = torch.cuda.ExternalStream(w.stream_handle)
print("fused cluster size", m.fused_path(), "env HB_ROWCHAIN", os.environ.get("HB_ROWCHAIN"), flush=True)
for b in batches:
    for _ in range(5):
        w.step(tX, ty, b, 0.0)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    n = 30
    e0.record(st)
    for _ in range(n):
        w.step(tX, ty, b, 0.0)
    e1.record(st)
    torch.cuda.synchronize()
    print(f"b={b:6d}: {e0.elapsed_time(e1) * 1000 / n:8.1f} us/step (direct launches incl. host encode)", flush=True)
if m.fused_path():
    for b in [x for x in batches if x in (32, 8192)] or batches[-1:]:
        cap = 1024 * 24 * 14
        hb.lib.hb_rc_trace(None, cap)
        w.step(tX, ty, b, 0.0)
        buf = (C.c_uint64 * cap)()
        hb.lib.hb_rc_trace(buf, cap)
        hb.lib.hb_rc_trace(None, 0) if False else None
        a = np.frombuffer(buf, dtype=np.uint64).reshape(1024, 24, 14).astype(np.int64)
        grid = m.fused_path(b) * ((b + 127) // 128)
        ctas = np.arange(grid)
        a = a[ctas]
        t0 = a[:, 0, 0].min()
        L = len(dims) - 1
        nct = grid
        base = 1024 * 24 * 14
        raw = np.frombuffer(buf, dtype=np.uint64).astype(np.int64)
        # the tail region is indexed with gridDim.x = nct CTAs
        tail = raw[nct * 24 * 14: nct * 24 * 14 + 3 * nct * 16].reshape(3, nct, 16)
        for ci in range(min(2, nct)):
            iss, crdy, wrdy = tail[0, ci, :8], tail[1, ci, :8], tail[2, ci, :8]
            rel = lambda v: [round(float(x - t0) / 1000, 2) for x in v]
            print(f"   cta{ci} step2 k-blocks (us from kernel start): issue {rel(iss)}\n"
                  f"        chunk ready {rel(crdy)}\n        W ready     {rel(wrdy)}")
        print(f"--- b={b}: {len(ctas)} CTAs, span {(a[a > 0].max() - t0) / 1000:.2f} us; per step (median over CTAs, us from kernel start):")
        print("   step  mma_start  first_w  mma_issued  epi_acc  epi_peer  epi_end  ld0  c0comp  c0sig  c1sig  c0fence  c0bar  c0copies  c0hstore")
        for s in range(2 * L - 1):
            v = a[:, s, :]
            row = [np.median(v[:, k][v[:, k] > 0] - t0) / 1000 if (v[:, k] > 0).any() else -1 for k in range(14)]
            print(f"   {s:4d}  " + "  ".join(f"{x:8.2f}" for x in row))

# device time per step (graph replay), whole step / chain only / dW only
import ctypes as C2
for b in batches:
    out = []
    for part in (0, 1, 2):
        us = C2.c_float()
        rc = hb.lib.mlp_step and hb.lib.hb_bench_step(w.h, C2.c_void_p(tX.data_ptr()), tX.stride(0),
                                                      C2.c_void_p(ty.data_ptr()), b, 20, part, C2.byref(us))
        out.append(us.value if rc == 0 else float("nan"))
    print(f"graph b={b:6d}: step {out[0]:8.1f} us  chain {out[1]:8.1f} us  dW {out[2]:8.1f} us"
          f"  -> {b / out[0]:.1f} samples/us", flush=True)
