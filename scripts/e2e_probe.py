"""Per-epoch wall time of hogbatch_run on the device dataset vs the pinned host dataset
(staged H2D inside the call), default covtype workload (tuning aid for the e2e leg)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import bench
import paper_conf_ipps_marws21_b200 as hb
from synth import init_params, params_to_flat

cfg = bench.CONFIGS["covtype"]
X_host, y_host, Xd, yd = bench.device_data(cfg, 0, cfg["N"], "cuda:0")
dims = cfg["dims"]
m = hb.MLP(dims)
m.set_params(params_to_flat(init_params(dims, seed=2)))
wl, ws = hb.Worker(m, 8192), hb.Worker(m, 2048)
kind = sys.argv[1] if len(sys.argv) > 1 else "adaptive"
if kind == "adaptive":
    workers, pol = [wl, ws], hb.Policy(kind=hb.HB_ADAPTIVE, workers=[hb.WorkerSpec(4096, 8192, 8192), hb.WorkerSpec(32, 2048, 32)], eta0=0.05, b0=32)
else:
    workers, pol = [wl], hb.Policy(kind=hb.HB_MINIBATCH, workers=[hb.WorkerSpec(8192, 8192, 8192)], eta0=0.05, b0=32)
for name, X, y in (("device", Xd, yd), ("host", X_host, y_host), ("device", Xd, yd), ("host", X_host, y_host)):
    ts = []
    for _ in range(5):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        st = hb.hogbatch_run(workers, pol, X, y, epochs=1)
        torch.cuda.synchronize()
        ts.append((time.perf_counter() - t0) * 1e3)
    print(name, kind, " ".join(f"{t:6.2f}" for t in ts), "ms/epoch", flush=True)
t0 = time.perf_counter(); Xd.copy_(X_host); torch.cuda.synchronize(); t = time.perf_counter() - t0
print(f"torch H2D copy of X: {t*1e3:.2f} ms = {X_host.numel()*2/t/1e9:.1f} GB/s")
