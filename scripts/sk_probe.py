"""Tuning build: per-stage phase stamps of the persistent small-batch step kernel (C2 net)."""
import ctypes as C, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ipps_marws21_b200 as hb
from synth import init_params, params_to_flat
from tests.helpers import dataset, to_device
dims = [54, 512, 512, 512, 512, 7]
b = int(sys.argv[1]) if len(sys.argv) > 1 else 32
X, y = dataset("covtype", b, seed=0)
tX, ty = to_device(X, y)
m = hb.MLP(dims); m.set_params(params_to_flat(init_params(dims))); m.set_option("step_kernel_max_b", 2048)
w = hb.Worker(m, b)
for _ in range(5): w.step(tX, ty, b, 0.0)
torch.cuda.synchronize()
cap = 148 * 16 * 8
hb.lib.hb_rc_trace(None, cap)
w.step(tX, ty, b, 0.0); torch.cuda.synchronize()
buf = (C.c_uint64 * cap)()
hb.lib.hb_rc_trace(buf, cap)
a = np.frombuffer(buf, dtype=np.uint64).reshape(148, 16, 8).astype(np.int64)
G = int((a[:, 0, 0] > 0).sum())
t0 = a[:G, 0, 0].min()
names = ["prod start", "prod past bar", "mma first ready", "mma first commit", "epi start", "epi past bar", "epi done", "arrived"]
print("grid", G)
for s in range(10):
    row = []
    for k in range(8):
        v = a[:G, s, k]
        v = v[v > 0]
        row.append(f"{names[k]} {(np.median(v) - t0) / 1e3:7.2f}/{(v.max() - t0) / 1e3:7.2f}" if len(v) else f"{names[k]} -")
    print(f"stage {s}: " + " | ".join(row))
