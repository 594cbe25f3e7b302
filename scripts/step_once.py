"""A few SGD steps of an MLP through the C ABI (target of ncu captures).
    python scripts/step_once.py <dims comma-separated> <batch> [steps] [option=value ...]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ipps_marws21_b200 as hb
from synth import init_params, params_to_flat
from tests.helpers import dataset, to_device
dims = [int(x) for x in sys.argv[1].split(",")]
b = int(sys.argv[2])
steps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
X, y = dataset("gauss", b, d=dims[0], seed=5)
y = (y % dims[-1]).astype(np.int32)
tX, ty = to_device(X, y)
m = hb.MLP(dims)
for kv in sys.argv[4:]:
    k, v = kv.split("=")
    m.set_option(k, int(v))
m.set_params(params_to_flat(init_params(dims)))
w = hb.Worker(m, b)
for _ in range(steps):
    w.step(tX, ty, b, 0.01)
torch.cuda.synchronize()
print("ok")
