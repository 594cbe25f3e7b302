"""One warm fused step at batch b (for ncu captures): python scripts/rc_one.py [b] [dims]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_marws21_b200 as hb
from tests.helpers import dataset, init_params, params_to_flat, to_device

b = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
dims = [int(x) for x in (sys.argv[2] if len(sys.argv) > 2 else "54,512,512,512,512,7").split(",")]
m = hb.MLP(dims, precision="bf16")
m.set_params(params_to_flat(init_params(dims)))
w = hb.Worker(m, b)
X, y = dataset("covtype", b, seed=1)
tX, ty = to_device(X, y)
for _ in range(3):
    w.step(tX, ty, b, 0.0)
torch.cuda.synchronize()
print("done", b, dims, "fused", m.fused_path())
