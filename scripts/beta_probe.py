"""Measure beta [PAPER.md L238] on B200: the surviving fraction of t concurrent sub-batch updates
of a nested worker under Hogwild read-modify-write vs atomic adds (tests/test_gpu_multi.py)."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ipps_marws21_b200 as hb
from tests.helpers import dataset, init_params, params_to_flat, to_device
dims, s = [54, 512, 512, 7], 128
X1, y1 = dataset("covtype", s, seed=11)
y1 = (y1 % 7).astype(np.int32)
P0 = params_to_flat(init_params(dims, seed=2))
def run(mode, t, lr_sub=1e-3, sub=True):
    X, y = np.tile(X1, (t, 1)), np.tile(y1, t)
    tX, ty = to_device(X, y)
    m = hb.MLP(dims); m.set_option("update", mode); m.set_params(P0)
    w = hb.Worker(m, t * s, sub_batches=t) if sub and t > 1 else hb.Worker(m, t * s)
    w.step(tX, ty, t * s, lr_sub * t if (sub and t > 1) else lr_sub)
    torch.cuda.synchronize()
    return m.get_params().astype(np.float64) - P0
d1 = run(hb.HB_UPDATE_HOGWILD, 1)
print("single |d1|", np.linalg.norm(d1))
for t in (2, 4, 8, 16):
    for mode, name in ((hb.HB_UPDATE_ATOMIC, "atomic"), (hb.HB_UPDATE_HOGWILD, "hogwild")):
        ds = [run(mode, t) for _ in range(3)]
        bs = [float(d @ d1 / (t * d1 @ d1)) for d in ds]
        print(json.dumps({"t": t, "mode": name, "beta_vs_t_single": [round(b, 4) for b in bs],
                          "norm_ratio": [round(float(np.linalg.norm(d) / (t * np.linalg.norm(d1))), 4) for d in ds]}))
