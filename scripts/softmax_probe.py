"""Standalone softmax-xent kernel at the delicious shape (b = 65,536, C = 983):
device time and achieved GB/s of the kernel from the library's per-launch CUDA events, against the
algorithmic bytes b*C*(4 + 2) + 8*b (fp32 logits read once, bf16 dZ written once, labels, losses)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ipps_marws21_b200 as hb
from synth import init_params, params_to_flat
from tests.helpers import dataset, to_device
dims, b = [500, 512, 983], 65536
X, y = dataset("delicious", b, seed=0)
tX, ty = to_device(X, y)
m = hb.MLP(dims)
m.set_params(params_to_flat(init_params(dims)))
w = hb.Worker(m, b)
for _ in range(3):
    w.step(tX, ty, b, 0.0)
torch.cuda.synchronize()
hb.prof_read(reset=True)
hb.prof_enable(True)
for _ in range(10):
    w.step(tX, ty, b, 0.0)
torch.cuda.synchronize()
p = hb.prof_read(reset=True)
hb.prof_enable(False)
sm = p["softmax_xent"]; print("bias partials", p["bias_sgd"])
peaks = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "MEASURED_PEAKS.json")))
us = sm["ms"] / sm["launches"] * 1e3
gbs = sm["bytes"] / (sm["ms"] * 1e-3) / 1e9
print(json.dumps({"kernel": "softmax_xent_kernel", "b": b, "C": dims[-1], "us_per_launch": us,
                  "alg_bytes_per_launch": sm["bytes"] / sm["launches"], "GB/s": gbs,
                  "frac_of_measured_hbm": gbs / peaks["hbm_gbs"], "launches": sm["launches"]}))
