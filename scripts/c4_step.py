"""A few C4 SGD steps (configs[3]: 20958-4096x4-2, b = 8192) through the C ABI — the target of the
ncu captures (scripts/gpu_round.sh).  One step = 14 tcgen05 GEMM launches (5 forward incl. the
fused softmax-xent head, 4 dX, 5 dW + fused SGD)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ipps_marws21_b200 as hb
from synth import init_params, params_to_flat
from tests.helpers import dataset, to_device
dims, b = [20958, 4096, 4096, 4096, 4096, 2], 8192
steps = int(sys.argv[1]) if len(sys.argv) > 1 else 3
X, y = dataset("realsim", b, d=dims[0], seed=5)
tX, ty = to_device(X, y)
m = hb.MLP(dims)
m.set_params(params_to_flat(init_params(dims)))
w = hb.Worker(m, b)
for _ in range(steps):
    w.step(tX, ty, b, 0.01 * b / 32)
torch.cuda.synchronize()
print("ok", hb.kernel_launches())
