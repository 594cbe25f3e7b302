import os, sys
sys.path.insert(0, os.getcwd())
import numpy as np
import paper_conf_ipps_marws21_b200 as hb
from tests.helpers import dataset, init_params, params_to_flat, to_device
dims, b = [54, 64, 64, 7], 32
X, y = dataset("covtype", b, seed=11)
m = hb.MLP(dims, precision="bf16", seed=0)
m.set_params(params_to_flat(init_params(dims, seed=2)))
w = hb.Worker(m, b)
tX, ty = to_device(X, y)
g, loss = w.step_grads(tX, ty, b)
print("ok", loss)
