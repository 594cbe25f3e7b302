"""Gradient errors vs the fp64 oracle, output-layer kernel on / off (HB_OPT_HEAD_KERNEL), per
tensor: normwise and element-wise (R13).  Usage: python scripts/head_errors.py"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import paper_conf_ipps_marws21_b200 as hb  # noqa: E402
from oracle import mlp64  # noqa: E402
from tests.helpers import dataset, grad_errors, init_params, params_to_flat, to_device  # noqa: E402

SHAPES = [([64, 8192, 2], "gauss", 129), ([512, 4096, 2], "gauss", 600), ([54, 3000, 3], "gauss", 99),
          ([300, 1024, 1024, 2], "w8a", 777), ([54, 512, 512, 7], "covtype", 1000)]
for dims, kind, b in SHAPES:
    X, y = dataset(kind, b, d=dims[0], seed=7)
    y = (y % dims[-1]).astype(np.int32)
    params = init_params(dims, seed=2)
    dW, db, l_ref = mlp64.grads(params, X.astype(np.float64), y)
    for hk in (1, 0):
        m = hb.MLP(dims, precision="bf16", seed=0)
        m.set_params(params_to_flat(params))
        m.set_option("head_kernel", hk)
        w = hb.Worker(m, b)
        tX, ty = to_device(X, y, "bf16")
        g, loss = w.step_grads(tX, ty, b)
        norm, elem = grad_errors(g, dims, dW, db)
        print(json.dumps({"dims": dims, "b": b, "head_kernel": hk, "norm": [round(v, 5) for v in norm],
                          "elem": [round(v, 5) for v in elem], "loss_rel": abs(loss - l_ref) / l_ref}), flush=True)
        del w, m
