"""Quick GPU sanity check of the step against the oracle (prints normwise errors)."""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_ipps_marws21_b200 as hb
from oracle import mlp64
from tests.helpers import dataset, init_params, params_to_flat, rel_err, split_flat, to_device

print("device_ok", hb.device_ok(0), torch.cuda.get_device_name(0), flush=True)
for prec in ("fp32", "bf16"):
    for dims, kind, b in [([54, 64, 64, 7], "covtype", 32), ([54, 512, 512, 7], "covtype", 300),
                          ([300, 1024, 2], "w8a", 1000)]:
        X, y = dataset(kind, b, seed=7)
        m = hb.MLP(dims, precision=prec)
        params = init_params(dims)
        m.set_params(params_to_flat(params))
        w = hb.Worker(m, b)
        tX, ty = to_device(X, y, "bf16" if prec == "bf16" else "f32")
        t = time.time()
        g, loss = w.step_grads(tX, ty, b)
        torch.cuda.synchronize()
        dW, db, lr = mlp64.grads(params, X.astype(np.float64), y)
        got = split_flat(g, dims)
        errs = [(round(rel_err(got[l][0], dW[l]), 6), round(rel_err(got[l][1], db[l]), 6)) for l in range(len(dims) - 1)]
        print(prec, dims, b, "loss", loss, lr, "errs", errs, "t", round(time.time() - t, 3), flush=True)
