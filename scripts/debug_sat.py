import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ipps_marws21_b200 as hb
from oracle import mlp64
from tests.helpers import dataset, init_params, params_to_flat, rel_err, split_flat, to_device

def case(dims, kind, b, prec, scale=1.0, keep=[]):
    X, y = dataset(kind, b, d=dims[0], seed=7); y = (y % dims[-1]).astype(np.int32)
    m = hb.MLP(dims, precision=prec); params = init_params(dims, seed=2, scale=scale)
    m.set_params(params_to_flat(params)); w = hb.Worker(m, b)
    tX, ty = to_device(X, y, "bf16" if prec == "bf16" else "f32")
    g, loss = w.step_grads(tX, ty, b)
    dW, db, lref = mlp64.grads(params, X.astype(np.float64), y)
    got = split_flat(g, dims)
    e = [(round(rel_err(got[l][0], dW[l]),4), round(rel_err(got[l][1], db[l]),4)) for l in range(len(dims)-1)]
    keep.append((m, w))
    return e, loss, lref

seq = sys.argv[1] if len(sys.argv) > 1 else "A"
pre = {"A": [], "B": [([54, 64, 64, 7], "covtype", 32, "fp32")], "C": [([54, 64, 64, 7], "covtype", 32, "bf16")],
       "D": [([24, 40, 3], "gauss", 77, "fp32")], "E": [([24, 40, 3], "gauss", 77, "bf16")]}[seq]
for c in pre:
    print("pre", c, case(*c)[0])
print(seq, "sat", case([54, 512, 512, 512, 512, 7], "covtype", 256, "bf16", 4.0))
print(seq, "sat again", case([54, 512, 512, 512, 512, 7], "covtype", 256, "bf16", 4.0))
print(seq, "nonsat", case([54, 512, 512, 512, 512, 7], "covtype", 256, "bf16", 1.0))
