"""Loss vs epochs for MINIBATCH / ADAPTIVE on a config (learning-rate exploration)."""
import sys, os, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ipps_marws21_b200 as hb
from synth import init_params, params_to_flat
import bench
cfg = bench.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "covtype"]
epochs = int(sys.argv[2]) if len(sys.argv) > 2 else 30
etas = [float(x) for x in (sys.argv[3] if len(sys.argv) > 3 else "0.003,0.01,0.03").split(",")]
dims = cfg["dims"]
Xh, yh, Xd, yd = bench.device_data(cfg, 0, cfg["N"], "cuda:0")
m = hb.MLP(dims)
p0 = params_to_flat(init_params(dims, seed=2))
wl, ws = hb.Worker(m, 8192), hb.Worker(m, 2048)
for eta in etas:
    for name, kind, wk, sp in [("minibatch", hb.HB_MINIBATCH, [wl], [hb.WorkerSpec(8192, 8192, 8192)]),
                               ("adaptive", hb.HB_ADAPTIVE, [wl, ws], [hb.WorkerSpec(4096, 8192, 8192), hb.WorkerSpec(32, 2048, 32)])]:
        m.set_params(p0)
        st = hb.hogbatch_run(wk, hb.Policy(kind=kind, workers=sp, eta0=eta, b0=32, eval_loss=True), Xd, yd, epochs=epochs)
        print(eta, name, "t=%.3fs" % sum(st["epoch_train_s"]), [round(x, 3) for x in st["epoch_loss"]][::3], flush=True)
