"""Small-batch steps of the C2 net (54-512x4-7): device time per step of a single-worker
hogbatch_run (graph replay, 2 steps in flight) at b = 32 .. 4096, to compare with the per-kernel
durations of an ncu launch list of the same command."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ipps_marws21_b200 as hb
from synth import init_params, params_to_flat
from tests.helpers import dataset, to_device
dims = [int(x) for x in os.environ.get("DIMS", "54,512,512,512,512,7").split(",")]
bs = [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "32,256,2048,4096").split(",")]
steps = int(os.environ.get("STEPS", "200"))
X, y = dataset("covtype", max(bs) * 64, seed=0)
tX, ty = to_device(X, y)
m = hb.MLP(dims)
m.set_params(params_to_flat(init_params(dims)))
m.set_option("step_kernel_max_b", int(os.environ.get("SKB", "0")))
for b in bs:
    w = hb.Worker(m, b)  # per-b worker: the persistent kernel's grid follows its max_batch
    n = b * steps
    reps = max(1, (n + tX.shape[0] - 1) // tX.shape[0])
    Xb, yb = (tX.repeat(reps, 1)[:n].contiguous(), ty.repeat(reps)[:n].contiguous()) if reps > 1 else (tX[:n], ty[:n])
    pol = hb.Policy(kind=hb.HB_MINIBATCH, workers=[hb.WorkerSpec(b, b, b)], eta0=0.0, b0=32)
    hb.hogbatch_run([w], pol, Xb, yb, epochs=1)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    st = hb.hogbatch_run([w], pol, Xb, yb, epochs=1)
    e1.record()
    torch.cuda.synchronize()
    us = e0.elapsed_time(e1) * 1e3 / st["n_steps"]
    print(json.dumps({"b": b, "us_per_step": round(us, 2), "fused": m.fused_path(b), "steps": st["n_steps"]}), flush=True)
