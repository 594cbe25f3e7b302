"""BASELINE configs[4]: batch-size x width sweep of the mini-batch SGD step (54-w^4-7 MLP,
covtype-shaped inputs), one B200.  Prints one JSON line per point: samples/s and the fraction of
the sustained bf16 tensor peak (MEASURED_PEAKS.json).  Device time with CUDA events over graph-
replayed hogbatch_run epochs of MINIBATCH (one worker, fixed b)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ipps_marws21_b200 as hb
from synth import covtype_like, init_params, pad_cols, params_to_flat
import bench

peaks = bench.load_peaks()
batches = [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "32,256,2048,8192,65536").split(",")]
widths = [int(x) for x in (sys.argv[2] if len(sys.argv) > 2 else "256,1024,4096,8192").split(",")]
N = 1 << 20
X, y = covtype_like(N, seed=0)
Xd = torch.from_numpy(pad_cols(X, 56)).to("cuda:0").to(torch.bfloat16)
yd = torch.from_numpy(y).to("cuda:0")
torch.cuda.synchronize()
for wdt in widths:
    dims = [54, wdt, wdt, wdt, wdt, 7]
    F = bench.flops_per_sample(dims)
    m = hb.MLP(dims)
    m.set_params(params_to_flat(init_params(dims, seed=2)))
    for b in batches:
        rows = min(N, max(b * 32, 262144)) // b * b  # >= 32 steps per epoch: stable device time
        w = hb.Worker(m, b)
        pol = hb.Policy(kind=hb.HB_MINIBATCH, workers=[hb.WorkerSpec(b, b, b)], eta0=0.0, b0=32)
        for _ in range(2):
            hb.hogbatch_run([w], pol, Xd, yd, epochs=1, n=rows)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record()
        st = hb.hogbatch_run([w], pol, Xd, yd, epochs=5, n=rows)
        e1.record()
        torch.cuda.synchronize()
        sps = st["total_samples"] / (e0.elapsed_time(e1) * 1e-3)
        print(json.dumps({"width": wdt, "batch": b, "samples_per_s": sps,
                          "tc_peak_frac": sps * F / (peaks["bf16_sus"] * 1e12),
                          "us_per_step": b / sps * 1e6}), flush=True)
        w.close()
    m.close()
