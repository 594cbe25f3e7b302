#!/usr/bin/env python
"""bench.py — MLP-SGD throughput of the Adaptive Hogbatch hot path on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--config realsim]

Workload (default) = BASELINE.json configs[3], the config that carries the north star's >= 60% of
bf16 tensor peak at the paper's largest batch (8,192): real-sim-shaped data
(72,309 x 20,958 per GPU, densified, 2 classes) on the MLP 20958-4096x4-2 (sigmoid hidden layers,
softmax cross-entropy), Adaptive Hogbatch with ONE worker per GPU (b in [min_b, 8192], min_b
calibrated per reading R17) and ONE coordinator for all GPUs: with N > 1 ranks (torchrun, one
process per GPU) the ranks share the coordinator through POSIX shared memory (hb_coord_create),
so the paper's single set 𝔹 of remaining examples [L218-L220] spans every GPU and Algorithm 2
compares the GPUs' update counts [L130, L185]; each GPU holds the whole N x 72,309-row data set
(weak scaling: 72,309 rows per GPU) and the per-GPU model replicas are merged over NCCL
(hb_merge) `--merges` times per epoch.  At N = 1 the single worker's batch
stays at 8,192 (Algorithm 2 needs two workers).

One STEP = one hogbatch_run epoch over the global data set: batch selection, forward GEMM chain,
softmax-xent head, dX/dW GEMMs with the fused in-place SGD, the adaptive rule (every §8(a) row).
Loss evaluation is excluded.

Timing: W warm-up steps, then K steps each bracketed by CUDA events on the legacy default stream
(the worker streams are blocking streams, so the events bracket all their work), the L2 flushed
(256 MiB write) before each timed step, a barrier on both sides, max over ranks; nvidia-smi
clocks sampled during the timed region.  `roofline`: the dominant kernel (by device time, per
weight layer) from a SERIALISED profiling pass of the same steps (one stream, every launch
bracketed by CUDA events, outside the timed region), against the measured burst bf16 peak (each
launch runs alone there); `tc_peak_frac` of the whole timed step uses the sustained peak.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time
import uuid

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "MLP SGD samples/sec at 1/2/4/8 B200 (% bf16 TC peak); time to target loss"  # BASELINE.json

CONFIGS = {
    # BASELINE.json configs[3] (default): the >= 60% target config, one worker per GPU
    "realsim": dict(data="realsim", dims=[20958, 4096, 4096, 4096, 4096, 2], N=72309, workers="per_gpu",
                    workload="configs[3]: real-sim-shaped 72309x20958 per GPU (dense bf16), 2 classes, "
                             "MLP 20958-4096x4-2 sigmoid/softmax-CE, Adaptive Hogbatch, one worker per GPU, "
                             "one shared coordinator, batch <= 8192"),
    # configs[1]: the paper's CPU+GPU pairing mapped onto two workers of one GPU
    "covtype": dict(data="covtype", dims=[54, 512, 512, 512, 512, 7], N=581012, workers="large_small",
                    workload="configs[1]: covtype-shaped 581012x54, 7 classes, MLP 54-512x4-7, Adaptive Hogbatch "
                             "with a large-batch and a small-batch worker"),
    # configs[2]
    "w8a": dict(data="w8a", dims=[300, 1024, 1024, 1024, 2], N=64700, workers="large_small",
                workload="configs[2]: w8a-shaped 64700x300, 2 classes, MLP 300-1024x3-2, large-batch + "
                         "small-batch workers"),
    # configs[0]
    "tiny": dict(data="covtype", dims=[54, 64, 64, 7], N=10000, workers="tiny",
                 workload="configs[0]: covtype-shaped 10000x54, MLP 54-64-64-7, mini-batch b = 32"),
}


def flops_per_sample(dims):
    P = sum(dims[i] * dims[i - 1] for i in range(1, len(dims)))
    return 6 * P - 2 * dims[0] * dims[1]


def load_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return dict(hbm=p["hbm_gbs"], bf16=p["bf16_tflops"], bf16_sus=p.get("bf16_tflops_sustained", p["bf16_tflops"]),
                    src="measured")
    except Exception:
        return dict(hbm=6650.0, bf16=1590.0, bf16_sus=1400.0, src="fallback (B200_PROFILING.md)")


class ClockSampler:
    """nvidia-smi clocks/throttle reasons sampled during the timed region (B200_PROFILING.md)."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index, self.lines, self.proc = index, [], None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), "--query-gpu=" + self.Q,
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=2)
        except Exception:
            self.proc.kill()
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                mx = float(f[2])
            except ValueError:
                continue
            for n, v in zip(names, f[5:9]):
                if v.lower() == "active":
                    reasons.add(n)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm)}


# --------------------------------------------------------------------------------------------
# synthetic data (synth/: seeded, shaped like the paper's data sets)
# --------------------------------------------------------------------------------------------
def shard_host(cfg, shard, N):
    """(X float32 [N, ld] zero-padded, y int32) of one shard, or the CSR of sparse-shaped data."""
    from synth import covtype_like, pad_cols
    from synth.data import sparse_like
    d = cfg["dims"][0]
    ld = (d + 7) // 8 * 8
    if cfg["data"] == "covtype":
        X, y = covtype_like(N, seed=shard)
        return ("dense", pad_cols(X, ld)), y
    if cfg["data"] == "w8a":
        csr, y = sparse_like(N, 300, 11.6, 0.03, True, seed=shard)
    else:
        csr, y = sparse_like(N, 20958, 51.5, 0.31, False, seed=shard)
    return ("csr", csr), y


def to_device_dense(kind_x, N, ld, device):
    """Densify on the device ("processed in dense format")."""
    import torch
    kind, x = kind_x
    if kind == "dense":
        return torch.from_numpy(x).to(device).to(torch.bfloat16)
    indptr, indices, vals = x
    Xd = torch.zeros(N, ld, dtype=torch.bfloat16, device=device)
    rows = torch.from_numpy(np.repeat(np.arange(N), np.diff(indptr))).to(device)
    Xd[rows, torch.from_numpy(indices.astype(np.int64)).to(device)] = torch.from_numpy(vals).to(device).to(torch.bfloat16)
    return Xd


# --------------------------------------------------------------------------------------------
# reference arm and cpu_baseline: the fp64 oracle on the host cores (bounded sample)
# --------------------------------------------------------------------------------------------
def oracle_rate(cfg, rows, b, reps, warmup, eta0, b0):
    """samples/s of the fp64 oracle's SGD steps (batch b) over the first `rows` rows of shard 0."""
    from threadpoolctl import threadpool_info
    from oracle import mlp64
    from synth import init_params
    from synth.data import csr_to_dense
    dims = cfg["dims"]
    (kind, x), y = shard_host(cfg, 0, max(rows, 2048))
    X = (x if kind == "dense" else csr_to_dense(x, dims[0]))[:rows, :dims[0]].astype(np.float64)
    y = y[:rows]
    params = init_params(dims, seed=2)
    lr = eta0 * b / b0

    def step(P):
        for s in range(0, rows - b + 1, b):
            P, _ = mlp64.sgd_step(P, X[s:s + b], y[s:s + b], lr)
        return P

    for _ in range(warmup):
        params = step(params)
    times = []
    for _ in range(reps):
        t0 = time.perf_counter()
        params = step(params)
        times.append(time.perf_counter() - t0)
    cores = sum(i.get("num_threads", 0) for i in threadpool_info() if i.get("internal_api") in ("openblas", "mkl")) or 1
    return (rows // b) * b / statistics.mean(times), cores, statistics.mean(times)


def oracle_sample(cfg):
    """bounded sample (~10-30 s of fp64 work on the box's cores): (rows, batch)"""
    if cfg["dims"][1] >= 4096:
        return 8192, 8192   # C4: one 8192-row step (~12 s on 16 cores)
    if cfg["dims"][1] <= 64:
        return 3200, 32     # C1: 100 steps of 32
    return 65536, 8192


# --------------------------------------------------------------------------------------------
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="realsim", choices=list(CONFIGS))
    ap.add_argument("--policy", default="adaptive", choices=["adaptive", "minibatch"])
    ap.add_argument("--eta0", type=float, default=None, help="lr at b0 (default: 0.01 for C4, 0.05 otherwise)")
    ap.add_argument("--b0", type=int, default=32)
    ap.add_argument("--merges", type=int, default=1, help="replica merges per epoch (N > 1, --sync merge)")
    ap.add_argument("--sync", default="merge", choices=["merge", "async"],
                    help="N > 1: NCCL replica merges at the coordinator's merge points, or NEXT f2: every "
                         "update also lands on every peer replica (CUDA IPC peer memory, atomic adds)")
    ap.add_argument("--async-scale", type=float, default=1.0, help="f2: stale-update damping of peer updates")
    ap.add_argument("--n", type=int, default=0, help="rows per GPU (default: the config's N)")
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--opt", action="append", default=[], help="model option key=value (HB_OPT_*, e.g. gemm_pair=1)")
    ap.add_argument("--no-prof", action="store_true")
    ap.add_argument("--ttt-epochs", type=int, default=None,
                    help="epochs per algorithm for time-to-target (0 disables; N=1 only)")
    ap.add_argument("--eta-grid", default="0.001,0.01,0.1,1",
                    help="powers-of-10 learning-rate grid for time-to-target (PAPER.md L258)")
    args = ap.parse_args()
    cfg = CONFIGS[args.config]
    eta0 = args.eta0 if args.eta0 is not None else (0.01 if cfg["dims"][1] >= 4096 else 0.05)
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    Nper = args.n or cfg["N"]
    dims = cfg["dims"]
    F = flops_per_sample(dims)

    if args.impl == "reference":
        # the fp64 oracle on the host cores, as it stands; each step a bounded sample of the workload
        if rank != 0:
            return
        rows, b = oracle_sample(cfg)
        rows, b = (min(rows, 1024), min(b, 1024)) if dims[1] >= 4096 else (rows, b)
        v, cores, t = oracle_rate(cfg, rows, b, args.steps, args.warmup, eta0, args.b0)
        sample = f"fp64 NumPy oracle SGD steps (batch {b}) over the first {rows} rows of shard 0 of the same workload"
        # n_gpus: the N this arm was launched for (the driver pairs the arms by N); the oracle itself
        # runs on the host cores of rank 0 and uses no GPU
        line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "samples/s", "n_gpus": world,
                "device": "host CPU (fp64 oracle, rank 0 only)",
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": t * 1e3, "higher_is_better": True,
                "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
                "config": {"workload": cfg["workload"], "sample_rows_per_step": rows, "batch": b},
                "cpu_baseline": {"value": v, "unit": "samples/s", "cores": cores, "kind": "oracle", "sample": sample},
                "e2e": {"value": v, "unit": "samples/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
        print(json.dumps(line), flush=True)
        return

    import torch
    import torch.distributed as dist
    torch.cuda.set_device(local)
    import paper_conf_ipps_marws21_b200 as hb  # noqa: F811
    from paper_conf_ipps_marws21_b200 import dist as hbd
    hbd.init("nccl", torch.device("cuda", local))
    from synth import init_params, params_to_flat
    dev = torch.device("cuda", local)
    ld = (dims[0] + 7) // 8 * 8

    # ---- data: this rank's shard generated on the host, densified on its GPU; with N > 1 every
    #      GPU holds every shard (all-gather over NVLink): the coordinator's 𝔹 spans all GPUs ----
    xs, y_shard = shard_host(cfg, rank, Nper)
    X_shard = to_device_dense(xs, Nper, ld, dev)
    y_shard_d = torch.from_numpy(y_shard.astype(np.int32)).to(dev)
    N = Nper * world
    if world > 1:
        Xd = torch.empty(N, ld, dtype=torch.bfloat16, device=dev)
        yd = torch.empty(N, dtype=torch.int32, device=dev)
        dist.all_gather_into_tensor(Xd, X_shard)
        dist.all_gather_into_tensor(yd, y_shard_d)
    else:
        Xd, yd = X_shard, y_shard_d
    # e2e inputs of this rank in pinned host memory: the sparse-shaped data sets as CSR (what a
    # user holds — LIBSVM-style rows — densified on the device by hogbatch_run), covtype dense
    y_host = torch.from_numpy(y_shard.astype(np.int32)).pin_memory()
    csr_host = None
    if xs[0] == "csr" and world == 1:
        indptr, indices, vals = xs[1]
        csr_host = hb.CSR(torch.from_numpy(indptr.astype(np.int64)).pin_memory(),
                          torch.from_numpy(indices.astype(np.int32)).pin_memory(),
                          torch.from_numpy(np.asarray(vals, np.float32)).to(torch.bfloat16).pin_memory(), dims[0], ld)
        X_host = None
    else:
        X_host = torch.empty(Nper, ld, dtype=torch.bfloat16, pin_memory=True)
        X_host.copy_(X_shard)
    torch.cuda.synchronize()

    model = hb.MLP(dims, precision="bf16", seed=0, device=local)
    for kv in args.opt:  # per-model launch options (include/hogbatch.h HB_OPT_*)
        k, v = kv.split("=")
        model.set_option(k, int(v))
    params0 = params_to_flat(init_params(dims, seed=2))
    model.set_params(params0)
    big_max = 8192

    # ---- workers and policy ----
    def step_rate(w, b, reps=10, trials=3):
        nb = max(1, N // b - 1)
        for i in range(5):
            w.step(Xd[(i % nb) * b:], yd[(i % nb) * b:], b, 0.0)
        best = 0.0
        for _ in range(trials):
            s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            s0.record()
            for i in range(reps):
                j = i % nb
                w.step(Xd[j * b:], yd[j * b:], b, 0.0)
            s1.record()
            torch.cuda.synchronize()
            best = max(best, b * reps / (s0.elapsed_time(s1) * 1e-3))
        return best

    def lower_threshold(w):
        # smallest power of 2 with >= 50% of the samples/s at the upper threshold (PAPER.md L258
        # "GPU utilization for the lower threshold is about 50%"), on this GPU, outside timing
        r_max = step_rate(w, big_max)
        lo, b = big_max, big_max // 2
        while b >= 64 and step_rate(w, b) >= 0.5 * r_max:
            lo, b = b, b // 2
        return lo

    coord = comm = None
    if cfg["workers"] == "per_gpu":
        wl = hb.Worker(model, big_max)
        workers = [wl]
        if args.policy == "adaptive" and world > 1:
            lo = int(hbd.reduce_scalar(float(lower_threshold(wl)), "max", dev))  # same thresholds on every GPU
            model.set_params(params0)
        else:
            lo = big_max
        specs = [hb.WorkerSpec(lo, big_max, big_max) for _ in range(world)]
        kind = hb.HB_ADAPTIVE if args.policy == "adaptive" else (hb.HB_MINIBATCH if world == 1 else hb.HB_HOGBATCH)
        pol = hb.Policy(kind=kind, workers=specs, eta0=eta0, b0=args.b0, first_worker=rank)
        desc = f"one worker per GPU, b in [{lo}, {big_max}], init {big_max}"
    elif cfg["workers"] == "large_small" and args.policy == "adaptive":
        wl = hb.Worker(model, big_max)
        lo = lower_threshold(wl)
        model.set_params(params0)
        ws = hb.Worker(model, 2048)
        workers = [wl, ws]
        specs = [hb.WorkerSpec(lo, big_max, big_max), hb.WorkerSpec(32, 2048, 32)] * world
        pol = hb.Policy(kind=hb.HB_ADAPTIVE, workers=specs, eta0=eta0, b0=args.b0, first_worker=2 * rank)
        desc = f"large worker [{lo}, {big_max}] init {big_max} + small worker [32, 2048] init 32 per GPU (Hogwild)"
    else:
        bsz = 32 if cfg["workers"] == "tiny" else big_max
        workers = [hb.Worker(model, bsz)]
        specs = [hb.WorkerSpec(bsz, bsz, bsz) for _ in range(world)]
        pol = hb.Policy(kind=hb.HB_MINIBATCH if world == 1 else hb.HB_HOGBATCH, workers=specs, eta0=eta0,
                        b0=args.b0, first_worker=rank)
        desc = f"mini-batch b = {bsz}"
    if world > 1:
        name = hbd.share_bytes(f"/hb_bench_{uuid.uuid4().hex[:12]}".encode() if rank == 0 else None).decode()
        if rank == 0:
            coord = hb.Coord(name, pol, N, world, rank)
        dist.barrier()
        if rank != 0:
            coord = hb.Coord(name, pol, N, world, rank)
        pol.coord = coord
        if args.sync == "merge":
            uid = hbd.share_bytes(hb.Comm.unique_id() if rank == 0 else None)
            comm = hb.Comm(uid, world, rank, local)
            model.merge_begin()
            pol.comm, pol.merges_per_epoch = comm, args.merges
        else:  # f2: asynchronous cross-GPU updates through peer memory (atomic, no merge round)
            handles = [None] * world
            dist.all_gather_object(handles, model.ipc_handle())
            model.set_option("update", hb.HB_UPDATE_ATOMIC)
            model.attach_ipc_peers([h for r, h in enumerate(handles) if r != rank], scale=args.async_scale)

    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)

    def run_epoch(X=Xd, y=yd):
        return hb.hogbatch_run(workers, pol, X, y, epochs=1, n=N)

    for _ in range(args.warmup):
        run_epoch()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clocks = ClockSampler(local)
    clocks.start()
    l0 = hb.kernel_launches()
    ms, samples, share = [], 0, np.zeros(len(specs))
    for _ in range(args.steps):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        e0.record()
        st = run_epoch()
        e1.record()
        torch.cuda.synchronize()
        ms.append(e0.elapsed_time(e1))
        samples += st["total_samples"]
        share += st["updates"][0]
    launches = hb.kernel_launches() - l0
    clk = clocks.stop()
    t_max = hbd.reduce_scalar(sum(ms), "max", dev)            # device ms, max over ranks
    s_tot = hbd.reduce_scalar(float(samples), "sum", dev)     # samples of all ranks
    value = s_tot / (t_max * 1e-3)
    ms_per_step = t_max / args.steps

    # ---- e2e through the public API with HOST inputs: every step the rank's rows are copied from
    #      pinned host memory (H2D; with N > 1 then all-gathered over NVLink so that 𝔹 spans the
    #      GPUs), hogbatch_run trains one epoch, and the trained parameters are read back (D2H) ----
    e2e_ms, e2e_samples, e2e_loss = [], 0, None
    if csr_host is not None:
        h2d = csr_host.indptr.numel() * 8 + csr_host.indices.numel() * 4 + csr_host.values.numel() * 2 + \
            y_host.numel() * 4
    else:
        h2d = X_host.numel() * 2 + y_host.numel() * 4
    d2h = 8 * len(workers)  # the step's result: the epoch's training loss (one fp64 sum per worker)
    if world == 1:   # hogbatch_run stages host data itself (chunked, overlapped; CSR densified on device)
        X_e2e, y_e2e = (csr_host if csr_host is not None else X_host), y_host
    else:
        X_e2e = torch.empty(N, ld, dtype=torch.bfloat16, device=dev)
        y_e2e = torch.empty(N, dtype=torch.int32, device=dev)
        xs_buf = torch.empty(Nper, ld, dtype=torch.bfloat16, device=dev)
        ys_buf = torch.empty(Nper, dtype=torch.int32, device=dev)

    def e2e_step():
        if world == 1:
            st_ = hb.hogbatch_run(workers, pol, X_e2e, y_e2e, epochs=1, train_loss=True)
        else:
            xs_buf.copy_(X_host, non_blocking=True)
            ys_buf.copy_(y_host, non_blocking=True)
            dist.all_gather_into_tensor(X_e2e, xs_buf)
            dist.all_gather_into_tensor(y_e2e, ys_buf)
            torch.cuda.synchronize()
            st_ = hb.hogbatch_run(workers, pol, X_e2e, y_e2e, epochs=1, n=N, train_loss=True)
        return st_

    if args.e2e_steps:
        for _ in range(max(3, args.warmup)):   # untimed, like the device leg's warm-up
            e2e_step()
    for _ in range(args.e2e_steps):
        flush.zero_()
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        st = e2e_step()
        e1.record()
        torch.cuda.synchronize()
        e2e_ms.append(e0.elapsed_time(e1))
        e2e_samples += st["total_samples"]
        e2e_loss = st["train_loss"]
    te = hbd.reduce_scalar(sum(e2e_ms), "max", dev)
    se = hbd.reduce_scalar(float(e2e_samples), "sum", dev)
    e2e_value = se / (te * 1e-3) if args.e2e_steps else None

    # ---- roofline: the same steps re-run SERIALISED (backward overlap off, every launch on the
    #      worker's stream bracketed by CUDA events, graphs off) -> per kernel class and per weight
    #      layer device time; the dominant kernel is judged against its roofline ----
    prof, prof_steps, prof_ms = None, 0, 0.0
    if not args.no_prof:
        model.set_params(params0)
        overlap = model.get_option("bwd_overlap")
        model.set_option("bwd_overlap", 0)
        hb.prof_read(reset=True)
        hb.prof_enable(True)
        prof_steps = max(1, min(args.steps, 3))
        for _ in range(prof_steps):
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            e0.record()
            run_epoch()
            e1.record()
            torch.cuda.synchronize()
            prof_ms += e0.elapsed_time(e1)
        prof = hb.prof_read(reset=True, per_layer=True)
        hb.prof_enable(False)
        model.set_option("bwd_overlap", overlap)

    # ---- time to target loss (PAPER.md L258 methodology; N = 1 only, outside the timing) ----
    ttt = None
    ttt_epochs = args.ttt_epochs if args.ttt_epochs is not None else (10 if dims[1] >= 4096 else 40)
    if ttt_epochs > 0 and world == 1:
        algos = {"minibatch": (hb.HB_MINIBATCH, [workers[0]], [hb.WorkerSpec(big_max, big_max, big_max)])}
        if len(workers) > 1:
            algos["adaptive"] = (hb.HB_ADAPTIVE, workers, specs)
        curves = {}
        for eta in [float(x) for x in args.eta_grid.split(",")]:
            for aname, (kind_, ws_, sp) in algos.items():
                model.set_params(params0)
                p2 = hb.Policy(kind=kind_, workers=sp, eta0=eta, b0=args.b0, eval_loss=True)
                st = hb.hogbatch_run(ws_, p2, Xd, yd, epochs=ttt_epochs)
                curves[(eta, aname)] = (np.cumsum(st["epoch_train_s"]).tolist(), st["epoch_loss"])

        def best(eta):
            return min(min([v for v in curves[(eta, a)][1] if v == v] or [float("inf")]) for a in algos)
        etas = sorted({e for e, _ in curves})
        eta_star = min(etas, key=best)
        l_min = best(eta_star)
        target = 1.1 * l_min
        res = {}
        for a in algos:
            t_cum, ls = curves[(eta_star, a)]
            hit = next((t for t, v in zip(t_cum, ls) if v <= target), None)
            res[a] = {"time_to_target_s": hit, "final_loss": ls[-1] if ls else None,
                      "epoch_loss": [round(x, 5) for x in ls], "epoch_end_s": [round(x, 4) for x in t_cum]}
        ttt = {"eta0": eta_star, "b0": args.b0, "epochs": ttt_epochs, "min_loss": l_min, "target_loss": target,
               "grid": {str(e): round(best(e), 5) for e in etas}, "algorithms": res,
               "method": "same epoch budget per algorithm, eta0 from the powers-of-10 grid with the lowest loss, "
                         "target = 1.1 x min loss across algorithms, training time only (PAPER.md L258, L264)"}
        model.set_params(params0)

    if rank == 0:
        peaks = load_peaks()
        roof = None
        if prof:
            layer_k = {k: v for k, v in prof.items() if "/l" in k and v["ms"] > 0}
            cls_k = {k: v for k, v in prof.items() if "/l" not in k and v["launches"] and v["ms"] > 0}
            pool = dict(layer_k)
            for k, v in cls_k.items():   # classes without per-layer tags (rowchain, softmax, merge)
                if not any(x.startswith(k + "/") for x in layer_k):
                    pool[k] = v
            dom = max(pool, key=lambda k: pool[k]["ms"])
            d = pool[dom]
            ai = d["flops"] / d["bytes"] if d["bytes"] else 0.0
            ridge = peaks["bf16_sus"] * 1e12 / (peaks["hbm"] * 1e9)
            if d["flops"] > 0 and ai >= ridge:
                # each launch of the serialised pass runs alone (nothing concurrent, short bursts
                # between event records): the burst peak is its ceiling (B200_PROFILING.md)
                ach, peak, unit, bound = d["flops"] / (d["ms"] * 1e-3) / 1e12, peaks["bf16"], "TFLOP/s", "tensor"
            else:
                ach, peak, unit, bound = d["bytes"] / (d["ms"] * 1e-3) / 1e9, peaks["hbm"], "GB/s", "hbm"
            traffic = None
            try:
                with open(os.path.join(ROOT, "profiles", "ncu_traffic.json")) as f:
                    tj = json.load(f).get(args.config, {})
                cls_name = dom.split("/")[0]
                t_ent = tj.get(cls_name + "/longest") if dom.endswith("/l0") else tj.get(cls_name)
                traffic = t_ent["dram_bytes"] if isinstance(t_ent, dict) else t_ent
            except Exception:
                pass
            total_cls_ms = sum(v["ms"] for v in cls_k.values())
            roof = {"bound": bound, "achieved": ach, "peak": peak, "unit": unit, "frac": ach / peak,
                    "traffic": traffic, "kernel": dom, "launches": d["launches"],
                    "ms_per_launch": d["ms"] / d["launches"],
                    "flops_per_launch": d["flops"] / d["launches"], "bytes_per_launch": d["bytes"] / d["launches"],
                    "share_of_step": d["ms"] / total_cls_ms if total_cls_ms else None,
                    "peak_source": f"{peaks['src']} ({'bf16_tflops (burst: every launch timed alone)' if bound == 'tensor' else 'hbm_gbs'})",
                    "timing": "serialised profiling pass (one stream, CUDA events around every launch, graphs off), "
                              "outside the timed region",
                    "kernels_ms_per_step": total_cls_ms / prof_steps,
                    "profiled_ms_per_step": prof_ms / prof_steps,
                    "classes": {k: {"ms_per_step": round(v["ms"] / prof_steps, 4), "launches": v["launches"],
                                    "TFLOP/s": round(v["flops"] / (v["ms"] * 1e-3) / 1e12, 1),
                                    "GB/s": round(v["bytes"] / (v["ms"] * 1e-3) / 1e9, 1)}
                                for k, v in sorted(pool.items(), key=lambda kv: -kv[1]["ms"])}}
        cpu = None
        if not args.no_cpu_baseline and world == 1:
            rows, b = oracle_sample(cfg)
            v, cores, t = oracle_rate(cfg, rows, b, 1, 0, eta0, args.b0)
            cpu = {"value": v, "unit": "samples/s", "cores": cores, "kind": "oracle",
                   "sample": f"fp64 NumPy oracle SGD steps (batch {b}) over the first {rows} rows of shard 0 of "
                             f"the same workload, {t:.1f} s"}
        line = {
            "metric": METRIC,
            "value": value, "unit": "samples/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
            "dtype": "bf16", "data": "synthetic",
            "config": {"workload": cfg["workload"], "workers": desc, "rows_per_gpu": Nper, "rows_global": N,
                       "step": "one hogbatch_run epoch over the global data set (one coordinator for all GPUs)",
                       "eta0_at_b0": [eta0, args.b0], "merges_per_epoch": args.merges if world > 1 else 0,
                       "sync": args.sync if world > 1 else None,
                       "l2": "flushed between timed steps (256 MiB write); the data set (3 GB per 72,309 rows) "
                             "exceeds the 126 MB L2"},
            "tc_peak_frac": value * F / (world * peaks["bf16_sus"] * 1e12),
            "flops_per_sample": F,
            "update_share": (share / share.sum()).round(4).tolist() if share.sum() else None,
            "roofline": roof,
            "cpu_baseline": cpu,
            "e2e": {"value": e2e_value, "unit": "samples/s", "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
                    "inputs": "CSR rows in pinned host memory, densified on the device" if csr_host is not None
                    else "dense rows in pinned host memory", "result": "epoch training loss read back",
                    "last_train_loss": e2e_loss},
            "gpu_launches": launches,
            "clocks": clk,
            "time_to_target": ttt,
        }
        print(json.dumps(line), flush=True)
    if comm is not None:
        comm.close()
    if world > 1:
        dist.barrier()
        if args.sync == "async":
            model.attach_ipc_peers([])
            dist.barrier()
        if coord is not None:
            coord.close()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
