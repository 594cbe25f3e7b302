"""Summarise an `ncu --set full` capture: per kernel launch its class, duration, DRAM bytes
(dram__bytes_read.sum + dram__bytes_write.sum), tensor-pipe activity and L2 traffic; and record in
profiles/ncu_traffic.json, per workload, the DRAM bytes per launch of every kernel class plus those
of the LONGEST launch of each class (the layer-1 GEMMs of C4 — the kernel bench.py's roofline
reports).  Usage:  python scripts/ncu_traffic.py <report.ncu-rep | raw.csv> <workload-key>
"""
import csv
import io
import json
import os
import subprocess
import sys

rep, config = sys.argv[1], sys.argv[2]
out = open(rep).read() if rep.endswith(".csv") else \
    subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
h = rows[0]


def col(name):
    return h.index(name) if name in h else None


ci = {k: col(k) for k in ["Kernel Name", "Grid Size", "gpu__time_duration.sum", "dram__bytes_read.sum",
                          "dram__bytes_write.sum", "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
                          "lts__t_sectors.sum", "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active"]}
units = rows[1]


def val(r, k):
    i = ci[k]
    if i is None or not r[i]:
        return None
    v = float(r[i].replace(",", ""))
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "usecond": 1e-6, "nsecond": 1e-9,
             "msecond": 1e-3, "us": 1e-6, "ns": 1e-9, "ms": 1e-3, "s": 1.0}.get(units[i], 1)
    return v * scale


# tc_gemm_kernel<BN, A_MN, B_MN, EPI, PAIR>: the epilogue is the FOURTH template argument
EPI = {"0": "fwd_gemm", "1": "head_gemm", "5": "head_gemm", "2": "dgrad_gemm", "3": "wgrad_sgd_gemm",
       "4": "wgrad_sgd_gemm"}


def kernel_class(name):
    if "rowchain" in name:
        return "rowchain"
    if "tc_gemm_kernel" in name:
        args = name.split("<", 1)[1].split(">", 1)[0].split(",")
        return EPI.get(args[3].strip(), "other") if len(args) >= 4 else "other"
    if "softmax_xent" in name:
        return "softmax_xent"
    if "head_fused_kernel" in name:
        return "head_kernel"
    if "head_update_kernel" in name:
        return "wgrad_sgd_gemm"
    return "other"


summary, traffic = [], {}
for r in rows[2:]:
    if ci["Kernel Name"] is None or len(r) <= ci["Kernel Name"]:
        continue
    name = r[ci["Kernel Name"]]
    cls = kernel_class(name)
    rd, wr = val(r, "dram__bytes_read.sum") or 0, val(r, "dram__bytes_write.sum") or 0
    d = dict(kernel=name[:80], grid=r[ci["Grid Size"]] if ci["Grid Size"] is not None else "", cls=cls,
             us=(val(r, "gpu__time_duration.sum") or 0) * 1e6, dram_read=rd, dram_write=wr,
             tensor_pct=val(r, "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed") or 0,
             l2_bytes=(val(r, "lts__t_sectors.sum") or 0) * 32,
             tensor_active=val(r, "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active") or 0)
    summary.append(d)
    traffic.setdefault(cls, []).append(d)
for d in summary:
    print(f"{d['cls']:15s} {d['grid']:14s} {d['us']:9.2f} us  dram {(d['dram_read'] + d['dram_write']) / 1e6:9.2f} MB  "
          f"tensor {d['tensor_pct']:5.1f}% of elapsed ({d['tensor_active']:5.1f}% of active)  "
          f"L2 {d['l2_bytes'] / 1e6:8.1f} MB  {d['kernel']}")
path = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles", "ncu_traffic.json")
allt = json.load(open(path)) if os.path.exists(path) else {}
entry = {}
for k, v in traffic.items():
    entry[k] = sum(x["dram_read"] + x["dram_write"] for x in v) / len(v)
    top = max(v, key=lambda x: x["us"])
    entry[k + "/longest"] = {"dram_bytes": top["dram_read"] + top["dram_write"], "us": top["us"], "grid": top["grid"],
                             "tensor_pct_elapsed": top["tensor_pct"]}
allt[config] = entry
json.dump(allt, open(path, "w"), indent=1)
print("wrote", path, config)
