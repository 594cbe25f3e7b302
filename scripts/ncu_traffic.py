"""Summarise an `ncu --set full` report: per kernel launch duration, DRAM bytes, tensor-pipe %,
and write profiles/ncu_traffic.json {config: {prof_class: dram_bytes_per_launch}}."""
import csv, io, json, subprocess, sys, os
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
    if i is None: return None
    v = float(r[i].replace(",", ""))
    u = units[i]
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "usecond": 1e-6, "nsecond": 1e-9,
             "msecond": 1e-3, "us": 1e-6, "ns": 1e-9, "ms": 1e-3, "s": 1.0}.get(u, 1)
    return v * scale
EPI = {"0": "fwd_gemm", "5": "head_gemm", "1": "head_gemm", "2": "dgrad_gemm", "3": "wgrad_sgd_gemm", "4": "wgrad_sgd_gemm"}
summary, traffic = [], {}
for r in rows[2:]:
    name = r[ci["Kernel Name"]]
    epi = name.split(">")[0].split(",")[-1].strip() if "tc_gemm" in name else None
    cls = "rowchain" if "rowchain" in name else EPI.get(epi, "other")
    rd, wr = val(r, "dram__bytes_read.sum") or 0, val(r, "dram__bytes_write.sum") or 0
    d = dict(kernel=name[:70], grid=r[ci["Grid Size"]], cls=cls, us=val(r, "gpu__time_duration.sum") * 1e6,
             dram_read=rd, dram_write=wr, tensor_pct=val(r, "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed"),
             l2_bytes=(val(r, "lts__t_sectors.sum") or 0) * 32,
             tensor_active=val(r, "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active") or 0)
    summary.append(d)
    traffic.setdefault(cls, []).append(rd + wr)
for d in summary:
    print(f"{d['cls']:15s} {d['grid']:14s} {d['us']:9.2f} us  dram {(d['dram_read']+d['dram_write'])/1e6:9.2f} MB  "
          f"tensor {d['tensor_pct'] or 0:5.1f}% of elapsed ({d['tensor_active']:5.1f}% of active)  "
          f"L2 {(d['l2_bytes'] or 0) / 1e6:8.1f} MB  {d['kernel']}")
path = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles", "ncu_traffic.json")
allt = json.load(open(path)) if os.path.exists(path) else {}
allt[config] = {k: sum(v) / len(v) for k, v in traffic.items()}
json.dump(allt, open(path, "w"), indent=1)
