"""Per-CTA phase timeline of one tensor-core GEMM launch (globaltimer ns)."""
import ctypes as C, sys, os
import numpy as np
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_marws21_b200 as hb
names = ["start", "prologue", "first_full", "mma_done", "epi_ready", "tmem_full", "epi_done", "exit",
         "parked", "synced", "reduced", "bias_done"] + [f"mma_issued_t{i}" for i in range(5)] + \
        [f"epi_start_t{i}" for i in range(5)] + [f"epi_done_t{i}" for i in range(5)] + \
        [f"t1_chunk{j}_computed" for j in range(4)] + ["t1_chunk0_loaded"]
for arg in sys.argv[1:]:
    kind, M, N, K = (int(x) for x in arg.split(','))
    cap = 32 * 4096
    buf = (C.c_uint64 * cap)()
    rc = hb.lib.hb_bench_gemm_phases(kind, M, N, K, buf, cap)
    if rc:
        print(arg, "error", hb.lib.hb_last_error()); continue
    a = np.frombuffer(buf, dtype=np.uint64).reshape(-1, 32).astype(np.int64)
    a = a[a[:, 0] > 0]
    t0 = a[:, 0].min()
    rel = a - t0
    rel[a == 0] = -1
    print(f"{arg}: {len(a)} CTAs, kernel span {(a[:, 7].max() - t0)/1000:.2f} us")
    for i, n in enumerate(names):
        v = rel[:, i][rel[:, i] >= 0]
        if len(v):
            print(f"   {n:11s} min {v.min()/1000:7.2f}  med {np.median(v)/1000:7.2f}  max {v.max()/1000:7.2f} us")
