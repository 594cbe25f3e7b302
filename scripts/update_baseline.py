"""the fused dW + SGD epilogue against the unfused baseline — the dW GEMM storing the
fp32 gradient (kind 3) plus a standalone update kernel (W -= lr G, shadow rewritten; 14 B per
weight) — for the C4 layer-1 and hidden dW shapes (tuning build, HB_GEMM_PAIR=1 as in the product).
Prints one JSON line per shape."""
import ctypes as C
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_marws21_b200 as hb  # noqa: E402

HBM = 6551.0  # GB/s, MEASURED_PEAKS.json hbm_gbs
for name, (M, N, K) in {"C4 layer-1 dW": (4096, 20958, 8192), "C4 hidden dW": (4096, 4096, 8192),
                        "C3 hidden dW": (1024, 1024, 8192)}.items():
    t = {}
    for kind in (2, 3):
        us = C.c_float()
        rc = hb.lib.hb_bench_gemm(kind, M, N, K, 10, C.byref(us))
        t[kind] = us.value if rc == 0 else float("nan")
    n = M * ((N + 7) // 8 * 8)
    us = C.c_float()
    hb.lib.hb_bench_sgd_apply(n, 10, C.byref(us))
    upd = us.value
    print(json.dumps({"shape": name, "M": M, "N": N, "K": K, "fused_dW_sgd_us": round(t[2], 1),
                      "dW_store_us": round(t[3], 1), "update_kernel_us": round(upd, 1),
                      "update_kernel_GBps": round(14.0 * n / (upd * 1e-6) / 1e9, 1),
                      "update_frac_of_hbm": round(14.0 * n / (upd * 1e-6) / 1e9 / HBM, 3),
                      "unfused_total_us": round(t[3] + upd, 1),
                      "fused_saves_us": round(t[3] + upd - t[2], 1)}), flush=True)
