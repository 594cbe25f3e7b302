"""Time single tensor-core GEMM launches (hb_bench_gemm) over shapes; prints TFLOP/s."""
import ctypes as C, sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_marws21_b200 as hb
shapes = [(0, 8192, 512, 54), (0, 8192, 512, 512), (0, 8192, 512, 64), (0, 8192, 512, 4096), (0, 8192, 4096, 4096),
          (1, 8192, 512, 512), (1, 8192, 4096, 4096), (2, 512, 512, 8192), (2, 512, 54, 8192), (2, 4096, 4096, 8192),
          (0, 256, 512, 512), (0, 1024, 512, 512), (2, 512, 512, 1024)]
if len(sys.argv) > 1:
    shapes = [tuple(int(x) for x in a.split(',')) for a in sys.argv[1:]]
for kind, M, N, K in shapes:
    us = C.c_float()
    rc = hb.lib.hb_bench_gemm(kind, M, N, K, 20, C.byref(us))
    if rc:
        print(kind, M, N, K, "error", hb.lib.hb_last_error()); continue
    print(f"kind={kind} M={M:6d} N={N:5d} K={K:5d}  {us.value:8.2f} us  {2*M*N*K/us.value/1e6:8.1f} TFLOP/s")
