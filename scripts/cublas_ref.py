"""cuBLAS (torch.matmul, bf16 in / bf16 out) time per GEMM shape, for comparison with
scripts/gemm_bench.py.  Args: M,N,K triples (C[M,N] = A[M,K] B[K,N]); random normal inputs."""
import sys
import torch
shapes = [tuple(int(x) for x in a.split(',')) for a in sys.argv[1:]]
for M, N, K in shapes:
    a = torch.randn(M, K, device="cuda", dtype=torch.bfloat16)
    b = torch.randn(K, N, device="cuda", dtype=torch.bfloat16)
    for _ in range(5):
        c = a @ b
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record()
    it = 50
    for _ in range(it):
        c = a @ b
    e1.record()
    torch.cuda.synchronize()
    us = e0.elapsed_time(e1) * 1e3 / it
    print(f"cublas M={M:6d} N={N:5d} K={K:5d}  {us:8.2f} us  {2*M*N*K/us/1e6:8.1f} TFLOP/s")
