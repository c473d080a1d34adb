"""Run one cuBLAS bf16 GEMM (torch.matmul) at a given shape, for ncu kernel-name / metric comparison.
    python tools/cublas_probe.py M N K"""
import sys
import torch
M, N, K = (int(x) for x in sys.argv[1:4])
A = torch.randn(M, K, device="cuda", dtype=torch.bfloat16)
W = torch.randn(N, K, device="cuda", dtype=torch.bfloat16)
for _ in range(5):
    C = A @ W.t()
torch.cuda.synchronize()
