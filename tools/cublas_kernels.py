"""Which cuBLAS kernel (tile / cluster shape in its name) torch.matmul picks per GEMM shape, and its
time: the reference point for the tile kernels' shape choices (tools/gemm_sweep.py).

    python tools/cublas_kernels.py > gpurun_out/cublas_kernels.txt
"""
import torch
from torch.profiler import ProfilerActivity, profile

SHAPES = [(m, n, k) for m in (2048, 4096, 8192, 16384) for (n, k) in ((2304, 768), (3072, 768), (768, 3072), (768, 768))]


def main():
    for (M, N, K) in SHAPES:
        A = torch.randn(M, K, device="cuda").to(torch.bfloat16)
        W = torch.randn(N, K, device="cuda").to(torch.bfloat16)
        for _ in range(3):
            torch.matmul(A, W.t())
        torch.cuda.synchronize()
        with profile(activities=[ProfilerActivity.CUDA]) as prof:
            for _ in range(5):
                torch.matmul(A, W.t())
            torch.cuda.synchronize()
        ev = [e for e in prof.events() if e.device_type.name == "CUDA"]
        names = {}
        for e in ev:
            names.setdefault(e.name, []).append(e.device_time)
        for nm, ts in names.items():
            us = sorted(ts)[len(ts) // 2]
            print(f"{M:6d} {N:5d} {K:5d}  {us:7.1f} us  {2 * M * N * K / us / 1e6:6.0f} TF  {nm[:150]}", flush=True)


if __name__ == "__main__":
    main()
