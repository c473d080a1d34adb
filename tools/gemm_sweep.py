"""Time the tcgen05 GEMM at several shapes / tile choices with CUDA events (warm L2).

    python tools/gemm_sweep.py [force ...]     force: 0 auto, 64/128/256 single CTA, -128/-256 CTA pair
"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icpp_tanlyl024_b200 import arlo  # noqa: E402

SHAPES = [(4096, 2304, 768), (4096, 3072, 768), (4096, 768, 3072), (8192, 8192, 8192), (4096, 4096, 8192),
          (16384, 3072, 768), (16384, 1024, 4096), (16384, 768, 3072), (8192, 2304, 768), (2048, 768, 768),
          (64, 2304, 768), (128, 768, 3072)]


def time_op(fn, reps=20):
    """Average device time per call: `reps` calls captured in one CUDA graph, replayed
    back to back (no host launch gaps inside the timed region)."""
    s = torch.cuda.Stream()
    torch.cuda.synchronize()
    with torch.cuda.stream(s):
        for _ in range(3):
            fn(s)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for _ in range(reps):
            fn(s)
    for _ in range(2):
        g.replay()
    torch.cuda.synchronize()
    best = 1e9
    for _ in range(5):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        g.replay()
        b.record()
        torch.cuda.synchronize()
        best = min(best, a.elapsed_time(b) / 1e3 / reps)
    return best


def main():
    forces = [int(x) for x in sys.argv[1:]] or [0, 256, 192, 128, -256, -192, -128]
    dev = torch.device("cuda")
    for (M, N, K) in SHAPES:
        A = torch.randn(M, K, device=dev).to(torch.bfloat16)
        W = (0.02 * torch.randn(N, K, device=dev)).to(torch.bfloat16)
        b = torch.zeros(N, device=dev)
        out = torch.empty(M, N, device=dev, dtype=torch.bfloat16)
        line = f"{M:6d} {N:5d} {K:5d}:"
        fl = 2.0 * M * N * K
        for f in forces:
            if N % abs(f or 64):
                line += f"  {f:5d}=   n/a  "
                continue
            t = time_op(lambda st: arlo.op_gemm(arlo.BF16, A, W, b, out, epi=0, force_bn=f, stream=st))
            line += f"  {f:5d}={fl / t / 1e12:6.0f}TF"
        t = time_op(lambda st: torch.matmul(A, W.t()))
        line += f"  cublas={fl / t / 1e12:6.0f}TF"
        print(line, flush=True)


if __name__ == "__main__":
    main()
