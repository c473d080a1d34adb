"""Time the tcgen05 GEMM at several shapes / tile choices with CUDA events (warm L2).

    python tools/gemm_sweep.py [--epi E] [--set base|large|small|all] [force ...]
        force: 0 auto, 64/128/192/256 single CTA, -128/-192/-256 CTA pair, 4064/4096/4128 dual
        (single-CTA tiles, two CTAs per SM)
        epi:   0 bias, 1 bias+GELU, 2 bias+residual
"""
import argparse
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icpp_tanlyl024_b200 import arlo  # noqa: E402

SETS = {
    "base": [(4096, 2304, 768), (4096, 3072, 768), (4096, 768, 3072), (4096, 768, 768),
             (16384, 2304, 768), (16384, 3072, 768), (16384, 768, 3072), (16384, 768, 768)],
    "large": [(32768, 3072, 1024), (32768, 4096, 1024), (32768, 1024, 4096), (32768, 1024, 1024),
              (16384, 3072, 1024), (16384, 4096, 1024), (16384, 1024, 4096), (16384, 1024, 1024),
              (8192, 8192, 8192)],
    "small": [(64, 2304, 768), (64, 3072, 768), (64, 768, 3072), (64, 768, 768),
              (128, 2304, 768), (128, 768, 3072), (512, 2304, 768), (512, 768, 3072),
              (128, 3072, 1024), (128, 1024, 4096)],
}
SETS["ffn2_small"] = [(m, 768, 3072) for m in (64, 128, 256, 384, 512)] + [(m, 1024, 4096) for m in (128, 256, 512)]
SETS["mid"] = [(m, n, k) for m in (1024, 2048, 8192) for (n, k) in ((2304, 768), (3072, 768), (768, 3072), (768, 768))]
SETS["all"] = SETS["base"] + SETS["large"] + SETS["small"] + SETS["mid"]


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
    ap = argparse.ArgumentParser()
    ap.add_argument("--epi", type=int, default=0, help="-1: each shape's own BERT epilogue (N = 4K GELU, N <= K residual, else bias)")
    ap.add_argument("--set", default="base")
    ap.add_argument("--no-cublas", action="store_true")
    ap.add_argument("forces", nargs="*", type=int)
    a = ap.parse_args()
    forces = a.forces or [0, 256, 192, 128, -256, -192, -128]
    dev = torch.device("cuda")
    for (M, N, K) in SETS[a.set]:
        epi = a.epi if a.epi >= 0 else (1 if N == 4 * K else 2 if N <= K else 0)
        A = torch.randn(M, K, device=dev).to(torch.bfloat16)
        W = (0.02 * torch.randn(N, K, device=dev)).to(torch.bfloat16)
        b = torch.zeros(N, device=dev)
        R = torch.randn(M, N, device=dev).to(torch.bfloat16) if epi == 2 else None
        out = torch.empty(M, N, device=dev, dtype=torch.bfloat16)
        line = f"{M:6d} {N:5d} {K:5d} epi={epi} choice={arlo.gemm_tile_choice(M, N, K):5d}:"
        fl = 2.0 * M * N * K
        for f in forces:
            bn = f - 4000 if f > 4000 else f - 2000 if f > 2000 else f - 1000 if f > 1000 else abs(f or 64)
            if N % bn:
                line += f"  {f:5d}=   n/a  "
                continue
            t = time_op(lambda st: arlo.op_gemm(arlo.BF16, A, W, b, out, epi=epi, residual=R, force_bn=f, stream=st))
            line += f"  {f:5d}={fl / t / 1e12:5.0f}TF/{t * 1e6:6.1f}us"
        if not a.no_cublas:
            t = time_op(lambda st: torch.matmul(A, W.t()))
            line += f"  cublas={fl / t / 1e12:5.0f}TF/{t * 1e6:6.1f}us"
        print(line, flush=True)


if __name__ == "__main__":
    main()
