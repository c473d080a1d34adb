"""How the L2 state before a timed launch changes the four L=128 b=32 GEMM times (bench roofline leg).

    python tools/roofline_flush.py [reps] [qkv out ffn1 ffn2 tile codes]

Variants, each launch bracketed by CUDA events on the launching stream:
  hot         no flush: A, W and the residual stay in L2 from the previous rep
  wflush      512 MB write (flush.zero_()), then A / residual rewritten (the bench's round-2 leg):
              L2 is left full of DIRTY lines of the flush buffer, which the GEMM's own misses
              must write back
  wrflush     512 MB write, then a 512 MB read (the dirty lines are written back before the
              events), then A / residual rewritten
  prev_ln     wrflush, then the producing LayerNorm kernel of the forward writes A (M x 768)
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icpp_tanlyl024_b200 import arlo  # noqa: E402


def main():
    reps = int(sys.argv[1]) if len(sys.argv) > 1 else 30
    dev = torch.device("cuda:0")
    stream = torch.cuda.Stream(dev)
    torch.cuda.set_stream(stream)
    flush = torch.empty(512 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)
    sink = torch.empty(1, dtype=torch.float32, device=dev)
    M, H, F = 4096, 768, 3072
    shapes = {"qkv": (M, 3 * H, H, arlo.EPI_BIAS), "out_proj": (M, H, H, arlo.EPI_BIAS_RESIDUAL),
              "ffn1": (M, F, H, arlo.EPI_BIAS_GELU), "ffn2": (M, H, F, arlo.EPI_BIAS_RESIDUAL)}
    codes = [int(c) for c in sys.argv[2:6]] if len(sys.argv) > 5 else [0, 0, 0, 0]
    g = torch.Generator(device=dev).manual_seed(0)
    for (name, (m, n, k, epi)), code in zip(shapes.items(), codes):
        A = torch.randn(m, k, device=dev, generator=g).to(torch.bfloat16)
        Wt = (0.02 * torch.randn(n, k, device=dev, generator=g)).to(torch.bfloat16)
        bias = torch.zeros(n, device=dev)
        res = torch.randn(m, n, device=dev, generator=g).to(torch.bfloat16) if epi == arlo.EPI_BIAS_RESIDUAL else None
        out = torch.empty(m, n, device=dev, dtype=torch.bfloat16)
        A0, R0 = A.clone(), (res.clone() if res is not None else None)
        gam, bet = torch.ones(k, device=dev), torch.zeros(k, device=dev)
        for _ in range(3):
            arlo.op_gemm(arlo.BF16, A, Wt, bias, out, epi=epi, residual=res, force_bn=code, stream=stream)
        row = []
        for variant in ("hot", "wflush", "wrflush", "prev_ln"):
            ts = []
            for _ in range(reps):
                if variant != "hot":
                    flush.zero_()
                    if variant in ("wrflush", "prev_ln"):
                        sink.copy_(flush.sum().view(1))
                    if variant == "prev_ln" and k == H:
                        arlo.op_layernorm(arlo.BF16, A0, gam, bet, 1e-12, A, stream=stream)
                    else:
                        A.copy_(A0)
                    if res is not None:
                        res.copy_(R0)
                a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(stream)
                arlo.op_gemm(arlo.BF16, A, Wt, bias, out, epi=epi, residual=res, force_bn=code, stream=stream)
                e.record(stream)
                torch.cuda.synchronize()
                ts.append(a.elapsed_time(e) * 1e3)
            t = float(np.mean(ts))
            row.append(f"{variant}={t:6.2f}us/{2 * m * n * k / t / 1e6:5.0f}TF")
        print(f"{name:9s} code={code:5d}  " + "  ".join(row), flush=True)


if __name__ == "__main__":
    main()
