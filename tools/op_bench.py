"""Graph-replayed device time of the non-GEMM hot-path ops at bench shapes (warm L2).

    python tools/op_bench.py
"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icpp_tanlyl024_b200 import arlo  # noqa: E402
from tools.gemm_sweep import time_op  # noqa: E402


def main():
    dev = torch.device("cuda")
    H = 768
    wp = (0.02 * torch.randn(H, H, device=dev)).to(torch.bfloat16)
    wc = (0.02 * torch.randn(2, H, device=dev)).to(torch.bfloat16)
    bp, bc = torch.zeros(H, device=dev), torch.zeros(2, device=dev)
    for B in (1, 8, 32):
        x = torch.randn(B * 128, H, device=dev).to(torch.bfloat16)
        logits = torch.empty(B, 2, device=dev)
        t = time_op(lambda st: arlo.op_head(arlo.BF16, B, 128, x, wp, bp, wc, bc, logits, stream=st))
        print(f"head (pooler + classifier) B={B:3d} H={H}: {t * 1e6:7.2f} us", flush=True)
    for (M, H) in ((64, 768), (4096, 768), (16384, 768), (32768, 1024)):
        x = torch.randn(M, H, device=dev).to(torch.bfloat16)
        g, bb = torch.ones(H, device=dev), torch.zeros(H, device=dev)
        out = torch.empty_like(x)
        t = time_op(lambda st: arlo.op_layernorm(arlo.BF16, x, g, bb, 1e-12, out, stream=st))
        print(f"layernorm M={M:6d} H={H}: {t * 1e6:7.2f} us  {4 * M * H / t / 1e9:7.0f} GB/s", flush=True)
    for (B, L, heads) in ((1, 64, 12), (32, 64, 12), (32, 128, 12), (32, 256, 12), (16, 512, 12), (64, 128, 16),
                          (64, 256, 16), (64, 512, 16)):
        for n in (L, L // 2 + 1):
            qkv = torch.randn(B * L, 3 * 64 * heads, device=dev).to(torch.bfloat16)
            lens = torch.full((B,), n, dtype=torch.int32, device=dev)
            out = torch.empty(B * L, 64 * heads, device=dev, dtype=torch.bfloat16)
            t = time_op(lambda st: arlo.op_attention(arlo.BF16, B, L, heads, qkv, lens, out, stream=st))
            fl = 4.0 * B * n * n * 64 * heads
            print(f"attention B={B:3d} L={L:3d} heads={heads} len={n:3d}: {t * 1e6:7.2f} us  {fl / t / 1e12:6.0f} TF(real)",
                  flush=True)


if __name__ == "__main__":
    main()
