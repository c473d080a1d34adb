"""Graph-replayed time of the bf16 attention kernel (20 launches captured back to back).

    python tools/attn_bench.py [B L heads len] ...   (default: the bench's L <= 512 shapes at b = 32)
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icpp_tanlyl024_b200 import arlo  # noqa: E402


def bench(B, L, heads, n, reps=20):
    dev = torch.device("cuda")
    s = torch.cuda.Stream()
    qkv = torch.randn(B * L, 3 * 64 * heads, device=dev).to(torch.bfloat16)
    lens = torch.full((B,), n, dtype=torch.int32, device=dev)
    out = torch.empty(B * L, 64 * heads, device=dev, dtype=torch.bfloat16)
    with torch.cuda.stream(s):
        for _ in range(3):
            arlo.op_attention(arlo.BF16, B, L, heads, qkv, lens, out, stream=s)
        s.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            for _ in range(reps):
                arlo.op_attention(arlo.BF16, B, L, heads, qkv, lens, out, stream=s)
        g.replay()
        ts = []
        for _ in range(10):
            a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            g.replay()
            e.record(s)
            s.synchronize()
            ts.append(a.elapsed_time(e) * 1e3 / reps)
    us = float(np.median(ts))
    exps = B * heads * n * n
    print(f"attention B={B} L={L} heads={heads} len={n}: {us:.2f} us/launch  "
          f"({4 * B * heads * 64 * n * n / us / 1e6:.0f} TF real work, {exps / us / 1e6:.2f} Gexp/ms)")


if __name__ == "__main__":
    a = [int(x) for x in sys.argv[1:]]
    cases = [a[i:i + 4] for i in range(0, len(a), 4)] or [[32, 64, 12, 64], [32, 128, 12, 128], [32, 256, 12, 256],
                                                          [32, 512, 12, 512], [64, 512, 16, 512]]
    for c in cases:
        bench(*c)
