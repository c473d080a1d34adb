"""Launch one hot-path kernel at a bench shape a few times (for ncu --set full captures).

    python tools/profile_ops.py gemm M N K epi [code]  # tcgen05 GEMM (epi 0 bias, 1 gelu, 2 residual; tile code)
    python tools/profile_ops.py attn B L heads len  # masked attention, all lengths = len
    python tools/profile_ops.py ln M H              # LayerNorm
    python tools/profile_ops.py embed B L           # embedding + LN (BERT-base tables)
    python tools/profile_ops.py head B L            # CLS pooler + classifier (BERT-base)
"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icpp_tanlyl024_b200 import arlo  # noqa: E402


def main():
    op = sys.argv[1]
    a = [int(x) for x in sys.argv[2:]]
    dev = torch.device("cuda")
    reps = 5
    if op == "gemm":
        M, N, K, epi = a[:4]
        code = a[4] if len(a) > 4 else 0
        A = torch.randn(M, K, device=dev).to(torch.bfloat16)
        W = (0.02 * torch.randn(N, K, device=dev)).to(torch.bfloat16)
        b = torch.zeros(N, device=dev)
        R = torch.randn(M, N, device=dev).to(torch.bfloat16)
        out = torch.empty(M, N, device=dev, dtype=torch.bfloat16)
        for _ in range(reps):
            arlo.op_gemm(arlo.BF16, A, W, b, out, epi=epi, residual=R if epi == 2 else None, force_bn=code)
    elif op == "attn":
        B, L, heads, n = a
        qkv = torch.randn(B * L, 3 * 64 * heads, device=dev).to(torch.bfloat16)
        lens = torch.full((B,), n, dtype=torch.int32, device=dev)
        out = torch.empty(B * L, 64 * heads, device=dev, dtype=torch.bfloat16)
        for _ in range(reps):
            arlo.op_attention(arlo.BF16, B, L, heads, qkv, lens, out)
    elif op == "ln":
        M, H = a
        x = torch.randn(M, H, device=dev).to(torch.bfloat16)
        g, bb = torch.ones(H, device=dev), torch.zeros(H, device=dev)
        out = torch.empty_like(x)
        for _ in range(reps):
            arlo.op_layernorm(arlo.BF16, x, g, bb, 1e-12, out)
    elif op == "embed":
        B, L = a
        H, V = 768, 30522
        ids = torch.randint(0, V, (B, L), dtype=torch.int32, device=dev)
        lens = torch.full((B,), L, dtype=torch.int32, device=dev)
        word = torch.randn(V, H, device=dev).to(torch.bfloat16)
        pos = torch.randn(512, H, device=dev).to(torch.bfloat16)
        typ = torch.randn(2, H, device=dev).to(torch.bfloat16)
        g, bb = torch.ones(H, device=dev), torch.zeros(H, device=dev)
        out = torch.empty(B * L, H, device=dev, dtype=torch.bfloat16)
        for _ in range(reps):
            arlo.op_embed(arlo.BF16, ids, lens, word, pos, typ, g, bb, 1e-12, out)
    elif op == "head":
        B, L = a
        H = 768
        x = torch.randn(B * L, H, device=dev).to(torch.bfloat16)
        wp = (0.02 * torch.randn(H, H, device=dev)).to(torch.bfloat16)
        wc = (0.02 * torch.randn(2, H, device=dev)).to(torch.bfloat16)
        bp, bc = torch.zeros(H, device=dev), torch.zeros(2, device=dev)
        logits = torch.empty(B, 2, device=dev)
        for _ in range(reps):
            arlo.op_head(arlo.BF16, B, L, x, wp, bp, wc, bc, logits)
    torch.cuda.synchronize()


if __name__ == "__main__":
    main()
