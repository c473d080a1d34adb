"""GEMM + residual + LayerNorm: fused kernel (op_gemm_ln, cluster st.async row statistics) vs
the residual GEMM followed by the LayerNorm kernel, graph-replayed (20 back-to-back pairs).

    python tools/ln_fusion_bench.py
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icpp_tanlyl024_b200 import arlo  # noqa: E402


def timed(fn, s, reps=20):
    with torch.cuda.stream(s):
        for _ in range(3):
            fn()
        s.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            for _ in range(reps):
                fn()
        g.replay()
        ts = []
        for _ in range(7):
            a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            g.replay()
            e.record(s)
            s.synchronize()
            ts.append(a.elapsed_time(e) * 1e3 / reps)
    return float(np.median(ts))


def main():
    s = torch.cuda.Stream()
    for M, N, K in [(4096, 768, 768), (4096, 768, 3072), (2048, 768, 768), (2048, 768, 3072),
                    (16384, 1024, 1024), (16384, 1024, 4096), (32768, 1024, 4096)]:
        A = torch.randn(M, K, device="cuda").to(torch.bfloat16)
        W = (0.02 * torch.randn(N, K, device="cuda")).to(torch.bfloat16)
        b = torch.zeros(N, device="cuda")
        R = torch.randn(M, N, device="cuda").to(torch.bfloat16)
        g, be = torch.ones(N, device="cuda"), torch.zeros(N, device="cuda")
        Y = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
        X = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
        code = arlo.gemm_tile_choice(M, N, K)
        t_un = {}
        for c in sorted({code, 192 if N % 192 == 0 else 256, -256 if N % 256 == 0 else -192}):
            def unfused(c=c):
                arlo.op_gemm(arlo.BF16, A, W, b, Y, epi=arlo.EPI_BIAS_RESIDUAL, residual=R, force_bn=c, stream=s)
                arlo.op_layernorm(arlo.BF16, Y, g, be, 1e-12, X, stream=s)
            t_un[c] = timed(unfused, s)
        t_g = timed(lambda: arlo.op_gemm(arlo.BF16, A, W, b, Y, epi=arlo.EPI_BIAS_RESIDUAL, residual=R, force_bn=code,
                                         stream=s), s)
        t_f = timed(lambda: arlo.op_gemm_ln(A, W, b, R, g, be, 1e-12, X, stream=s), s)
        best = min(t_un, key=t_un.get)
        print(f"M={M} N={N} K={K}: gemm({code}) {t_g:.2f} us; gemm+LN best {t_un[best]:.2f} us (tile {best}) "
              f"{ {k: round(v, 2) for k, v in t_un.items()} }; fused {t_f:.2f} us", flush=True)


if __name__ == "__main__":
    main()
