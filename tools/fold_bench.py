"""Time the LayerNorm-fold GEMM epilogues against the plain ones (graph-replayed, warm L2).

    python tools/fold_bench.py > gpurun_out/fold_bench.txt
Per shape (BERT-base at M = 4096 / 16384): EPI_BIAS vs EPI_LNFOLD (QKV), EPI_BIAS_GELU vs
EPI_LNFOLD_GELU (FFN1), EPI_BIAS_RESID vs EPI_RESID_LN with statistics in and out (out-proj, FFN2),
each at the chooser's tile.
"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icpp_tanlyl024_b200 import arlo  # noqa: E402
from gemm_sweep import time_op  # noqa: E402


def main():
    dev = torch.device("cuda")
    for M in (4096, 16384):
        for (name, N, K, plain, fold) in (("qkv", 2304, 768, 0, 3), ("ffn1", 3072, 768, 1, 4),
                                          ("out", 768, 768, 2, 5), ("ffn2", 768, 3072, 2, 5)):
            A = torch.randn(M, K, device=dev).to(torch.bfloat16)
            W = (0.02 * torch.randn(N, K, device=dev)).to(torch.bfloat16)
            v0 = torch.randn(N, device=dev) * 0.02
            v1 = torch.randn(N, device=dev) * 0.1 + 1
            v2 = torch.randn(N, device=dev) * 0.1
            R = torch.randn(M, N, device=dev).to(torch.bfloat16)
            Hs = N if fold == 5 else K
            st_in = torch.rand(Hs // 32, M, 2, device=dev) + 1
            st_out = torch.zeros(N // 32, M, 2, device=dev)
            out = torch.empty(M, N, device=dev, dtype=torch.bfloat16)
            code = arlo.gemm_tile_choice(M, N, K)
            t0 = time_op(lambda s: arlo.op_gemm(arlo.BF16, A, W, v0, out, epi=plain, residual=R if plain == 2 else None,
                                                 force_bn=code, stream=s))
            t1 = time_op(lambda s: arlo.op_gemm_fold(A, W, v0, out, fold, v1=v1, v2=v2 if fold == 5 else None,
                                                     st_in=st_in, st_out=st_out if fold == 5 else None, eps=1e-12,
                                                     residual=R if fold == 5 else None, force_bn=code, stream=s))
            t2 = time_op(lambda s: arlo.op_gemm_fold(A, W, v0, out, fold, v1=v1, v2=v2 if fold == 5 else None,
                                                     st_in=None if fold == 5 else st_in, st_out=None, eps=1e-12,
                                                     residual=R if fold == 5 else None, force_bn=code, stream=s))
            print(f"M={M:6d} {name:5s} code={code:5d}: plain {t0 * 1e6:7.1f} us  fold {t1 * 1e6:7.1f} us"
                  f"  fold-without-stats-io {t2 * 1e6:7.1f} us", flush=True)


if __name__ == "__main__":
    main()
