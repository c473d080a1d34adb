"""GEMMs of a BERT-base forward in isolation vs chained (12 layers, distinct weights).

    python tools/gemm_chain.py M
Prints per-GEMM device time (graph of 20 identical launches) and the time of a
graph with the 48 chained GEMMs of 12 layers (weights streamed from HBM,
activations handed from one GEMM to the next as in the runtime).
"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icpp_tanlyl024_b200 import arlo  # noqa: E402


def graph_time(fn, reps):
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        fn(s)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for _ in range(reps):
            fn(s)
    g.replay()
    torch.cuda.synchronize()
    best = 1e9
    for _ in range(5):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        g.replay()
        b.record()
        torch.cuda.synchronize()
        best = min(best, a.elapsed_time(b) * 1e3 / reps)
    return best


def main():
    M = int(sys.argv[1]) if len(sys.argv) > 1 else 4096
    H, F, layers = 768, 3072, 12
    dev = torch.device("cuda")
    bf = torch.bfloat16
    X = torch.randn(M, H, device=dev).to(bf)
    O = torch.randn(M, H, device=dev).to(bf)
    QKV = torch.empty(M, 3 * H, device=dev, dtype=bf)
    Y = torch.empty(M, H, device=dev, dtype=bf)
    Fb = torch.empty(M, F, device=dev, dtype=bf)
    Ws = [dict(qkv=(0.02 * torch.randn(3 * H, H, device=dev)).to(bf), o=(0.02 * torch.randn(H, H, device=dev)).to(bf),
               f1=(0.02 * torch.randn(F, H, device=dev)).to(bf), f2=(0.02 * torch.randn(H, F, device=dev)).to(bf))
          for _ in range(layers)]
    bq, bh, bf_ = (torch.zeros(n, device=dev) for n in (3 * H, H, F))
    ops = {
        "qkv": lambda w, s: arlo.op_gemm(arlo.BF16, X, w["qkv"], bq, QKV, epi=0, stream=s),
        "o": lambda w, s: arlo.op_gemm(arlo.BF16, O, w["o"], bh, Y, epi=2, residual=X, stream=s),
        "f1": lambda w, s: arlo.op_gemm(arlo.BF16, X, w["f1"], bf_, Fb, epi=1, stream=s),
        "f2": lambda w, s: arlo.op_gemm(arlo.BF16, Fb, w["f2"], bh, Y, epi=2, residual=X, stream=s),
    }
    flops = {"qkv": 2 * M * 3 * H * H, "o": 2 * M * H * H, "f1": 2 * M * F * H, "f2": 2 * M * F * H}
    tot_iso = 0.0
    for k, fn in ops.items():
        t = graph_time(lambda s: fn(Ws[0], s), 20)
        tot_iso += t
        print(f"{k:4s} isolated {t:8.2f} us  {flops[k] / t / 1e6:7.0f} TF   tile {arlo.gemm_tile_choice(M, *{'qkv': (3 * H, H), 'o': (H, H), 'f1': (F, H), 'f2': (H, F)}[k])}")

    def chain(s):
        for w in Ws:
            for fn in ops.values():
                fn(w, s)
    t = graph_time(chain, 1)
    print(f"chain of {4 * layers} GEMMs: {t:.1f} us vs {layers} x isolated sum {layers * tot_iso:.1f} us "
          f"({sum(flops.values()) * layers / t / 1e6:.0f} TF)")


if __name__ == "__main__":
    main()
