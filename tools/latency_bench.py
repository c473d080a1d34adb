"""Batch-1 latency of the two runtime families and the split-K GEMMs at small M.

    python tools/latency_bench.py [bert-base|bert-large] [families,...] > gpurun_out/latency.json

Per runtime L: median of 50 graph replays (CUDA events per replay) of a b = 1 forward in
the latency family (LayerNorm fold), the throughput family (bucket 1 of a max_batch = 32
runtime), the split-K family and, at L <= 128, the fused family (one persistent kernel).  Per GEMM shape at M = 64: the split-K kernel vs the skinny /
tile kernel the chooser picks, as weight-streaming bandwidth (weight bytes / time) with
the weights cold (L2 flushed before each launch) and the activations warm.
"""
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_icpp_tanlyl024_b200 import arlo, workload as wl  # noqa: E402


def time_forward(rt, cfg, L, n, stream, reps=50):
    lens = np.full(n, L, np.int32)
    ids = torch.from_numpy(wl.sample_token_ids(cfg, lens, L, seed=5)).cuda()
    ld = torch.from_numpy(lens).cuda()
    o = torch.empty((n, 2), device="cuda")
    for _ in range(5):
        rt.enqueue(n, ids, ld, o)
    ev = []
    for _ in range(reps):
        a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        rt.enqueue(n, ids, ld, o)
        e.record(stream)
        ev.append((a, e))
    torch.cuda.synchronize()
    return float(np.median([a.elapsed_time(e) for a, e in ev]))


def time_gemm(M, N, K, epi, code, stream, flush, reps=30):
    A = torch.randn(M, K, device="cuda").to(torch.bfloat16)
    W = (0.02 * torch.randn(N, K, device="cuda")).to(torch.bfloat16)
    b = torch.zeros(N, device="cuda")
    R = torch.randn(M, N, device="cuda").to(torch.bfloat16) if epi == 2 else None
    out = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
    A2 = A.clone()
    for _ in range(3):
        arlo.op_gemm(arlo.BF16, A, W, b, out, epi=epi, residual=R, force_bn=code, stream=stream)
    ev = []
    for _ in range(reps):
        flush.zero_()
        A.copy_(A2)  # the predecessor's output is L2-resident, the weights are not
        a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        arlo.op_gemm(arlo.BF16, A, W, b, out, epi=epi, residual=R, force_bn=code, stream=stream)
        e.record(stream)
        ev.append((a, e))
    torch.cuda.synchronize()
    us = 1e3 * float(np.median([a.elapsed_time(e) for a, e in ev]))
    return {"us": us, "weight_GBps": N * K * 2 / (us * 1e-6) / 1e9}


def main():
    name = sys.argv[1] if len(sys.argv) > 1 else "bert-base"
    cfg = wl.CONFIGS[name]
    stream = torch.cuda.Stream()
    torch.cuda.set_stream(stream)
    flush = torch.empty(256 * 1024 * 1024 // 4, device="cuda")
    W = arlo.Weights(cfg, arlo.upload_weights(cfg, wl.make_weights(cfg), arlo.BF16), arlo.BF16)
    out = {"config": name, "forward_ms": {}, "gemm_M64": {}}
    for L in ((64, 128, 256, 512) if name == "bert-base" else (128, 256, 512)):
        row = {}
        fams = [("latency", 1, arlo.RUNTIME_LATENCY), ("throughput", 32, arlo.RUNTIME_THROUGHPUT),
                ("splitk", 1, arlo.RUNTIME_SPLITK)]
        if L <= 128:
            fams.append(("fused", 1, arlo.RUNTIME_FUSED))
        if len(sys.argv) > 2:
            fams = [f for f in fams if f[0] in sys.argv[2].split(",")]
        for fam, mb, code in fams:
            rt = arlo.Runtime(W, L, mb, code)
            rt.set_stream(stream)
            row[fam] = time_forward(rt, cfg, L, 1, stream)
            row[fam + "_tiles"] = rt.gemm_tiles(1)
            rt.close()
        out["forward_ms"][str(L)] = row
    H, F = cfg.hidden, cfg.ffn
    weight_bytes = cfg.layers * 2 * (3 * H * H + H * H + 2 * H * F)
    out["layer_weight_bytes_total"] = weight_bytes
    for nm, (N, K, epi) in {"qkv": (3 * H, H, 0), "out_proj": (H, H, 2), "ffn1": (F, H, 1),
                            "ffn2": (H, F, 2)}.items():
        out["gemm_M64"][nm] = {"splitk": time_gemm(64, N, K, epi, arlo.SPLITK_CODE + 32, stream, flush),
                               "chooser": time_gemm(64, N, K, epi, 0, stream, flush),
                               "chooser_code": arlo.gemm_tile_choice(64, N, K)}
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
