"""Cluster replay only (BASELINE configs[3] / [4]): ILP-placed runtimes on G virtual GPUs.

    python tools/cluster_replay.py [base|roberta|ablation|batch1|realloc] [n_requests] [G (realloc)] [load (realloc)]

batch1: the dispatch ablation with the paper's batch-1 runtimes (max_batch = 1, so an
instance's capacity M_i = floor(SLO / latency) and Algorithm 1's congestion P = N/M reaches lambda
near saturation, L215-221, L258), Poisson and MMPP arrivals at 0.7 / 0.9 / 0.97 of saturation.
"""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icpp_tanlyl024_b200 import arlo, replay  # noqa: E402
from paper_conf_icpp_tanlyl024_b200 import workload as wl  # noqa: E402


def main():
    model = sys.argv[1] if len(sys.argv) > 1 else "base"
    ablation = model == "ablation"
    realloc = model == "realloc"
    batch1 = model == "batch1"
    if ablation or realloc or batch1:
        model = "base"
    n = int(sys.argv[2]) if len(sys.argv) > 2 else 6000
    cfg = wl.ROBERTA_LARGE if model == "roberta" else wl.BERT_BASE
    slo = 450.0 if model == "roberta" else 150.0  # PAPER.md:L297 (R uses the BERT-large SLO)
    dev = torch.device("cuda")
    s = torch.cuda.Stream()
    W = arlo.Weights(cfg, arlo.upload_weights(cfg, wl.make_weights(cfg), arlo.BF16, dev), arlo.BF16)
    rts = {}
    for L in wl.RUNTIME_LENGTHS:
        rts[L] = arlo.Runtime(W, L, 1 if batch1 else 32)
        rts[L].set_stream(s)
    if batch1:
        # SLO 150 ms and an SLO scaled to B200 batch-1 latencies (0.4-0.6 ms: about
        # 20x the paper's 3090 figures), where M_i = floor(SLO / latency) is ~20 requests and
        # Algorithm 1's congestion test (P = N/M vs lambda) actually fires
        res = {"model": cfg.name, "note": "batch-1 runtimes (PAPER.md:L282), G = 8 virtual GPUs"}
        for slo_b1 in (slo, 10.0):
            for bursty in (False, True):
                res[f"slo{int(slo_b1)}_" + ("mmpp" if bursty else "poisson")] = replay.dispatch_ablation(
                    arlo, torch, rts, cfg, G=8, n_requests=n, slo_ms=slo_b1, max_batch=1, stream=s,
                    loads=(0.7, 0.9, 0.97, 1.1), bursty=bursty)
        print(json.dumps(res))
        return
    if realloc:
        G = int(sys.argv[3]) if len(sys.argv) > 3 else 8
        load = float(sys.argv[4]) if len(sys.argv) > 4 else 0.9
        res = replay.realloc_replay(arlo, torch, rts, cfg, G=G, window_requests=n // 2, slo_ms=slo, max_batch=32,
                                    stream=s, load=load)
        res["model"] = cfg.name
        print(json.dumps(res))
        return
    if ablation:
        res = replay.dispatch_ablation(arlo, torch, rts, cfg, G=8, n_requests=n, slo_ms=slo, max_batch=32, stream=s)
        res["model"] = cfg.name
        print(json.dumps(res))
        return
    Gs = (8,) if model == "roberta" else (1, 2, 4, 8)
    res = replay.cluster_replay(arlo, torch, rts, cfg, Gs=Gs, n_requests=n, slo_ms=slo, max_batch=32, stream=s)
    res["model"] = cfg.name
    print(json.dumps(res))


if __name__ == "__main__":
    main()
