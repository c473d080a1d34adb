"""Forward latency of a few per-L runtimes, for A/B runs of library variants.

    [ARLO_LIB_VARIANT=name] python tools/ab_forward.py [quick]
Prints one line per (model, L, b): median ms of back-to-back graph replays and static TFLOP/s.
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icpp_tanlyl024_b200 import arlo, metrics  # noqa: E402
from paper_conf_icpp_tanlyl024_b200 import workload as wl  # noqa: E402

CASES = [("base", 64, 1), ("base", 128, 1), ("base", 64, 32), ("base", 128, 32), ("base", 256, 32), ("base", 512, 32),
         ("large", 256, 64), ("large", 512, 64)]


def main():
    quick = "quick" in sys.argv
    dev = torch.device("cuda")
    s = torch.cuda.Stream()
    tag = os.environ.get("ARLO_LIB_VARIANT", "default")
    Ws = {}
    for model, L, b in CASES:
        if quick and model == "large":
            continue
        cfg = wl.BERT_LARGE if model == "large" else wl.BERT_BASE
        if model not in Ws:
            Ws[model] = arlo.Weights(cfg, arlo.upload_weights(cfg, wl.make_weights(cfg), arlo.BF16, dev), arlo.BF16)
        rt = arlo.Runtime(Ws[model], L, b)
        rt.set_stream(s)
        lens = np.full(b, L, np.int32)
        ids = torch.from_numpy(wl.sample_token_ids(cfg, lens, L, seed=5)).to(dev)
        ld = torch.from_numpy(lens).to(dev)
        out = torch.empty((b, cfg.num_labels), device=dev)
        for _ in range(5):
            rt.enqueue(b, ids, ld, out)
        reps = 10 if model == "large" else 30
        ts = []
        for _ in range(reps):
            a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            rt.enqueue(b, ids, ld, out)
            e.record(s)
            ts.append((a, e))
        torch.cuda.synchronize()
        ms = float(np.median([a.elapsed_time(e) for a, e in ts]))
        tf = metrics.forward_flops(cfg, b, L) / (ms / 1e3) / 1e12
        print(f"{tag:10s} {model:5s} L={L:3d} b={b:2d}: {ms:8.3f} ms  {tf:7.1f} TF", flush=True)
        rt.close()


if __name__ == "__main__":
    main()
