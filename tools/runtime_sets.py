"""the B200 latency staircase and the runtime-count sweep (Fig. 11,
L369-371 5.2.3: N = 8 vs 16 runtimes).

    python tools/runtime_sets.py staircase        # BERT-base forward latency at L = 16..512 step 16, b = 1, 8, 32
    python tools/runtime_sets.py count [G]        # N in {2, 4, 8, 16} runtimes (step 512/N), ILP on G GPUs
The staircase output includes the runtime set replay.derive_runtime_set() reads off it at b = 1, 8, 32.
Prints one JSON object.
"""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icpp_tanlyl024_b200 import arlo, metrics, replay  # noqa: E402
from paper_conf_icpp_tanlyl024_b200 import workload as wl  # noqa: E402


def staircase(W, cfg, s):
    dev = torch.device("cuda")
    out = {}
    for L in range(16, 513, 16):
        rt = arlo.Runtime(W, L, 32)
        rt.set_stream(s)
        row = {}
        for b in (1, 8, 32):
            lens = np.full(b, L, np.int32)
            ids = torch.from_numpy(wl.sample_token_ids(cfg, lens, L, seed=5)).to(dev)
            ld = torch.from_numpy(lens).to(dev)
            o = torch.empty((b, cfg.num_labels), device=dev)
            for _ in range(3):
                rt.enqueue(b, ids, ld, o)
            ev = []
            for _ in range(10):
                a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(s)
                rt.enqueue(b, ids, ld, o)
                e.record(s)
                ev.append((a, e))
            torch.cuda.synchronize()
            ms = float(np.median([a.elapsed_time(e) for a, e in ev]))
            row[str(b)] = {"ms": ms, "tflops": metrics.forward_flops(cfg, b, L) / (ms / 1e3) / 1e12}
        out[str(L)] = row
        rt.close()
    return out


def count(W, cfg, s, G):
    res = {}
    for n in (2, 4, 8, 16):
        step = 512 // n
        rts = {}
        for k in range(1, n + 1):
            rts[k * step] = arlo.Runtime(W, k * step, 32)
            rts[k * step].set_stream(s)
        r = replay.cluster_replay(arlo, torch, rts, cfg, Gs=(G,), n_requests=4000, slo_ms=150.0, max_batch=32,
                                  stream=s, loads=(0.7, 0.9))
        g = r["per_G"][str(G)]
        res[str(n)] = {"runtimes": sorted(rts), "instances": g["arlo"]["instances"],
                       "saturation_req_s": g["arlo"]["saturation_req_s"],
                       "at_0.7": {k: g["arlo"]["load_sweep"]["points"][0][k] for k in ("offered_req_s", "mean_ms",
                                                                                         "p98_ms", "p99_ms")},
                       "st512_saturation_req_s": g["st512"]["saturation_req_s"]}
        for rt in rts.values():
            rt.close()
    return res


def main():
    mode = sys.argv[1]
    cfg = wl.BERT_BASE
    dev = torch.device("cuda")
    s = torch.cuda.Stream()
    W = arlo.Weights(cfg, arlo.upload_weights(cfg, wl.make_weights(cfg), arlo.BF16, dev), arlo.BF16)
    if mode == "staircase":
        st = staircase(W, cfg, s)
        derived = {b: replay.derive_runtime_set({int(L): row[b]["ms"] for L, row in st.items()}) for b in ("1", "8", "32")}
        print(json.dumps({"staircase_ms": st, "derived_runtime_set_tol5pct": derived}))
    else:
        G = int(sys.argv[2]) if len(sys.argv) > 2 else 16
        print(json.dumps({"runtime_count": count(W, cfg, s, G), "G": G}))


if __name__ == "__main__":
    main()
