"""Trace replay at the SURVEY §8(d) size: 100k BERT-base requests of the skewed length
distribution on the four per-length runtimes of one B200, dispatched by Algorithm 1
(replay.replay), Poisson ("Twitter-Stable") and MMPP ("Twitter-Bursty") arrivals at 70 % of
the saturation rate measured by the same replay with every request at t = 0.

    python tools/trace_replay_100k.py [n_requests] [--sweep]

--sweep adds the SURVEY §8(d) load sweep: offered rate = f x saturation for f in 0.5 .. 1.0, Poisson and
MMPP arrivals; "req/s at SLO" is the highest offered rate whose p99 latency stays within the 150 ms SLO.
"""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icpp_tanlyl024_b200 import arlo, replay  # noqa: E402
from paper_conf_icpp_tanlyl024_b200 import workload as wl  # noqa: E402


def main():
    args = [a for a in sys.argv[1:] if not a.startswith("--")]
    n = int(args[0]) if args else 100000
    cfg = wl.BERT_BASE
    dev = torch.device("cuda")
    s = torch.cuda.Stream()
    W = arlo.Weights(cfg, arlo.upload_weights(cfg, wl.make_weights(cfg), arlo.BF16, dev), arlo.BF16)
    rts = {}
    for L in (64, 128, 256, 512):
        rts[L] = arlo.Runtime(W, L, 32)
        rts[L].set_stream(s)
    lat = replay.profile_runtimes(torch, rts, cfg, 32, s)
    per_L = {L: {b: lat[k][b - 1] for b in range(1, 33)} for k, L in enumerate(sorted(rts))}
    sat = replay.replay(arlo, torch, rts, cfg, n, 1e9, slo_ms=150.0, max_batch=32, per_L_ms=per_L, stream=s)
    out = {"requests": n, "saturation_req_s": sat["served_rate"], "runtimes": sorted(rts)}
    for bursty in (False, True):
        out["bursty" if bursty else "stable"] = replay.replay(arlo, torch, rts, cfg, n, 0.7 * sat["served_rate"],
                                                              bursty=bursty, slo_ms=150.0, max_batch=32,
                                                              per_L_ms=per_L, stream=s)
    if "--sweep" in sys.argv:
        sweep = {}
        for bursty in (False, True):
            pts = []
            for f in (0.5, 0.7, 0.8, 0.9, 0.95, 1.0):
                r = replay.replay(arlo, torch, rts, cfg, n, f * sat["served_rate"], bursty=bursty, slo_ms=150.0,
                                  max_batch=32, per_L_ms=per_L, stream=s)
                pts.append({"load": f, "offered_req_s": f * sat["served_rate"], "served_req_s": r["served_rate"],
                            "mean_ms": r["mean_ms"], "p99_ms": r["p99_ms"], "slo_violations": r["slo_violations"]})
            ok = [p["offered_req_s"] for p in pts if p["p99_ms"] <= 150.0]
            sweep["bursty" if bursty else "stable"] = {"points": pts, "req_s_at_slo": max(ok) if ok else None}
        out["load_sweep"] = sweep
    print(json.dumps(out))


if __name__ == "__main__":
    main()
