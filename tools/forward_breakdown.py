"""Run forwards of one BERT-base (or BERT-large: 4th arg "large") runtime (for an ncu launch list / per-kernel breakdown).

    python tools/forward_breakdown.py L b [reps] [base|large] [default|latency|throughput]
    ncu --profile-from-start off --metrics gpu__time_duration.sum --cache-control none --clock-control none \
        --csv --log-file out.csv python tools/forward_breakdown.py 128 32
    python tools/forward_breakdown.py --summarize out.csv
"""
import collections
import csv
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def summarize(path):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h, data = rows[hi], rows[hi + 1:]
    ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    agg = collections.defaultdict(lambda: [0, 0.0])
    for r in data:
        if len(r) <= vi:
            continue
        name = r[ki].split("(")[0].replace("arlo::<unnamed>::", "").replace("void ", "")[:44]
        v = float(r[vi].replace(",", ""))
        v *= {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0,
              "msecond": 1e3, "ms": 1e3}.get(r[ui], 1.0)
        agg[name][0] += 1
        agg[name][1] += v
    tot = sum(v[1] for v in agg.values())
    for k, v in sorted(agg.items(), key=lambda x: -x[1][1]):
        print(f"{v[1] / tot * 100:6.2f}%  n={v[0]:5d}  avg={v[1] / v[0]:8.2f} us  {k}")
    print(f"total {tot:.1f} us over {sum(v[0] for v in agg.values())} launches")


def main():
    if sys.argv[1] == "--summarize":
        summarize(sys.argv[2])
        return
    import numpy as np
    import torch
    from paper_conf_icpp_tanlyl024_b200 import arlo
    from paper_conf_icpp_tanlyl024_b200 import workload as wl
    L, b = int(sys.argv[1]), int(sys.argv[2])
    reps = int(sys.argv[3]) if len(sys.argv) > 3 else 2
    cfg = wl.BERT_LARGE if len(sys.argv) > 4 and sys.argv[4] == "large" else wl.BERT_BASE
    W = arlo.Weights(cfg, arlo.upload_weights(cfg, wl.make_weights(cfg), arlo.BF16), arlo.BF16)
    fam = {"default": 0, "latency": 1, "throughput": 2}[sys.argv[5] if len(sys.argv) > 5 else "default"]
    rt = arlo.Runtime(W, L, b, fam)
    lens = np.full(b, L, np.int32)
    ids = torch.from_numpy(wl.sample_token_ids(cfg, lens, L)).cuda()
    ld = torch.from_numpy(lens).cuda()
    out = torch.empty((b, cfg.num_labels), device="cuda")
    rt.enqueue(b, ids, ld, out)  # warm-up, outside the profiled range
    torch.cuda.synchronize()
    torch.cuda.cudart().cudaProfilerStart()  # with `ncu --profile-from-start off`: only these forwards
    for _ in range(reps):
        rt.enqueue(b, ids, ld, out)
    torch.cuda.synchronize()
    torch.cuda.cudart().cudaProfilerStop()


if __name__ == "__main__":
    main()
