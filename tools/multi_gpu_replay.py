"""Arlo on the physical GPUs of this box: ILP placement (arlo_allocate) of the eight BERT-base
runtimes, one instance per GPU, Algorithm 1 dispatch (arlo_dispatch) from one
host dispatcher, one worker thread per GPU (paper_conf_icpp_tanlyl024_b200/cluster.py).
Reports aggregate req/s (saturation: every request queued at t = 0) and a Poisson replay at
`load` x that rate, for Arlo and for ST-512 (every GPU an L = 512 instance).

    python tools/multi_gpu_replay.py [G] [n_requests] [max_batch]     (G defaults to all GPUs)
"""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icpp_tanlyl024_b200 import arlo, cluster, replay  # noqa: E402
from paper_conf_icpp_tanlyl024_b200 import workload as wl  # noqa: E402

SLO_MS = 150.0


def main():
    G = int(sys.argv[1]) if len(sys.argv) > 1 else torch.cuda.device_count()
    n = int(sys.argv[2]) if len(sys.argv) > 2 else 20000
    mb = int(sys.argv[3]) if len(sys.argv) > 3 else 32
    assert G <= torch.cuda.device_count(), f"{G} GPUs requested, {torch.cuda.device_count()} visible"
    cfg = wl.BERT_BASE
    Ls = list(wl.RUNTIME_LENGTHS)
    w = wl.make_weights(cfg)
    lengths = wl.sample_lengths(n, seed=wl.SEED_ARRIVALS + 1)
    ids_all = wl.sample_token_ids(cfg, lengths, 512, seed=wl.SEED_ARRIVALS + 2)
    # offline profile (A4) on GPU 0: forward latency per runtime and batch
    torch.cuda.set_device(0)
    s0 = torch.cuda.Stream()
    W0 = arlo.Weights(cfg, arlo.upload_weights(cfg, w, arlo.BF16, "cuda:0"), arlo.BF16, 0)
    prof = {L: arlo.Runtime(W0, L, mb) for L in Ls}
    for rt in prof.values():
        rt.set_stream(s0)
    lat = replay.profile_runtimes(torch, prof, cfg, mb, s0)
    for rt in prof.values():
        rt.close()
    ideal = wl.ideal_runtime(lengths, Ls)
    shares = [float((ideal == k).mean()) for k in range(len(Ls))]
    caps = [replay.slo_capacity(row, SLO_MS) for row in lat]

    weights = {}

    def build(N_alloc):
        insts = cluster.place(N_alloc, Ls)
        ctx = {}
        for x in insts:
            dev = torch.device("cuda", x.gpu)
            if x.gpu not in weights:
                weights[x.gpu] = arlo.Weights(cfg, arlo.upload_weights(cfg, w, arlo.BF16, dev), arlo.BF16, x.gpu)
            with torch.cuda.device(x.gpu):
                st = torch.cuda.Stream(dev)
                rt = arlo.Runtime(weights[x.gpu], x.L, mb)
                rt.set_stream(st)
                ctx[x.gpu] = (rt, st, torch.empty((mb, x.L), dtype=torch.int32, device=dev),
                              torch.empty((mb,), dtype=torch.int32, device=dev),
                              torch.empty((mb, cfg.num_labels), device=dev),
                              torch.empty((mb, x.L), dtype=torch.int32).pin_memory(),
                              torch.empty((mb,), dtype=torch.int32).pin_memory())
        return insts, ctx

    def executor_for(ctx):
        def run(x, idx):
            rt, st, ids_d, len_d, out_d, ids_h, len_h = ctx[x.gpu]
            k = len(idx)
            ids_h[:k].copy_(torch.from_numpy(np.ascontiguousarray(ids_all[idx, :x.L])))
            len_h[:k].copy_(torch.from_numpy(lengths[idx].astype(np.int32)))
            with torch.cuda.device(x.gpu):
                a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                ids_d[:k].copy_(ids_h[:k], non_blocking=True)  # (on the current stream of that device)
                len_d[:k].copy_(len_h[:k], non_blocking=True)
                torch.cuda.current_stream().synchronize()
                a.record(st)
                rt.enqueue(k, ids_d, len_d, out_d)
                e.record(st)
                e.synchronize()
                return a.elapsed_time(e) / 1e3
        return run

    def serve(N_alloc, arrivals):
        insts, ctx = build(N_alloc)
        dLs = [Ls[k] for k in range(len(Ls)) if N_alloc[k] > 0]
        dcaps = [caps[k] for k in range(len(Ls)) if N_alloc[k] > 0]
        sched = arlo.Scheduler(dLs, [int(N_alloc[k]) for k in range(len(Ls)) if N_alloc[k] > 0], dcaps,
                               0.85, 0.9, 6)
        cl = cluster.Cluster(insts, sched, executor_for(ctx), mb)
        arr_t, done_t, lv = cl.run(arrivals, lengths)
        res = cluster.summarize(arr_t, done_t, lv, dLs, lengths, SLO_MS)
        res["busy_s_per_gpu"] = {str(x.gpu): round(x.busy_s, 4) for x in insts}
        res["instances"] = {str(L): int(N_alloc[k]) for k, L in enumerate(Ls) if N_alloc[k]}
        sched.close()
        for v in ctx.values():
            v[0].close()
        return res

    zero = np.zeros(n)
    out = {"G": G, "requests": n, "max_batch": mb, "slo_ms": SLO_MS,
           "profile_ms_b1_b32": {str(L): [round(lat[k][0], 4), round(lat[k][-1], 4)] for k, L in enumerate(Ls)}}
    st = [0] * (len(Ls) - 1) + [G]
    out["st512_saturation"] = serve(st, zero)
    N, _Q, _M = replay.plan_cluster(arlo, G, Ls, lat, shares, 2.0 * out["st512_saturation"]["req_s"], SLO_MS)
    out["arlo_saturation"] = serve(N, zero)
    rate = 0.7 * out["arlo_saturation"]["req_s"]
    out["arlo_poisson_0.7"] = serve(N, wl.poisson_arrivals(n, rate, seed=wl.SEED_ARRIVALS))
    out["speedup_saturation"] = out["arlo_saturation"]["req_s"] / out["st512_saturation"]["req_s"]
    print(json.dumps(out))


if __name__ == "__main__":
    main()
