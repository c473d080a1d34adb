"""Trace replay on one GPU: arrivals -> Request Scheduler -> per-length runtimes.

A request stream (Poisson "Twitter-Stable" or MMPP "Twitter-Bursty" arrivals,
PAPER.md:L297; skewed lengths, workload.py) is served by one instance of each
per-length runtime on this GPU.  Dispatch is the paper's Algorithm 1 over the
multi-level queue (arlo_dispatch; lambda 0.85, alpha 0.9,
peek 6, L299).  Each instance's capacity M_i is its max batch that meets the
SLO, from the offline profile ("M_i representing the maximum
capacity within SLO").  The GPU executes one batch at a time (instances on one
GPU are time-multiplexed on a stream; the paper avoids co-location across
GPUs, L155): whenever it is free it serves the instance whose oldest waiting
request arrived first, with up to max_batch of that instance's requests.
Every batch is a real forward (arlo_enqueue); its device time (CUDA events)
advances the replay clock, so latencies = queueing + measured service time.

Host logic only around the runtimes: all compute runs in libarlo's kernels.
"""
from __future__ import annotations

import collections

import numpy as np

from . import workload as wl


def capacities(per_L_ms: dict, slo_ms: float, max_batch: int):
    """M_i: largest profiled batch whose forward latency fits the SLO (>= 1)."""
    caps = {}
    for L, row in per_L_ms.items():
        ok = [b for b, ms in row.items() if ms <= slo_ms]
        caps[L] = max(ok) if ok else 1
    return caps


def replay(arlo, torch, runtimes: dict, cfg, n_requests: int, rate: float, seed: int = wl.SEED_ARRIVALS,
           bursty: bool = False, slo_ms: float = 150.0, max_batch: int = 32, per_L_ms: dict | None = None,
           stream=None):
    """Replay n_requests arriving at `rate` req/s.  Returns per-request records and a summary."""
    Ls = sorted(runtimes)
    dev = torch.device("cuda")
    arrivals = (wl.mmpp_arrivals if bursty else wl.poisson_arrivals)(n_requests, rate, seed=seed)
    lengths = wl.sample_lengths(n_requests, seed=seed + 1)
    per_L_ms = per_L_ms or {L: {b: 1.0 for b in (1, max_batch)} for L in Ls}
    caps = capacities(per_L_ms, slo_ms, max_batch)
    sched = arlo.Scheduler(Ls, [1] * len(Ls), [float(caps[L]) for L in Ls], 0.85, 0.9, 6)
    # device-resident ids for every request at every L it could run on (pre-staged)
    max_len = max(Ls)
    ids_all = wl.sample_token_ids(cfg, lengths, max_len, seed=seed + 2)
    queues = {L: collections.deque() for L in Ls}
    out = torch.empty((max_batch, cfg.num_labels), device=dev)
    bufs = {L: (torch.empty((max_batch, L), dtype=torch.int32, device=dev),
                torch.empty((max_batch,), dtype=torch.int32, device=dev)) for L in Ls}
    t = 0.0  # replay clock (s)
    i = 0
    done = np.zeros(n_requests)
    runtime_of = np.zeros(n_requests, dtype=np.int32)
    busy_s = 0.0
    while i < n_requests or any(queues.values()):
        # admit everything that has arrived by t (Algorithm 1 picks the runtime)
        while i < n_requests and arrivals[i] <= t:
            r, inst = sched.dispatch(int(lengths[i]))
            queues[Ls[r]].append(i)
            runtime_of[i] = r
            i += 1
        ready = [L for L in Ls if queues[L]]
        if not ready:
            t = arrivals[i]
            continue
        L = min(ready, key=lambda x: arrivals[queues[x][0]])  # oldest head request first
        batch = [queues[L].popleft() for _ in range(min(max_batch, len(queues[L])))]
        n = len(batch)
        ids_d, len_d = bufs[L]
        ids_d[:n].copy_(torch.from_numpy(ids_all[batch, :L]))
        len_d[:n].copy_(torch.from_numpy(lengths[batch].astype(np.int32)))
        a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        runtimes[L].enqueue(n, ids_d, len_d, out)
        e.record(stream)
        e.synchronize()
        dt = a.elapsed_time(e) / 1e3
        t += dt
        busy_s += dt
        for j in batch:
            done[j] = t
            sched.complete(int(runtime_of[j]), 0)
    lat_ms = (done - arrivals) * 1e3
    summary = {"requests": n_requests, "offered_rate": rate, "bursty": bursty, "slo_ms": slo_ms,
               "makespan_s": float(done.max() - arrivals[0]),
               "served_rate": float(n_requests / (done.max() - arrivals[0])),
               "gpu_busy_frac": float(busy_s / (done.max() - arrivals[0])),
               "mean_ms": float(lat_ms.mean()), "p98_ms": float(np.percentile(lat_ms, 98)),
               "p99_ms": float(np.percentile(lat_ms, 99)),
               "slo_violations": float((lat_ms > slo_ms).mean()), "capacities": {str(k): v for k, v in caps.items()},
               "per_bucket": {}}
    ideal = wl.ideal_runtime(lengths, Ls)
    for k, L in enumerate(Ls):
        m = ideal == k
        if m.any():
            summary["per_bucket"][str(L)] = {"requests": int(m.sum()), "mean_ms": float(lat_ms[m].mean()),
                                             "p99_ms": float(np.percentile(lat_ms[m], 99)),
                                             "demoted": float((runtime_of[m] != k).mean())}
    sched.close()
    return summary
