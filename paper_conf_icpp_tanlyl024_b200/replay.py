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


def derive_runtime_set(curve: dict, tol: float = 0.05, max_len: int = 512):
    """Runtime max_lengths from a latency staircase (§3.3: within one step the
    latency changes < 5 %, so a runtime per step): walk L upwards from the start of the current
    step; when lat(L) exceeds (1 + tol) * lat(step start) the previous L ends the step and
    becomes a runtime.  curve: {L: latency}.  The last runtime is max_len (Eq. 7)."""
    Ls = sorted(int(k) for k in curve)
    out, start, prev = [], Ls[0], Ls[0]
    for L in Ls[1:]:
        if curve[L] > (1.0 + tol) * curve[start]:
            out.append(prev)
            start = L
        prev = L
    if not out or out[-1] != max_len:
        out.append(max_len)
    return out


def capacities(per_L_ms: dict, slo_ms: float, max_batch: int):
    """M_i per runtime for Algorithm 1's congestion P = N / M, the same reading
    as the cluster replays (reading S18, slo_capacity): the requests one instance finishes inside one
    SLO window with every batch meeting the SLO.  per_L_ms[L] = {batch: profiled latency ms}; batches
    missing from the profile are interpolated linearly (reading S15)."""
    caps = {}
    for L, row in per_L_ms.items():
        bs = sorted(row)
        lat = np.interp(np.arange(1, max_batch + 1), bs, [row[b] for b in bs])
        caps[L] = slo_capacity(lat, slo_ms)
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


# ----------------------------------------------------------------------------------------------
# Cluster replay: G GPUs, runtime instances placed by the Runtime Scheduler (arlo_allocate,
# PAPER.md:L181-203 §3.3), one instance per GPU (no co-location, L155), requests routed by the
# Request Scheduler (Algorithm 1).  Instances are independent replicas (north_star: no
# collective), so a G-GPU cluster is simulated exactly by G virtual device clocks: every batch is
# executed for real on this process's GPU (service_fn) and its measured device time advances the
# clock of the virtual GPU that owns the instance.  Discrete-event simulation: arrivals and batch
# completions are processed in time order, so Algorithm 1 sees the outstanding counts it would
# see online.


def slo_capacity(lat_ms_row, slo_ms: float) -> float:
    """M_i ("maximum capacity within SLO"): the most requests one instance can finish
    inside one SLO window while each of its batches meets the SLO: max_b b * floor(SLO / lat(b))
    over the profiled batch sizes (reading of an unstated definition)."""
    best = 0.0
    for b, ms in enumerate(lat_ms_row, start=1):
        if ms <= slo_ms:
            best = max(best, b * np.floor(slo_ms / ms))
    return max(best, 1.0)


def plan_cluster(arlo, G: int, Ls, lat_ms, shares, rate: float, slo_ms: float):
    """Runtime Scheduler inputs and decision for G GPUs.  lat_ms[i][b-1]: profiled forward latency
    of runtime i at batch b; shares[i]: fraction of requests whose ideal runtime is i; rate: offered
    req/s.  Q_i = requests per SLO window in bin i; M_i = slo_capacity.  Returns (N, Q, M)."""
    lat = np.asarray(lat_ms, np.float64)
    M = np.array([slo_capacity(row, slo_ms) for row in lat])
    # Eq. 3 (N_i >= floor(Q_i / M_i)) with Eq. 7 can need more than G GPUs at a high offered
    # rate (EINFEASIBLE): plan for the highest rate the G GPUs can hold, lowering it by 10 % steps
    for _ in range(200):
        Q = np.asarray(shares, np.float64) * rate * slo_ms / 1e3
        try:
            N, _obj = arlo.allocate(G, Q, M, lat)
            return list(N), Q, M
        except arlo.ArloError as e:
            if e.code != arlo.EINFEASIBLE:
                raise
            rate *= 0.9
    raise RuntimeError(f"no feasible allocation on {G} GPUs")


def simulate_cluster(arrivals, lengths, Ls, n_inst, capacity, service_fn, max_batch: int,
                     sched_factory, lam: float = 0.85, alpha: float = 0.9, peek: int = 6):
    """Discrete-event replay of requests (arrivals [s], lengths) on the instances n_inst[i] of
    runtimes Ls[i] (each instance = one GPU).  service_fn(L, idx) -> seconds for a batch of request
    indices idx on runtime L.  sched_factory(max_len, n_inst, capacity, lam, alpha, peek) builds the
    Request Scheduler (arlo.Scheduler, or a test double).  Returns (done_s, runtime_of, busy_s)."""
    import heapq
    deployed = [k for k in range(len(Ls)) if n_inst[k] > 0]
    dLs = [Ls[k] for k in deployed]
    sched = sched_factory(dLs, [n_inst[k] for k in deployed], [float(capacity[k]) for k in deployed],
                          lam, alpha, peek)
    n = len(arrivals)
    queues = {(r, j): collections.deque() for r in range(len(dLs)) for j in range(n_inst[deployed[r]])}
    busy_until = {key: None for key in queues}
    done = np.zeros(n)
    runtime_of = np.zeros(n, np.int32)
    inst_of = np.zeros(n, np.int32)
    busy_s = {key: 0.0 for key in queues}
    # (time, kind, seq, payload); at equal times: 0 completion, 1 arrival, 2 start of an idle instance
    # (deferred so a batch takes every request that has arrived by its start time)
    events = []
    seq = 0
    for i in range(n):
        heapq.heappush(events, (float(arrivals[i]), 1, seq, i))
        seq += 1

    def start(key, t):
        nonlocal seq
        q = queues[key]
        batch = [q.popleft() for _ in range(min(max_batch, len(q)))]
        dt = service_fn(dLs[key[0]], batch)
        busy_s[key] += dt
        busy_until[key] = t + dt
        heapq.heappush(events, (t + dt, 0, seq, (key, batch)))
        seq += 1

    while events:
        t, kind, _s, payload = heapq.heappop(events)
        if kind == 1:
            i = payload
            r, j = sched.dispatch(int(lengths[i]))
            runtime_of[i], inst_of[i] = deployed[r], j
            queues[(r, j)].append(i)
            if busy_until[(r, j)] is None:
                busy_until[(r, j)] = t  # start pending
                heapq.heappush(events, (t, 2, seq, (r, j)))
                seq += 1
        elif kind == 2:
            start(payload, t)
        else:
            key, batch = payload
            for i in batch:
                done[i] = t
                sched.complete(key[0], key[1])
            busy_until[key] = None
            if queues[key]:
                start(key, t)
    sched.close()
    return done, runtime_of, inst_of, busy_s


def summarize(arrivals, lengths, done, runtime_of, Ls, slo_ms: float):
    lat_ms = (done - arrivals) * 1e3
    span = float(done.max() - arrivals.min())
    out = {"requests": int(len(arrivals)), "served_rate": float(len(arrivals) / span), "makespan_s": span,
           "mean_ms": float(lat_ms.mean()), "p98_ms": float(np.percentile(lat_ms, 98)),
           "p99_ms": float(np.percentile(lat_ms, 99)), "slo_violations": float((lat_ms > slo_ms).mean()),
           "per_bucket": {}}
    ideal = wl.ideal_runtime(lengths, Ls)
    out["demoted"] = float((runtime_of != ideal).mean())  # served by a longer runtime than its ideal one
    for k, L in enumerate(Ls):
        m = ideal == k
        if m.any():
            out["per_bucket"][str(L)] = {"requests": int(m.sum()), "mean_ms": float(lat_ms[m].mean()),
                                         "p99_ms": float(np.percentile(lat_ms[m], 99)),
                                         "demoted": float((runtime_of[m] != k).mean())}
    return out


def profile_runtimes(torch, runtimes: dict, cfg, max_batch: int, stream, reps: int = 5):
    """lat_ms[i][b-1], b = 1..max_batch: device time of one forward (a batch of b pads to the
    runtime's bucket, so b is timed at every bucket size and assigned to the b it covers)."""
    dev = torch.device("cuda")
    table = []
    for L in sorted(runtimes):
        rt = runtimes[L]
        row = [0.0] * max_batch
        lens = np.full(max_batch, L, np.int32)
        ids = torch.from_numpy(wl.sample_token_ids(cfg, lens, L, seed=5)).to(dev)
        ld = torch.from_numpy(lens).to(dev)
        out = torch.empty((max_batch, cfg.num_labels), device=dev)
        cache = {}
        for b in range(1, max_batch + 1):
            bucket = rt.bucket_of(b)
            if bucket not in cache:
                for _ in range(2):
                    rt.enqueue(bucket, ids, ld, out)
                ev = []
                for _ in range(reps):
                    a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    a.record(stream)
                    rt.enqueue(bucket, ids, ld, out)
                    e.record(stream)
                    ev.append((a, e))
                torch.cuda.synchronize()
                cache[bucket] = float(np.median([a.elapsed_time(e) for a, e in ev]))
            row[b - 1] = cache[bucket]
        table.append(row)
    return table


def cluster_replay(arlo, torch, runtimes: dict, cfg, Gs=(1, 2, 4, 8), n_requests: int = 8000,
                   slo_ms: float = 150.0, max_batch: int = 32, stream=None, load: float = 0.7,
                   loads=(0.5, 0.7, 0.9, 0.97)):
    """Aggregate req/s and latency of Arlo (ILP placement + Algorithm 1 over len(runtimes) runtimes)
    and of ST (every GPU an L = max runtime instance) on G = 1, 2, 4, 8 GPUs.
    Saturation replay (all requests at t = 0) gives req/s; Poisson replays at `loads` x that rate
    give mean / p98 / p99 latency (per length bucket at `load`) and req/s at SLO.
    Service times are real forwards on this GPU."""
    Ls = sorted(runtimes)
    dev = torch.device("cuda")
    lat = profile_runtimes(torch, runtimes, cfg, max_batch, stream)
    lengths = wl.sample_lengths(n_requests, seed=wl.SEED_ARRIVALS + 1)
    ids_all = wl.sample_token_ids(cfg, lengths, max(Ls), seed=wl.SEED_ARRIVALS + 2)
    ideal = wl.ideal_runtime(lengths, Ls)
    shares = [float((ideal == k).mean()) for k in range(len(Ls))]
    caps = [slo_capacity(row, slo_ms) for row in lat]
    bufs = {L: (torch.empty((max_batch, L), dtype=torch.int32, device=dev),
                torch.empty((max_batch,), dtype=torch.int32, device=dev)) for L in Ls}
    out = torch.empty((max_batch, cfg.num_labels), device=dev)

    def service(L, batch):
        n = len(batch)
        ids_d, len_d = bufs[L]
        ids_d[:n].copy_(torch.from_numpy(np.ascontiguousarray(ids_all[batch, :L])))
        len_d[:n].copy_(torch.from_numpy(lengths[batch].astype(np.int32)))
        a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        runtimes[L].enqueue(n, ids_d, len_d, out)
        e.record(stream)
        e.synchronize()
        return a.elapsed_time(e) / 1e3

    def factory(max_len, n_inst, capacity, lam, alpha, peek):
        return arlo.Scheduler(max_len, n_inst, capacity, lam, alpha, peek)

    def run(n_inst, arrivals):
        done, rof, _inst, busy = simulate_cluster(arrivals, lengths, Ls, n_inst, caps, service, max_batch, factory)
        return summarize(arrivals, lengths, done, rof, Ls, slo_ms)

    res = {"runtimes": Ls, "requests": n_requests, "slo_ms": slo_ms, "capacity_per_slo_window": caps,
           "profile_ms": {str(L): {str(b): round(lat[k][b - 1], 4) for b in (1, 2, 4, 8, 16, 32) if b <= max_batch}
                          for k, L in enumerate(Ls)}, "per_G": {}}
    zero = np.zeros(n_requests)
    for G in Gs:
        st = [0] * (len(Ls) - 1) + [G]
        st_sat = run(st, zero)
        # plan Arlo at twice the rate ST saturates at, measure its saturation, re-plan at load x that
        N, Q, M = plan_cluster(arlo, G, Ls, lat, shares, 2.0 * st_sat["served_rate"], slo_ms)
        arlo_sat = run(N, zero)
        N, Q, M = plan_cluster(arlo, G, Ls, lat, shares, load * arlo_sat["served_rate"], slo_ms)
        arlo_sat = run(N, zero)
        # load sweep (Poisson arrivals): req/s at SLO = highest offered rate whose p99 <= SLO
        sweep = {}
        for name, n_inst, sat in (("arlo", N, arlo_sat["served_rate"]), ("st512", st, st_sat["served_rate"])):
            pts = []
            for f in loads:
                r = run(n_inst, wl.poisson_arrivals(n_requests, f * sat, seed=wl.SEED_ARRIVALS))
                pts.append({"load": f, "offered_req_s": f * sat, "mean_ms": r["mean_ms"], "p98_ms": r["p98_ms"],
                            "p99_ms": r["p99_ms"], "slo_violations": r["slo_violations"],
                            "per_bucket": r["per_bucket"] if f == load else None})
            ok = [p for p in pts if p["p99_ms"] <= slo_ms]
            sweep[name] = {"points": pts, "req_s_at_slo": max((p["offered_req_s"] for p in ok), default=None)}
        res["per_G"][str(G)] = {
            "arlo": {"instances": {str(L): int(N[k]) for k, L in enumerate(Ls)},
                     "saturation_req_s": arlo_sat["served_rate"], "load_sweep": sweep["arlo"]},
            "st512": {"saturation_req_s": st_sat["served_rate"], "load_sweep": sweep["st512"]},
            "speedup_saturation": arlo_sat["served_rate"] / st_sat["served_rate"]}
    return res


def dispatch_ablation(arlo, torch, runtimes: dict, cfg, G: int = 8, n_requests: int = 6000, slo_ms: float = 150.0,
                      max_batch: int = 32, stream=None, loads=(0.7, 0.9), bursty: bool = True):
    """Table 4 of the paper: the Request Scheduler (RS, Algorithm 1) against the
    ILB and IG dispatchers on the same ILP deployment of G GPUs, Twitter-Bursty-like (MMPP)
    arrivals at `loads` x the RS saturation rate.  Mean / p98 / p99 latency per policy."""
    Ls = sorted(runtimes)
    dev = torch.device("cuda")
    lat = profile_runtimes(torch, runtimes, cfg, max_batch, stream)
    lengths = wl.sample_lengths(n_requests, seed=wl.SEED_ARRIVALS + 11)
    ids_all = wl.sample_token_ids(cfg, lengths, max(Ls), seed=wl.SEED_ARRIVALS + 12)
    ideal = wl.ideal_runtime(lengths, Ls)
    shares = [float((ideal == k).mean()) for k in range(len(Ls))]
    caps = [slo_capacity(row, slo_ms) for row in lat]
    bufs = {L: (torch.empty((max_batch, L), dtype=torch.int32, device=dev),
                torch.empty((max_batch,), dtype=torch.int32, device=dev)) for L in Ls}
    out = torch.empty((max_batch, cfg.num_labels), device=dev)

    def service(L, batch):
        n = len(batch)
        ids_d, len_d = bufs[L]
        ids_d[:n].copy_(torch.from_numpy(np.ascontiguousarray(ids_all[batch, :L])))
        len_d[:n].copy_(torch.from_numpy(lengths[batch].astype(np.int32)))
        a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        runtimes[L].enqueue(n, ids_d, len_d, out)
        e.record(stream)
        e.synchronize()
        return a.elapsed_time(e) / 1e3

    codes = {"rs": arlo.DISPATCH_RS, "ilb": arlo.DISPATCH_ILB, "ig": arlo.DISPATCH_IG}

    def run(n_inst, arrivals, policy):
        def factory(max_len, n, capacity, lam, alpha, peek):
            s = arlo.Scheduler(max_len, n, capacity, lam, alpha, peek)
            s.set_policy(codes[policy])
            return s
        done, rof, _inst, _busy = simulate_cluster(arrivals, lengths, Ls, n_inst, caps, service, max_batch, factory)
        return summarize(arrivals, lengths, done, rof, Ls, slo_ms)

    zero = np.zeros(n_requests)
    N, _Q, _M = plan_cluster(arlo, G, Ls, lat, shares, 1e5, slo_ms)
    sat = run(N, zero, "rs")["served_rate"]
    N, _Q, _M = plan_cluster(arlo, G, Ls, lat, shares, 0.7 * sat, slo_ms)
    sat = run(N, zero, "rs")["served_rate"]
    arrivals_fn = wl.mmpp_arrivals if bursty else wl.poisson_arrivals
    res = {"G": G, "max_batch": max_batch, "capacity_per_slo_window": {str(L): caps[k] for k, L in enumerate(Ls)},
           "instances": {str(L): int(N[k]) for k, L in enumerate(Ls)}, "rs_saturation_req_s": sat,
           "arrivals": "MMPP (Twitter-Bursty-like)" if bursty else "Poisson", "points": []}
    for f in loads:
        arr = arrivals_fn(n_requests, f * sat, seed=wl.SEED_ARRIVALS)
        row = {"load": f, "offered_req_s": f * sat}
        for pol in ("rs", "ilb", "ig"):
            r = run(N, arr, pol)
            row[pol] = {k: r[k] for k in ("mean_ms", "p98_ms", "p99_ms", "slo_violations", "demoted")}
        res["points"].append(row)
    return res


def periodic_plans(arlo, N0, window_shares, plan_fn):
    """Deployments of the periodic policy: window 0 runs N0; at the start of
    window w >= 1 the allocation plan_fn(shares observed in window w-1) is deployed on the GPUs
    with the minimum-replacement plan (arlo_replace_plan).  Returns [(N per runtime, replaced)]
    per window.  Host logic only (tests run it on the CPU)."""
    I = len(N0)
    G = int(sum(N0))
    gpus = [k for k, n in enumerate(N0) for _ in range(n)]  # runtime index per GPU
    out = [(list(N0), 0)]
    for w in range(1, len(window_shares)):
        N_new = list(plan_fn(window_shares[w - 1]))
        assert sum(N_new) <= G
        gpus, n_rep = arlo.replace_plan(gpus, N_new)
        out.append(([gpus.count(k) for k in range(I)], n_rep))
    return out


def realloc_replay(arlo, torch, runtimes: dict, cfg, G: int = 8, window_requests: int = 3000,
                   scales=(1.0, 1.0, 1.6, 1.6, 2.2, 2.2, 1.3, 1.3), slo_ms: float = 150.0, max_batch: int = 32,
                   stream=None, load: float = 0.9):
    """Periodic re-allocation + instance replacement.
    The length distribution drifts window by window (workload.drifting_lengths, `scales`); each
    window is one Runtime Scheduler period.  "static": the allocation planned on window 0 is kept.
    "periodic": at the start of window w the allocation is re-solved (arlo_allocate) on the bucket
    shares OBSERVED in window w-1 and deployed with the minimum-replacement plan
    (arlo_replace_plan); on B200 a replacement only switches which pre-captured graphs a GPU
    replays (every GPU holds all runtimes' graphs, the paper's "hot instances pre-loaded in GPU
    RAM").  Each length level lasts two windows, so the lagged re-plan catches up in the second.
    Poisson arrivals at `load` x the saturation rate of the window-0 plan on the HEAVIEST window
    (so the static plan runs near saturation there); windows are
    simulated one after another (instances drain at the boundary).  Service times are real
    forwards on this GPU.  Returns per-window latency / SLO violations for both policies and the
    replacements made."""
    Ls = sorted(runtimes)
    dev = torch.device("cuda")
    lat = profile_runtimes(torch, runtimes, cfg, max_batch, stream)
    caps = [slo_capacity(row, slo_ms) for row in lat]
    bufs = {L: (torch.empty((max_batch, L), dtype=torch.int32, device=dev),
                torch.empty((max_batch,), dtype=torch.int32, device=dev)) for L in Ls}
    out = torch.empty((max_batch, cfg.num_labels), device=dev)
    windows = []
    for w, sc in enumerate(scales):
        lens = wl.drifting_lengths(window_requests, sc, seed=wl.SEED_ARRIVALS + 100 + w)
        ids = wl.sample_token_ids(cfg, lens, max(Ls), seed=wl.SEED_ARRIVALS + 200 + w)
        windows.append((lens, ids))

    def shares_of(lens):
        ideal = wl.ideal_runtime(lens, Ls)
        return [float((ideal == k).mean()) for k in range(len(Ls))]

    def factory(max_len, n_inst, capacity, lam, alpha, peek):
        return arlo.Scheduler(max_len, n_inst, capacity, lam, alpha, peek)

    def run_window(w, n_inst, arrivals):
        lens, ids = windows[w]

        def service(L, batch):
            n = len(batch)
            ids_d, len_d = bufs[L]
            ids_d[:n].copy_(torch.from_numpy(np.ascontiguousarray(ids[batch, :L])))
            len_d[:n].copy_(torch.from_numpy(lens[batch].astype(np.int32)))
            a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            runtimes[L].enqueue(n, ids_d, len_d, out)
            e.record(stream)
            e.synchronize()
            return a.elapsed_time(e) / 1e3

        done, rof, _inst, _busy = simulate_cluster(arrivals, lens, Ls, n_inst, caps, service, max_batch, factory)
        return summarize(arrivals, lens, done, rof, Ls, slo_ms)

    # offered rate: `load` x the saturation rate of the window-0 plan on window 0
    sh0 = shares_of(windows[0][0])

    def feasible_plan(shares, r):  # Eq. 3 lower bounds can exceed G at a too-high offered rate
        while True:
            try:
                return plan_cluster(arlo, G, Ls, lat, shares, r, slo_ms)[0], r
            except arlo.ArloError:
                r *= 0.8

    heavy = int(np.argmax(scales))
    N0, r0 = feasible_plan(sh0, 1e5)
    sat = run_window(heavy, N0, np.zeros(window_requests))["served_rate"]
    N0, rate = feasible_plan(sh0, load * sat)
    sat = run_window(heavy, N0, np.zeros(window_requests))["served_rate"]
    rate = load * sat
    res = {"runtimes": Ls, "G": G, "window_requests": window_requests, "scales": list(scales), "slo_ms": slo_ms,
           "offered_req_s": rate, "windows": []}
    plans = periodic_plans(arlo, N0, [shares_of(lens) for lens, _ids in windows],
                           lambda sh: feasible_plan(sh, rate)[0])
    for w in range(len(scales)):
        arrivals = wl.poisson_arrivals(window_requests, rate, seed=wl.SEED_ARRIVALS + 300 + w)
        N_cur, n_rep = plans[w]
        st = run_window(w, list(N0), arrivals)
        pe = run_window(w, N_cur, arrivals)
        res["windows"].append({
            "scale": scales[w], "mean_len": float(windows[w][0].mean()),
            "static": {"instances": {str(L): int(N0[k]) for k, L in enumerate(Ls)}, "mean_ms": st["mean_ms"],
                       "p99_ms": st["p99_ms"], "slo_violations": st["slo_violations"]},
            "periodic": {"instances": {str(L): int(N_cur[k]) for k, L in enumerate(Ls)}, "replaced": n_rep,
                         "mean_ms": pe["mean_ms"], "p99_ms": pe["p99_ms"], "slo_violations": pe["slo_violations"]}})
    for pol in ("static", "periodic"):
        res[pol + "_overall_slo_violations"] = float(np.mean([w_[pol]["slo_violations"] for w_ in res["windows"]]))
        res[pol + "_worst_p99_ms"] = float(max(w_[pol]["p99_ms"] for w_ in res["windows"]))
        res[pol + "_mean_ms"] = float(np.mean([w_[pol]["mean_ms"] for w_ in res["windows"]]))
    res["replacements_total"] = int(sum(w_["periodic"]["replaced"] for w_ in res["windows"]))
    return res
