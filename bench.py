#!/usr/bin/env python
"""Benchmark of the polymorphed BERT-base runtimes on B200 (BASELINE.json configs[1]).

One STEP = serving R synthetic requests (skewed Twitter-like lengths,
paper_conf_icpp_tanlyl024_b200/workload.py) through the per-length runtimes
L in {64, 128, 256, 512} (batch buckets up to 32, bf16): every request goes to
its ideal runtime (smallest max_length >= len, §3.2 / Alg. 1
with idle instances) and each runtime runs ceil(n_L / 32) static-shape
forwards (embedding -> 12 x {QKV, masked attention, out-proj, LN, FFN1, FFN2,
LN} -> pooler/classifier).  value = requests / second over the timed steps.

Usage:  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl arlo|reference] [--full]
The last stdout line is one compact JSON object (the headline: value, per-bucket latency,
roofline, cpu_baseline, e2e, clocks); the per-L tables, the ST-512 baseline, the BERT-large
table, the GEMM roofline table and the oracle-timing details go to --extras-out.
Under torchrun each rank serves its own R requests per step on its own GPU
(independent replicas, no data-path collective; weak scaling); timing is
the max over ranks.  `--impl reference` times the fp64 CPU oracle on the
same workload definition (rank 0 only).
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from paper_conf_icpp_tanlyl024_b200 import metrics  # noqa: E402
from paper_conf_icpp_tanlyl024_b200 import replicas  # noqa: E402
from paper_conf_icpp_tanlyl024_b200 import workload as wl  # noqa: E402

RUNTIME_LS = (64, 128, 256, 512)
MAX_BATCH = 32
METRIC = "BERT-base req/s & mean/p99 latency per length bucket; tensor-pipe util"
WORKLOAD = "bert-base polymorphed runtimes L{64,128,256,512}, batch buckets <=32 (BASELINE configs[1])"


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=20)
    p.add_argument("--warmup", type=int, default=5)
    p.add_argument("--impl", default="arlo", choices=["arlo", "reference"])
    p.add_argument("--requests", type=int, default=512, help="requests per step per GPU")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-extras", action="store_true", help="skip per-L table / ST-512 / e2e (profiling runs)")
    p.add_argument("--full", action="store_true", help="also run the trace replay and the cluster replay")
    p.add_argument("--extras-out", default=os.path.join(ROOT, "gpurun_out", "bench_extras.json"),
                   help="where the per-L tables, ST-512, BERT-large and oracle-timing details are written")
    p.add_argument("--cpu-trace-requests", type=int, default=64, help="oracle trace-sample size (cpu_baseline)")
    p.add_argument("--ref-requests", type=int, default=4, help="--impl reference: requests per step")
    return p.parse_args()


# ------------------------------------------------------------------------- workload plan
def make_step_requests(step: int, rank: int, R: int, cfg):
    lengths = wl.sample_lengths(R, seed=replicas.step_seed(wl.SEED_LENGTHS, step, rank))
    return lengths


def plan_forwards(lengths, runtime_ls=RUNTIME_LS, max_batch=MAX_BATCH):
    """Group requests by ideal runtime; chunks of <= max_batch. Returns [(L, [request idx])]."""
    idx = wl.ideal_runtime(lengths, runtime_ls)
    out = []
    for r, L in enumerate(runtime_ls):
        members = np.nonzero(idx == r)[0]
        for s in range(0, len(members), max_batch):
            out.append((L, members[s:s + max_batch]))
    return out


# ------------------------------------------------------------------------- clocks
class ClockSampler:
    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index: int):
        self.gpu, self.rows, self.proc = gpu_index, [], None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            parts = [x.strip() for x in line.split(",")]
            if len(parts) == 8:
                self.rows.append(parts)

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        self.t.join(timeout=2)
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4) if r[4 + i].lower().startswith("active")})
        loaded = [s for s in sm if s > 500] or sm
        return {"sm_mhz": float(np.median(loaded)) if loaded else None,
                "sm_max_mhz": max(mx) if mx else None, "reasons": reasons, "samples": len(self.rows)}


# ------------------------------------------------------------------------- oracle timing
def cpu_model() -> str:
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    import platform
    return platform.processor() or "unknown"


def blas_threads() -> int:
    import threadpoolctl
    return max((d.get("num_threads", 1) for d in threadpoolctl.threadpool_info()), default=1)


def run_reference(args, rank):
    """The oracle, as it stands, timed on this host's cores on bounded samples of the workload
    (each step: the first `--ref-requests` requests of that step's skewed draw, real prefixes)."""
    from oracle import encoder as orc
    cfg = wl.BERT_BASE
    w = wl.make_weights(cfg)
    per_step = args.ref_requests
    times, n_req = [], 0
    for step in range(args.warmup + args.steps):
        lengths = make_step_requests(step, rank, args.requests, cfg)[:per_step]
        ids = wl.sample_token_ids(cfg, lengths, int(lengths.max()), seed=wl.SEED_TOKENS + step)
        t0 = time.perf_counter()
        for i, n in enumerate(lengths):
            orc.forward_request(cfg, w, ids[i, :n])
        dt = time.perf_counter() - t0
        if step >= args.warmup:
            times.append(dt)
            n_req += len(lengths)
    total = sum(times)
    value = n_req / total
    sample = (f"{per_step} requests/step of the skewed length distribution (real prefixes, fp64 numpy), "
              f"{os.cpu_count()} host cores ({cpu_model()})")
    return {"metric": METRIC, "value": value, "unit": "req/s", "impl": "reference", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * total / len(times),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "config": {"workload": WORKLOAD, "sample": sample},
            "cpu_baseline": {"value": value, "unit": "req/s", "cores": blas_threads(), "kind": "oracle",
                             "sample": sample},
            "e2e": {"value": value, "unit": "req/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}


def cpu_baseline(trace_requests=64, one_thread_requests=8):
    """Oracle timing plan: the oracle as it stands on this host's cores, on
    bounded samples: (i) the tiny config (configs[0], L=32 b=4); (ii) a per-L subsample (BERT-base
    b=2 per L, BERT-large b=1 per L, every request of length L); (iii) a subsample of the skewed
    trace (the compact line's value, req/s); (iv) the same trace requests with BLAS limited to one
    thread."""
    import threadpoolctl
    from oracle import encoder as orc
    out = {"kind": "oracle", "unit": "req/s", "cores": blas_threads(), "host_cpus": os.cpu_count(),
           "cpu_model": cpu_model()}
    # (i) tiny
    cfg = wl.TINY
    w = wl.make_weights(cfg)
    lens = np.array([32, 17, 1, 2], np.int32)
    ids = wl.sample_token_ids(cfg, lens, 32)
    t0 = time.perf_counter()
    orc.forward_batch(cfg, w, ids, lens)
    out["tiny_L32_b4_ms"] = 1e3 * (time.perf_counter() - t0)
    # (ii) per-L subsample
    per_L = {}
    for cfg, Ls, b in ((wl.BERT_BASE, (64, 128, 256, 512), 2), (wl.BERT_LARGE, (128, 256, 512), 1)):
        w = wl.make_weights(cfg)
        row = {}
        for L in Ls:
            lens = np.full(b, L, np.int32)
            ids = wl.sample_token_ids(cfg, lens, L, seed=5)
            t0 = time.perf_counter()
            orc.forward_batch(cfg, w, ids, lens)
            row[str(L)] = 1e3 * (time.perf_counter() - t0) / b
        per_L[cfg.name] = row
    out["per_L_ms_per_request"] = per_L
    # (iii) trace subsample
    cfg = wl.BERT_BASE
    w = wl.make_weights(cfg)
    lengths = wl.sample_lengths(trace_requests, seed=wl.SEED_LENGTHS + 999)
    ids = wl.sample_token_ids(cfg, lengths, 512, seed=wl.SEED_TOKENS + 999)
    t0 = time.perf_counter()
    for i in range(trace_requests):
        orc.forward_request(cfg, w, ids[i, :lengths[i]])
    dt = time.perf_counter() - t0
    out["value"] = trace_requests / dt
    out["sample"] = (f"{trace_requests} requests of the skewed trace (mean len {lengths.mean():.1f}), real prefixes, "
                     f"numpy fp64 on {os.cpu_count()} host cores, {dt:.1f} s")
    # (iv) one BLAS thread, first requests of the same sample
    with threadpoolctl.threadpool_limits(1):
        t0 = time.perf_counter()
        for i in range(one_thread_requests):
            orc.forward_request(cfg, w, ids[i, :lengths[i]])
        dt1 = time.perf_counter() - t0
    out["one_thread_value"] = one_thread_requests / dt1
    out["one_thread_sample"] = f"first {one_thread_requests} requests of the same sample, 1 BLAS thread"
    return out


def load_peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))), "MEASURED_PEAKS.json"
    except Exception:
        return {"bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0, "hbm_gbs": 6650.0}, \
            "fallback (B200_PROFILING.md)"


# ------------------------------------------------------------------------- main arm
def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))

    if args.impl == "reference":
        if rank == 0:
            print(json.dumps(run_reference(args, rank)), flush=True)
        return

    import torch
    import torch.distributed as dist
    from paper_conf_icpp_tanlyl024_b200 import arlo

    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    cfg = wl.BERT_BASE
    w = wl.make_weights(cfg)
    W = arlo.Weights(cfg, arlo.upload_weights(cfg, w, arlo.BF16, dev), arlo.BF16, local_rank)
    stream = torch.cuda.Stream(dev)  # runtimes, events and the L2 flush all on this stream
    torch.cuda.set_stream(stream)
    runtimes = {}
    for L in RUNTIME_LS:
        rt = arlo.Runtime(W, L, MAX_BATCH)
        rt.set_stream(stream)
        runtimes[L] = rt

    R = args.requests
    n_steps = args.warmup + args.steps
    # pre-stage every step's inputs in HBM (device-resident timing)
    steps = []
    for s in range(n_steps):
        lengths = make_step_requests(s, rank, R, cfg)
        fwd = []
        for L, members in plan_forwards(lengths):
            lens = lengths[members].astype(np.int32)
            ids = wl.sample_token_ids(cfg, lens, L, seed=wl.SEED_TOKENS + 31 * s + L)
            fwd.append((L, len(members), torch.from_numpy(ids).to(dev), torch.from_numpy(lens).to(dev),
                        torch.empty((len(members), cfg.num_labels), device=dev), ids, lens))
        steps.append((lengths, fwd))
    flush = torch.empty(512 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)  # 512 MB > 126 MB L2

    def run_step(fwd, ev_pairs=None):
        for j, (L, n, ids_d, lens_d, out_d, _, _) in enumerate(fwd):
            if ev_pairs is not None:
                ev_pairs[j][0].record(stream)
            runtimes[L].enqueue(n, ids_d, lens_d, out_d)
            if ev_pairs is not None:
                ev_pairs[j][1].record(stream)

    for s in range(args.warmup):
        run_step(steps[s][1])
        flush.zero_()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()

    # ncu launch lists (tools/profile_round.sh): with ARLO_PROFILE_TIMED=1 and
    # `ncu --profile-from-start off` only the timed steps are captured, not runtime creation
    # (its build-time tile timing launches every tile variant) or warm-up
    profile_timed = os.environ.get("ARLO_PROFILE_TIMED") == "1"
    if profile_timed:
        torch.cuda.cudart().cudaProfilerStart()
    sampler = ClockSampler(local_rank)
    sampler.start()
    time.sleep(0.3)
    step_ms, per_fwd = [], []
    launches = 0
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    for s in range(args.warmup, n_steps):
        fwd = steps[s][1]
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in fwd]
        st, en = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        st.record(stream)
        run_step(fwd, ev)
        en.record(stream)
        flush.zero_()  # between timed steps, outside [st, en]
        launches += sum(runtimes[L].kernel_count(n) for (L, n, *_rest) in fwd)
        per_fwd.append((fwd, ev))
        step_ms.append((st, en))
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clocks = sampler.stop()
    if profile_timed:
        torch.cuda.cudart().cudaProfilerStop()
    step_times = [a.elapsed_time(b) for a, b in step_ms]
    total_ms = float(sum(step_times))
    # per-bucket latency: a request's latency = its forward's duration (all arrive at step start,
    # forwards run back to back: completion time from step start is also reported)
    lat = {L: [] for L in RUNTIME_LS}
    done = {L: [] for L in RUNTIME_LS}
    for (fwd, ev), (st, _) in zip(per_fwd, step_ms):
        for (L, n, *_r), (a, b) in zip(fwd, ev):
            lat[L] += [a.elapsed_time(b)] * n
            done[L] += [st.elapsed_time(b)] * n
    total_req = R * args.steps
    # whole job: requests summed over ranks / max over ranks of the timed region
    value, t_max, _ = replicas.aggregate_throughput(float(total_req), total_ms)
    e2e_res = None
    if not args.no_extras:
        e2e_res = e2e(runtimes, torch, stream, steps[args.warmup:], R, cfg, flush)

    result = None
    extras = {}
    if rank == 0:
        rnd = lambda x, k=4: None if x is None else float(f"{x:.{k}g}")  # noqa: E731
        result = {"metric": METRIC, "value": rnd(value, 6), "unit": "req/s", "n_gpus": world, "steps": args.steps,
                  "warmup": args.warmup, "ms_per_step": rnd(t_max / args.steps, 5), "higher_is_better": True,
                  "scaling": "weak", "vs_baseline": None, "dtype": "bf16", "data": "synthetic",
                  "config": {"workload": WORKLOAD, "requests_per_step_per_gpu": R,
                             "lengths": "LogNormal(ln21,0.6)<=125 x512/125", "weights": "random N(0,0.02) seed 0",
                             "l2": "flushed (512 MB write) between steps", "parallelism": f"replicas x{world}"},
                  "latency_ms_per_bucket": {
                      str(L): {"n": len(lat[L]),
                               "mean": rnd(np.mean(lat[L])) if lat[L] else None,
                               "p99": rnd(np.percentile(lat[L], 99)) if lat[L] else None,
                               "completion_mean": rnd(np.mean(done[L])) if done[L] else None,
                               "completion_p99": rnd(np.percentile(done[L], 99)) if done[L] else None}
                      for L in RUNTIME_LS},
                  "gpu_launches": int(launches), "clocks": clocks}
        pad_tokens = sum(L * n for (_, fwd) in steps[args.warmup:] for (L, n, *_r) in fwd)
        real_tokens = sum(int(x.sum()) for (x, _) in steps[args.warmup:])
        static_flops = sum(metrics.forward_flops(cfg, n, L) for (_, fwd) in steps[args.warmup:] for (L, n, *_r) in fwd)
        result["padding_efficiency"] = rnd(real_tokens / pad_tokens)
        result["static_tflops"] = rnd(static_flops / (total_ms / 1e3) / 1e12)
        result["useful_tflops"] = rnd(sum(metrics.useful_flops(cfg, x) for (x, _) in steps[args.warmup:])
                                      / (total_ms / 1e3) / 1e12)

    if rank == 0 and not args.no_extras:
        roof, gemm_table = roofline_dominant(arlo, torch, dev, stream, runtimes[128], flush)
        result["roofline"] = roof
        extras["gemm_roofline_L128_b32"] = gemm_table
        extras["gemm_tiles"] = {"note": "QKV, out-proj, FFN1, FFN2 tile codes per batch bucket, timed on the device "
                                        "at runtime creation (BN single CTA, -BN CTA pair, 1000+BN skinny)",
                                **{str(L): {str(n): rt.gemm_tiles(n) for n in (1, 8, 16, 32)}
                                   for L, rt in runtimes.items()}}
        extras["per_L_latency_ms"] = per_L_table(runtimes, torch, dev, stream, cfg)
        extras["per_L_latency_ms_restricted"] = per_L_table(runtimes, torch, dev, stream, cfg, restricted=True)
        pl = extras["per_L_latency_ms"]
        result["per_L_b1_ms"] = {L: rnd(pl[L]["1"]["median"]) for L in pl}
        # the paper's batch-1 runtimes in the LATENCY family (LayerNorm folded into
        # the GEMMs): max_batch = 1 runtimes, one forward of b = 1 at length L
        lat_rts = {}
        for L in RUNTIME_LS:
            lat_rts[L] = arlo.Runtime(W, L, 1, arlo.RUNTIME_LATENCY)
            lat_rts[L].set_stream(stream)
        lt = per_L_table(lat_rts, torch, dev, stream, cfg, b_list=(1,))
        extras["per_L_latency_family_b1_ms"] = lt
        result["per_L_b1_latency_family_ms"] = {L: rnd(lt[L]["1"]["median"]) for L in lt}
        for rt in lat_rts.values():
            rt.close()
        extras["paper_context"] = {
            "note": "context only: RTX 3090, FP32 TensorRT static shape, batch 1 (BASELINE.md section 1)",
            "bert_base_L512_b1_ms": {"paper_rtx3090": 4.86, "this_b200_bf16": pl["512"]["1"]["median"],
                                     "source": "PAPER.md:L101 (Fig. 2a)"},
            "latency_ratio_L512_over_L64_b1": {"paper_rtx3090": 4.22,
                                               "this_b200_bf16": pl["512"]["1"]["median"] / pl["64"]["1"]["median"],
                                               "source": "PAPER.md:L95"}}
        st512 = uniform_512(runtimes, torch, dev, stream, steps[args.warmup:], flush, R, cfg)
        extras["uniform_512"] = st512
        result["uniform_512_req_s"] = rnd(st512["value"], 5)
        result["e2e"] = e2e_res
        bl = bert_large_per_L(arlo, torch, dev, stream, local_rank, flush)
        extras["bert_large"] = bl
        result["bert_large_frac_of_burst"] = {f"L{L}_b{b}": rnd(bl["per_L"][str(L)][str(b)]["frac_of_peak"], 3)
                                              for L in (256, 512) for b in (32, 64)}
        result["bert_large_b1_latency_family_ms"] = {L: rnd(v) for L, v in bl["latency_family_b1_ms"].items()}
        if args.full:
            extras["trace_replay"] = trace_replay(arlo, torch, runtimes, cfg, stream, result, pl)
            extras["cluster_replay"] = cluster_replay(arlo, torch, W, runtimes, cfg, stream)
        if not args.no_cpu_baseline:
            cb = cpu_baseline(args.cpu_trace_requests)
            extras["cpu_baseline"] = cb
            result["cpu_baseline"] = {k: (rnd(v) if isinstance(v, float) else v) for k, v in cb.items()
                                      if k in ("value", "unit", "cores", "kind", "sample", "cpu_model", "host_cpus",
                                               "one_thread_value")}
        result["extras_file"] = os.path.relpath(args.extras_out, ROOT)
        extras["headline"] = result
        os.makedirs(os.path.dirname(os.path.abspath(args.extras_out)), exist_ok=True)
        with open(args.extras_out, "w") as f:
            json.dump(extras, f, indent=1)
    if rank == 0:
        print(json.dumps(result, separators=(",", ":")), flush=True)
    for rt in runtimes.values():
        rt.close()
    if world > 1:
        dist.destroy_process_group()


def trace_replay(arlo, torch, runtimes, cfg, stream, result, per_L_ms):
    """Mean / p98 / p99 latency per length bucket under Poisson and MMPP arrivals at
    70% of the measured saturation throughput, requests dispatched by Algorithm 1
    (replay.py); SLO 150 ms for BERT-base."""
    from paper_conf_icpp_tanlyl024_b200 import replay
    per_L = {int(L): {int(b): v["median"] for b, v in row.items()} for L, row in per_L_ms.items()}
    rate = 0.7 * result["value"] / max(1, result["n_gpus"])
    out = {}
    for bursty in (False, True):
        out["bursty" if bursty else "stable"] = replay.replay(arlo, torch, runtimes, cfg, 20000, rate, bursty=bursty,
                                                              slo_ms=150.0, max_batch=MAX_BATCH, per_L_ms=per_L,
                                                              stream=stream)
    return out


def cluster_replay(arlo, torch, W, runtimes, cfg, stream):
    """BASELINE configs[3]: BERT-base polymorphing with 8 runtimes (L = 64..512 step 64) placed by
    the ILP (arlo_allocate) on G = 1, 2, 4, 8 GPUs, requests routed by Algorithm 1, vs ST-512.
    Instances are independent replicas, so the G-GPU cluster is simulated with G virtual device
    clocks driven by real forwards on this GPU (replay.cluster_replay)."""
    from paper_conf_icpp_tanlyl024_b200 import replay
    rts = dict(runtimes)
    extra = []
    for L in wl.RUNTIME_LENGTHS:
        if L not in rts:
            rt = arlo.Runtime(W, L, MAX_BATCH)
            rt.set_stream(stream)
            rts[L] = rt
            extra.append(rt)
    t0 = time.time()
    res = replay.cluster_replay(arlo, torch, rts, cfg, Gs=(1, 2, 4, 8), n_requests=6000, slo_ms=150.0,
                                max_batch=MAX_BATCH, stream=stream)
    res["wall_s"] = time.time() - t0
    res["note"] = ("one runtime instance per GPU (PAPER.md:L155), G virtual device clocks advanced by real "
                   "forwards on this B200 (replicas never communicate); saturation = all requests at t=0; "
                   "latencies from a Poisson replay at 70% of the saturation rate")
    for rt in extra:
        rt.close()
    return res


def bert_large_per_L(arlo, torch, dev, stream, device_index, flush, reps=20):
    """north_star target: per-L bf16 BERT-large forward at L >= 256 as a fraction of
    the B200 tensor peak (BASELINE configs[2]: L in {128,256,512}, batch up to 64).
    Per (L, b): 3 warm-up forwards, then `reps` timed forwards (CUDA events around each,
    L2 flushed before each, outside the events), median reported, with the SM clocks
    sampled by nvidia-smi during the row."""
    cfg = wl.BERT_LARGE
    W = arlo.Weights(cfg, arlo.upload_weights(cfg, wl.make_weights(cfg, seed=wl.SEED_WEIGHTS), arlo.BF16, dev),
                     arlo.BF16, device_index)
    peaks, src = load_peaks()
    peak, peak_sus = peaks["bf16_tflops"], peaks["bf16_tflops_sustained"]
    out = {}
    for L in (128, 256, 512):
        rt = arlo.Runtime(W, L, 64)
        rt.set_stream(stream)
        row = {}
        for b in (1, 16, 32, 64):
            lens = np.full(b, L, np.int32)
            ids = torch.from_numpy(wl.sample_token_ids(cfg, lens, L, seed=5)).to(dev)
            ld = torch.from_numpy(lens).to(dev)
            o = torch.empty((b, cfg.num_labels), device=dev)
            for _ in range(3):
                rt.enqueue(b, ids, ld, o)
            torch.cuda.synchronize()
            sampler = ClockSampler(device_index)
            sampler.start()
            ev = []
            for _ in range(reps):
                flush.zero_()
                a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(stream)
                rt.enqueue(b, ids, ld, o)
                e.record(stream)
                ev.append((a, e))
            torch.cuda.synchronize()
            clk = sampler.stop()
            ts = sorted(a.elapsed_time(e) for a, e in ev)
            ms = float(np.median(ts))
            tf = metrics.forward_flops(cfg, b, L) / (ms / 1e3) / 1e12
            row[str(b)] = {"ms": ms, "min_ms": ts[0], "max_ms": ts[-1], "static_tflops": tf,
                           "frac_of_peak": tf / peak, "frac_of_sustained_peak": tf / peak_sus,
                           "sm_mhz": clk.get("sm_mhz"), "clock_reasons": clk.get("reasons")}
        out[str(L)] = row
        rt.close()
    # the paper's batch-1 runtimes for BERT-large too, LATENCY family
    lat_rts = {}
    for L in (128, 256, 512):
        lat_rts[L] = arlo.Runtime(W, L, 1, arlo.RUNTIME_LATENCY)
        lat_rts[L].set_stream(stream)
    lat_b1 = per_L_table(lat_rts, torch, dev, stream, cfg, b_list=(1,))
    for rt in lat_rts.values():
        rt.close()
    W.close()
    return {"per_L": out, "latency_family_b1_ms": {L: lat_b1[L]["1"]["median"] for L in lat_b1}, "peak_tflops": peak, "peak_sustained_tflops": peak_sus, "peak_source": src, "reps": reps,
            "note": "static FLOPs = layers*(24bLH^2+4bL^2H)+b(2H^2+2HC); median of per-forward CUDA-event times, "
                    "L2 flushed before each forward"}


def roofline_dominant(arlo, torch, dev, stream, rt128, flush, reps=30):
    """Roofline of the dominant kernel.  The four GEMMs of the L=128, b=32 runtime (the bucket
    that serves the most requests, 43 %; M = 4096) are timed in the tile configuration its
    CUDA graph actually replays (rt.gemm_tiles(32), chosen by timing at runtime creation).
    Each GEMM is timed the way the forward runs it, inside a CUDA graph, after its inputs were
    written: graph G1 = `reps` x [L2 flush, A (and residual) rewritten, GEMM], graph G0 = the
    same without the GEMM, both replayed on the launching stream between CUDA events; the
    launch time is (t(G1) - t(G0)) / reps.  A is L2-resident (just written, as the previous
    kernel leaves it), the layer's weights come from HBM, and the GEMM's prologue is not
    overlapped with its predecessor (no PDL edge from a copy), so this is conservative against
    the forward.  `single_launch_us` is the same launch timed alone with events on the stream
    outside a graph: it adds ~8 us of launch overhead that the kernel's own globaltimer span
    does not show (tools/roofline_ctx.py, profiles/r02_roofline_ctx.txt).  The dominant kernel
    is the GEMM with the largest time; achieved = 2MNK / its launch time."""
    H, F = 768, 3072
    M = 128 * 32
    codes = rt128.gemm_tiles(32)
    shapes = {"qkv": (M, 3 * H, H, arlo.EPI_BIAS, codes[0]), "out_proj": (M, H, H, arlo.EPI_BIAS_RESIDUAL, codes[1]),
              "ffn1": (M, F, H, arlo.EPI_BIAS_GELU, codes[2]), "ffn2": (M, H, F, arlo.EPI_BIAS_RESIDUAL, codes[3])}
    peaks, src = load_peaks()
    peak = peaks["bf16_tflops"]
    table = {}
    g = torch.Generator(device=dev).manual_seed(0)
    for name, (m, n, k, epi, code) in shapes.items():
        A = torch.randn(m, k, device=dev, generator=g).to(torch.bfloat16)
        Wt = (0.02 * torch.randn(n, k, device=dev, generator=g)).to(torch.bfloat16)
        bias = torch.zeros(n, device=dev)
        res = torch.randn(m, n, device=dev, generator=g).to(torch.bfloat16) if epi == arlo.EPI_BIAS_RESIDUAL else None
        out = torch.empty(m, n, device=dev, dtype=torch.bfloat16)
        A0, R0 = A.clone(), (res.clone() if res is not None else None)

        def gemm():
            arlo.op_gemm(arlo.BF16, A, Wt, bias, out, epi=epi, residual=res, force_bn=code, stream=stream)

        def prep():
            flush.zero_()
            A.copy_(A0)  # the predecessor's output: L2-resident, the weights are not
            if res is not None:
                res.copy_(R0)

        for _ in range(3):
            gemm()
        ev = []
        for _ in range(reps):
            prep()
            a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            gemm()
            e.record(stream)
            ev.append((a, e))
        torch.cuda.synchronize()
        t_single = 1e3 * float(np.mean([a.elapsed_time(e) for a, e in ev]))
        g1 = graph_us(torch, stream, lambda: (prep(), gemm()), reps)
        g0 = graph_us(torch, stream, prep, reps)
        t_us = (g1 - g0) / reps
        fl = metrics.gemm_flops(m, n, k)
        table[name] = {"M": m, "N": n, "K": k, "tile_code": code, "launch_us": t_us, "single_launch_us": t_single,
                       "tflops": fl / (t_us / 1e6) / 1e12, "frac": fl / (t_us / 1e6) / 1e12 / peak}
    dom = max(table, key=lambda k: table[k]["launch_us"])
    d = table[dom]
    traffic = None
    try:
        tj = json.load(open(os.path.join(ROOT, "profiles", "traffic.json")))
        key = f"{dom}_L128_b32_tile{d['tile_code']}_dram_bytes"
        traffic = tj.get(key)
    except Exception:
        pass
    code = d["tile_code"]
    kname = (f"gemm_skinny_kernel<{code - 1000}>" if code > 1000 else
             f"gemm_tc_pair_kernel<{-code}>" if code < 0 else f"gemm_tc_kernel<{code}>")
    roof = {"kernel": f"{kname} ({dom}, M={d['M']} N={d['N']} K={d['K']}, L=128 b=32 graph tile)", "bound": "tensor",
            "achieved": round(d["tflops"], 1), "peak": peak, "unit": "TFLOP/s", "frac": round(d["frac"], 4),
            "traffic": traffic, "peak_source": src + " bf16_tflops (burst)", "launch_us": round(d["launch_us"], 2),
            "single_launch_us": round(d["single_launch_us"], 2), "algorithmic_flops_per_launch": metrics.gemm_flops(d["M"], d["N"], d["K"]),
            "l2": "flushed before each launch, then A / residual rewritten (L2-resident as in the forward), W cold",
            "timing": "in a CUDA graph: (graph[flush, rewrite, GEMM] - graph[flush, rewrite]) / reps, CUDA events"}
    return roof, table


def graph_us(torch, stream, body, n):
    """Device time (us) of one replay of a CUDA graph of n x body(), median of 5, CUDA events on `stream`."""
    with torch.cuda.stream(stream):
        for _ in range(2):
            body()
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=stream):
            for _ in range(n):
                body()
        g.replay()
        ts = []
        for _ in range(5):
            a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            g.replay()
            e.record(stream)
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(e) * 1e3)
    del g
    return float(np.median(ts))


def per_L_table(runtimes, torch, dev, stream, cfg, restricted=False, b_list=None):
    """Offline-profiler table (A4): latency of one forward vs batch bucket for every runtime.
    restricted=False: every request has length L (roofline mode);
    restricted=True: lengths drawn from the skewed distribution restricted to (L-64, L] (8(d)(ii)),
    where attention skips the key chunks past each request's length."""
    table = {}
    for L, rt in runtimes.items():
        row = {}
        for b in b_list or ((1, 8, 32) if restricted else (1, 2, 4, 8, 16, 32)):
            lens = (wl.sample_lengths(b, seed=7 + b, lo=L - 64, hi=L) if restricted else np.full(b, L)).astype(np.int32)
            ids = torch.from_numpy(wl.sample_token_ids(cfg, lens, L, seed=5)).to(dev)
            ld = torch.from_numpy(lens).to(dev)
            out = torch.empty((b, cfg.num_labels), device=dev)
            for _ in range(3):
                rt.enqueue(b, ids, ld, out)
            ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(20)]
            for a, e in ev:
                a.record(stream)
                rt.enqueue(b, ids, ld, out)
                e.record(stream)
            torch.cuda.synchronize()
            ts = [a.elapsed_time(e) for a, e in ev]
            row[str(b)] = {"median": float(np.median(ts)), "p99": float(np.percentile(ts, 99)),
                           "tflops": metrics.forward_flops(cfg, b, L) / (np.median(ts) / 1e3) / 1e12}
            if restricted:
                row[str(b)]["mean_len"] = float(lens.mean())
        table[str(L)] = row
    return table


def uniform_512(runtimes, torch, dev, stream, steps, flush, R, cfg):
    """Baseline ST: the same requests, all zero-padded to L=512."""
    rt = runtimes[512]
    tot = 0.0
    nsteps = min(3, len(steps))
    for lengths, _ in steps[:nsteps]:
        evs = []
        for s0 in range(0, len(lengths), MAX_BATCH):
            lens = lengths[s0:s0 + MAX_BATCH].astype(np.int32)
            ids = torch.from_numpy(wl.sample_token_ids(cfg, lens, 512, seed=3)).to(dev)
            ld = torch.from_numpy(lens).to(dev)
            out = torch.empty((len(lens), cfg.num_labels), device=dev)
            evs.append((len(lens), ids, ld, out))
        a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        for n, ids, ld, out in evs:
            rt.enqueue(n, ids, ld, out)
        e.record(stream)
        flush.zero_()
        torch.cuda.synchronize()
        tot += a.elapsed_time(e)
    return {"value": nsteps * R / (tot / 1e3), "unit": "req/s", "steps": nsteps,
            "note": "same requests, uniform zero-padding to L=512 (ST baseline)"}


def e2e(runtimes, torch, stream, steps, R, cfg, flush):
    """Same metric through the public C ABI with HOST buffers: arlo_infer on pinned host ids/lengths/
    logits per forward (H2D of the inputs and D2H of the logits inside the timed region)."""
    h2d = d2h = 0
    host = []
    for lengths, fwd in steps:
        hf = []
        for (L, n, _i, _l, _o, ids_np, lens_np) in fwd:
            ids_h = torch.zeros((MAX_BATCH, L), dtype=torch.int32).pin_memory()
            ids_h[:n] = torch.from_numpy(ids_np)
            len_h = torch.zeros(MAX_BATCH, dtype=torch.int32).pin_memory()
            len_h[:n] = torch.from_numpy(lens_np)
            out_h = torch.zeros((MAX_BATCH, cfg.num_labels), dtype=torch.float32).pin_memory()
            hf.append((L, n, ids_h, len_h, out_h))
        host.append(hf)
    tot = 0.0
    for hf in host:
        a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        for (L, n, ids_h, len_h, out_h) in hf:
            runtimes[L].infer(ids_h, len_h, out_h)
        e.record(stream)
        torch.cuda.synchronize()
        tot += a.elapsed_time(e)
        flush.zero_()
    for hf in host:
        for (L, n, *_r) in hf:
            h2d += 16 + 4 * MAX_BATCH + 4 * n * L
            d2h += 4 * n * cfg.num_labels + 4
    h2d /= len(host)
    d2h /= len(host)
    value, _, _ = replicas.aggregate_throughput(float(len(host) * R), tot)  # all ranks, max time
    return {"value": value, "unit": "req/s", "h2d_bytes_per_step": int(h2d),
            "d2h_bytes_per_step": int(d2h), "api": "arlo_infer (synchronous, pinned host buffers)"}


if __name__ == "__main__":
    main()
