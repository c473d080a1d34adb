"""Serving across the GPUs of one box: Arlo's deployment on physical devices.

The Runtime Scheduler's allocation N_i (arlo_allocate, Eqs. 1-7) is
placed one instance per GPU with no co-location (L155; Eq. 2: sum N_i = G), every GPU
holding its own copy of the weights and its runtime's captured graphs.  One host
dispatcher runs the Request Scheduler (arlo_dispatch, Algorithm 1) over the
live outstanding counts; one worker thread per GPU drains its instance's queue in batches
of up to max_batch (arlo_enqueue on that device's stream), and reports completions back
(arlo_complete).  Instances never exchange data: there is no collective on the data path.

Host logic only: every forward runs in libarlo's kernels on the worker's device.  The
worker/dispatcher machinery takes an `executor` callable so the host side is testable on
CPU (tests/test_cluster_host.py) with a stand-in service time.
"""
from __future__ import annotations

import collections
import threading
import time

import numpy as np


class Instance:
    """One runtime instance = one GPU: a FIFO of (request index, arrival time)."""

    def __init__(self, runtime_index: int, instance_index: int, L: int, gpu: int):
        self.r, self.i, self.L, self.gpu = runtime_index, instance_index, L, gpu
        self.queue = collections.deque()
        self.cv = threading.Condition()
        self.busy_s = 0.0
        self.batches = 0


def place(N_alloc, Ls):
    """Instances of an allocation N (N[k] instances of runtime Ls[k]) on GPUs 0..G-1, in runtime
    order (one instance per GPU).  Returns [Instance] with their scheduler (level, instance) ids
    over the DEPLOYED runtimes (levels with N_k > 0)."""
    out, gpu, level = [], 0, 0
    for k, L in enumerate(Ls):
        if N_alloc[k] <= 0:
            continue
        for j in range(int(N_alloc[k])):
            out.append(Instance(level, j, L, gpu))
            gpu += 1
        level += 1
    return out


class Cluster:
    """Dispatcher + one worker per instance.  executor(inst, idx) serves a batch of request
    indices on inst's GPU and returns its device time in seconds (it runs on the worker
    thread).  sched is an arlo.Scheduler (or any object with dispatch/complete/close) built
    over the deployed runtimes."""

    def __init__(self, instances, sched, executor, max_batch: int):
        self.inst = instances
        self.by_key = {(x.r, x.i): x for x in instances}
        self.sched, self.exec, self.max_batch = sched, executor, max_batch
        self.lock = threading.Lock()  # the scheduler's state is shared by the dispatcher and the workers
        self.stop = False
        self.done_t = None
        self.runtime_of = None

    def _worker(self, x: Instance):
        while True:
            with x.cv:
                while not x.queue and not self.stop:
                    x.cv.wait()
                if not x.queue and self.stop:
                    return
                batch = [x.queue.popleft() for _ in range(min(self.max_batch, len(x.queue)))]
            idx = [i for i, _t in batch]
            dt = self.exec(x, idx)
            x.busy_s += dt
            x.batches += 1
            now = time.perf_counter()
            with self.lock:
                for i in idx:
                    self.done_t[i] = now
                    self.sched.complete(x.r, x.i)

    def run(self, arrivals_s, lengths):
        """Replay: request k arrives at arrivals_s[k] seconds after the start (wall clock; all 0 =
        saturation).  Returns (arrival wall times, completion wall times, level of each request)."""
        n = len(arrivals_s)
        self.done_t = np.zeros(n)
        self.runtime_of = np.zeros(n, np.int32)
        self.stop = False
        threads = [threading.Thread(target=self._worker, args=(x,), daemon=True) for x in self.inst]
        for t in threads:
            t.start()
        t0 = time.perf_counter()
        arr_t = t0 + np.asarray(arrivals_s, np.float64)
        for k in range(n):
            wait = arr_t[k] - time.perf_counter()
            if wait > 0:
                time.sleep(wait)
            with self.lock:
                r, i = self.sched.dispatch(int(lengths[k]))
            self.runtime_of[k] = r
            x = self.by_key[(r, i)]
            with x.cv:
                x.queue.append((k, arr_t[k]))
                x.cv.notify()
        self.stop = True
        for x in self.inst:
            with x.cv:
                x.cv.notify_all()
        for t in threads:
            t.join()
        return arr_t, self.done_t, self.runtime_of


def summarize(arr_t, done_t, levels, deployed_Ls, lengths, slo_ms: float):
    lat = (done_t - arr_t) * 1e3
    span = float(done_t.max() - arr_t.min())
    ideal = np.searchsorted(np.asarray(deployed_Ls), np.asarray(lengths), side="left")
    return {"requests": int(len(arr_t)), "req_s": float(len(arr_t) / span), "makespan_s": span,
            "mean_ms": float(lat.mean()), "p98_ms": float(np.percentile(lat, 98)),
            "p99_ms": float(np.percentile(lat, 99)), "slo_violations": float((lat > slo_ms).mean()),
            "demoted": float((levels != ideal).mean())}
