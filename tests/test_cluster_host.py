"""Host side of the multi-GPU deployment (cluster.py) on CPU: placement, dispatcher and
workers with a stand-in executor (no GPU), scheduler state through the C ABI."""
import threading
import time

import numpy as np

from paper_conf_icpp_tanlyl024_b200 import cluster


def test_place_one_instance_per_gpu():
    insts = cluster.place([0, 2, 0, 1], [64, 128, 192, 256])
    assert [(x.r, x.i, x.L, x.gpu) for x in insts] == [(0, 0, 128, 0), (0, 1, 128, 1), (1, 0, 256, 2)]


def test_cluster_serves_every_request_and_releases_load(arlo_lib):
    Ls = [64, 128, 512]
    N = [1, 2, 1]
    insts = cluster.place(N, Ls)
    sched = arlo_lib.Scheduler(Ls, N, [4.0, 4.0, 8.0], 0.85, 0.9, 6)
    seen = {}
    lock = threading.Lock()

    def executor(x, idx):  # stand-in for a forward: time grows with L and the batch
        with lock:
            for i in idx:
                seen[i] = x.L
        time.sleep(1e-4 * x.L / 64)
        return 1e-4 * x.L / 64

    rng = np.random.default_rng(0)
    lengths = rng.integers(2, 513, 400)
    cl = cluster.Cluster(insts, sched, executor, max_batch=4)
    arr, done, lv = cl.run(np.zeros(400), lengths)
    assert sorted(seen) == list(range(400))
    assert all(seen[i] >= lengths[i] for i in range(400))  # a request runs only on max_length >= len
    assert np.all(done >= arr)
    for x in insts:
        assert sched.outstanding(x.r, x.i) == 0
    s = cluster.summarize(arr, done, lv, Ls, lengths, 150.0)
    assert s["requests"] == 400 and s["req_s"] > 0
    assert 0.0 < s["demoted"] < 1.0  # the burst overloads the short runtimes: Algorithm 1 demotes
    sched.close()
