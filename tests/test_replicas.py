"""Multi-process (gloo, world size 2, CPU) coverage of the replica layout:
per-rank request streams, instance placement and whole-job throughput
aggregation (max over ranks of the timed region, units summed)."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

from paper_conf_icpp_tanlyl024_b200 import replicas
from paper_conf_icpp_tanlyl024_b200 import workload as wl


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out):
    import torch
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world),
                      LOCAL_RANK=str(rank))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    r, lr, w = replicas.rank_info()
    lengths = wl.sample_lengths(64, seed=replicas.step_seed(wl.SEED_LENGTHS, 3, r))
    local_ms = 10.0 * (r + 1)  # rank 1 is the slowest
    thr, tmax, ws = replicas.aggregate_throughput(100.0, local_ms)
    gathered = [None] * world
    dist.all_gather_object(gathered, lengths.tolist())
    if rank == 0:
        out.put((thr, tmax, ws, gathered))
    dist.barrier()
    dist.destroy_process_group()


def test_two_rank_aggregation_and_distinct_streams():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    thr, tmax, ws, gathered = q.get(timeout=120)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert ws == 2
    assert tmax == 20.0                      # max over ranks
    assert abs(thr - 200.0 / 0.020) < 1e-6   # units summed over ranks / max time
    assert gathered[0] != gathered[1]        # each rank serves its own requests


def test_assign_runtimes_one_instance_per_gpu():
    assert replicas.assign_runtimes((0, 1, 2, 0, 1), 4) == [1, 2, 2, 4]
    with pytest.raises(ValueError):
        replicas.assign_runtimes((1, 1), 3)


def test_single_process_fallback():
    thr, tmax, ws = replicas.aggregate_throughput(50.0, 5.0)
    assert ws == 1 and abs(thr - 10000.0) < 1e-9


def test_step_seeds_distinct():
    seeds = {replicas.step_seed(1, s, r) for s in range(50) for r in range(8)}
    assert len(seeds) == 400
    a = wl.sample_lengths(16, seed=replicas.step_seed(1, 0, 0))
    b = wl.sample_lengths(16, seed=replicas.step_seed(1, 0, 1))
    assert not np.array_equal(a, b)
