"""Multi-GPU layout of Arlo's runtime instances: independent replicas, one per GPU.

Arlo places whole runtime instances on GPUs, one per GPU, with no co-location
(§3.3) and the instance count per runtime decided by the
allocation program (Eqs. 2 and 7, L186, L198).  Requests are independent, so
the data path has no collective: each rank serves its own requests on its own
GPU.  The only cross-rank traffic is measurement plumbing (a barrier and a MAX
reduction of the timed region, bench.py), never inside the timed forward.

Host-side helpers only (no CUDA): shard assignment, per-rank seeds and the
aggregation of per-rank timings into a whole-job throughput.
"""
from __future__ import annotations

import os


def rank_info():
    """(rank, local_rank, world_size) from the torchrun environment (defaults: single process)."""
    return (int(os.environ.get("RANK", "0")), int(os.environ.get("LOCAL_RANK", "0")),
            int(os.environ.get("WORLD_SIZE", "1")))


def step_seed(base: int, step: int, rank: int) -> int:
    """Distinct, reproducible request stream per (step, rank) (weak scaling: each rank
    serves its own requests)."""
    return base + 7919 * step + 104729 * rank


def assign_runtimes(N_alloc, world: int):
    """Place runtime instances on GPUs from an allocation N (arlo_allocate's N_i,
    sum(N) == world): returns, per rank, the runtime index it hosts (one instance
    per GPU, no co-location)."""
    if sum(N_alloc) != world:
        raise ValueError(f"allocation {N_alloc} does not use exactly {world} GPUs (Eq. 2)")
    out = []
    for i, n in enumerate(N_alloc):
        out.extend([i] * int(n))
    return out


def aggregate_throughput(units_per_rank: float, local_ms: float, group=None):
    """Whole-job throughput: units summed over ranks / max over ranks of the timed
    region.  Uses torch.distributed (any backend) when initialised."""
    import torch
    import torch.distributed as dist
    if dist.is_available() and dist.is_initialized():
        world = dist.get_world_size(group)
        dev = "cuda" if dist.get_backend(group) == "nccl" else "cpu"
        t = torch.tensor([local_ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
        u = torch.tensor([units_per_rank], dtype=torch.float64, device=dev)
        dist.all_reduce(u, op=dist.ReduceOp.SUM, group=group)
        return float(u.item()) / (float(t.item()) / 1e3), float(t.item()), world
    return units_per_rank / (local_ms / 1e3), local_ms, 1
