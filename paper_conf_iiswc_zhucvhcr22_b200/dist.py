"""Multi-GPU plumbing for independent per-GPU arenas: the path shards
with no data-path exchange; the only collective is one all-reduce of the counters plus a
max-reduce of the iteration time at the end of a run (north_star)."""
from __future__ import annotations


def world():
    import torch.distributed as dist
    if dist.is_available() and dist.is_initialized():
        return dist.get_rank(), dist.get_world_size()
    return 0, 1


def reduce_run(stats: dict, iter_ms: float, device=None):
    """Sum the integer counters `stats` over ranks (int64, exact) and take the max of
    `iter_ms` (timing is max over ranks).  Returns (stats_sum, iter_ms_max).  Works with
    nccl (device = cuda) or gloo (cpu)."""
    import torch
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()):
        return dict(stats), iter_ms
    keys = sorted(stats)
    dev = device if device is not None else torch.device("cpu")
    v = torch.tensor([int(stats[k]) for k in keys], dtype=torch.int64, device=dev)
    t = torch.tensor([float(iter_ms)], dtype=torch.float64, device=dev)
    dist.all_reduce(v, op=dist.ReduceOp.SUM)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return {k: int(x) for k, x in zip(keys, v.cpu().tolist())}, float(t.item())


def bind_to_gpu_numa_node(cpus):
    """Restrict this process (and the host memory it pins afterwards, by first touch) to
    the host cores of its GPU's NUMA node: per-rank host chunks are then NUMA-local
    (SURVEY §8(d) row C5).  `cpus` = the node's cores; no-op if empty."""
    import os
    if cpus:
        os.sched_setaffinity(0, set(cpus))


def barrier():
    import torch.distributed as dist
    if dist.is_available() and dist.is_initialized():
        dist.barrier()
