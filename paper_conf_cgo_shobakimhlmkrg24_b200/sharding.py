"""Multi-GPU sharding of independent regions.

Regions are independent (configs 3 and 5), so they shard across ranks with NO
data-path collective: every rank runs aco_schedule_batch on its own regions.
Region ids are global and key the Philox streams (R26), so a region produces
the same schedule whichever rank runs it.  torch.distributed is used only to
gather per-region results for reporting (gather_object) and, in bench.py,
for the barrier and the max-over-ranks time.
"""
from __future__ import annotations

from typing import Dict, List, Sequence


def estimated_work(n: int, ants: int, iterations: int) -> int:
    """Work estimate of one region: ants x iterations x n x (n + 16) (each ant
    step scans a ready list that grows with n)."""
    return ants * iterations * n * (n + 16)


def lpt_partition(sizes: Sequence[int], world: int, ants: int = 1024, iterations: int = 10) -> List[List[int]]:
    """Deterministic longest-processing-time assignment (strong scaling):
    regions sorted by estimated work (descending, ties by index) go to the
    least-loaded rank (ties to the lowest rank).  Returns per-rank index lists
    in ascending index order."""
    order = sorted(range(len(sizes)), key=lambda i: (-estimated_work(int(sizes[i]), ants, iterations), i))
    load = [0] * world
    parts: List[List[int]] = [[] for _ in range(world)]
    for i in order:
        r = min(range(world), key=lambda k: (load[k], k))
        parts[r].append(i)
        load[r] += estimated_work(int(sizes[i]), ants, iterations)
    return [sorted(p) for p in parts]


def weak_ids(per_rank: int, rank: int) -> List[int]:
    """Weak scaling: rank r owns the global ids [r * per_rank, (r+1) * per_rank)."""
    return list(range(rank * per_rank, (rank + 1) * per_rank))


def gather_results(local: Dict[int, dict], world: int, rank: int, group=None) -> Dict[int, dict]:
    """Gather {region_id: result} from every rank to rank 0 (reporting only)."""
    import torch.distributed as dist
    if world == 1:
        return dict(local)
    buf = [None] * world if rank == 0 else None
    dist.gather_object(local, buf, dst=0, group=group)
    if rank != 0:
        return {}
    out: Dict[int, dict] = {}
    for part in buf:
        for k, v in part.items():
            assert k not in out, f"region {k} scheduled twice"
            out[k] = v
    return out


# ---------------------------------------------------------------- shared colony (config 4)
# The only data-path exchange of the shared colony: per
# region and iteration every rank contributes ONE int64, its local best ant's
# key, and a MIN all-reduce picks the global iteration winner.  The key is
# (cost << 32 | global ant) XOR 2^63 (csrc/aco_internal.h kKeyBias), so a
# signed int64 MIN orders keys like the unsigned (cost, ant) pair: lowest
# cost, ties to the lowest ant id (R10); an invalid ant has cost 0xFFFFFFFF
# (R35).  The kernels build these keys on the device (k_local_keys); the
# helpers below are the host-side statement of the encoding.
KEY_BIAS = 1 << 63
INVALID_COST = 0xFFFFFFFF


def colony_key(cost: int, ant: int) -> int:
    """Biased winner key as a signed int64 value."""
    u = ((int(cost) << 32) | int(ant)) ^ KEY_BIAS
    return u - (1 << 64) if u >= (1 << 63) else u


def colony_decode(key: int):
    """(cost, global ant) of a biased key."""
    u = (int(key) + (1 << 64)) % (1 << 64) ^ KEY_BIAS
    return u >> 32, u & 0xFFFFFFFF


def local_best_key(costs: Sequence[int], ant_base: int) -> int:
    """The key of this rank's best ant: lexicographic (cost, ant) minimum."""
    best = min(range(len(costs)), key=lambda a: (int(costs[a]), a))
    return colony_key(int(costs[best]), ant_base + best)


def colony_allreduce(keys, group=None):
    """MIN all-reduce of a per-region int64 key tensor, in place (the shared
    colony's exchange; NCCL on the GPU path, any backend here)."""
    import torch.distributed as dist
    dist.all_reduce(keys, op=dist.ReduceOp.MIN, group=group)
    return keys
