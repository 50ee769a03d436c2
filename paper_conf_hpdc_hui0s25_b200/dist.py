"""N-GPU path of the search: one process per GPU, torch.distributed NCCL.

Every rank stages the same tables and holds the whole request batch.  For each stage
count k the flattened (request, cut mask) task list is cut into equal pieces dealt
round-robin to the ranks one warp-sized chunk of 32 pieces at a time (``task_shard``, the same integer formula the search kernel uses), so
shards are equal in candidates even with skewed chain lengths and sample the whole batch
(equal in pruning too).  Each rank writes the
minimum key of its range per request; one ``all_reduce(keys, MIN)`` over NCCL combines
them (valid keys < INT64_MAX, the "none" sentinel, so MIN is exact and order-free).
Each rank then decodes its own contiguous slice of the requests (``request_slice``).

Pruning: the search skips candidates that cannot beat the request's running best key,
seeded by the earlier (cheaper) segments.  A rank's shard of segment k covers other
requests than its shards of the earlier ones, so without exchange it would prune against
(almost) nothing: measured on C5 at 8 ranks, 30 ms per rank instead of 13.4
(tools/shard_emulation.py).  ``plan_step`` therefore all-reduces the keys after every
segment (``ffs_plan_keys_range``, K collectives of 8 B x R): every rank prunes exactly
as one GPU does.
"""
from __future__ import annotations

import numpy as np


def task_shard(T: int, rank: int, world: int, chunks_per_rank: int, grain: int = 32) -> list[tuple[int, int]]:
    """[lo, hi) pieces of a segment of T tasks owned by `rank`: the list is cut into
    NC = world * chunks_per_rank chunks of `grain` (the warp) equal contiguous pieces
    (floor(T*u/(NC*grain)) boundaries) and rank g owns chunks j*world + g (the rule of
    k_plan_search, where chunks_per_rank = warps per launch x kDyn and the rank's warps
    grab its chunks dynamically)."""
    NT = world * chunks_per_rank * grain
    us = [(j * world + rank) * grain + i for j in range(chunks_per_rank) for i in range(grain)]
    return [(T * u // NT, T * (u + 1) // NT) for u in us]


def request_slice(R: int, rank: int, world: int) -> tuple[int, int]:
    """[lo, hi) of the requests whose plans `rank` decodes."""
    return R * rank // world, R * (rank + 1) // world


def allreduce_min_(keys, group=None):
    """In-place element-wise MIN of int64 keys over the process group (NCCL on GPUs,
    gloo in the CPU tests)."""
    import torch.distributed as dist
    if dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(keys, op=dist.ReduceOp.MIN, group=group)
    return keys


def search_sharded(planner, req, slo, k_max: int, rank: int, world: int, keys, group=None, stream=None):
    """Keys of the whole batch on every rank: for k = 1..K, shard segment k ->
    all_reduce(MIN).  Each segment then prunes against the best key of every earlier
    segment over all shards, as on one GPU (without the exchange the KS = 3 shard at 8
    ranks costs 0.8x the whole single-GPU segment, measured).  One GPU: one ffs_plan_keys."""
    if world == 1:
        planner.plan_keys(req, slo, k_max, rank, world, keys=keys, stream=stream)
        return keys
    for k in range(1, k_max + 1):
        planner.plan_keys_range(req, slo, k_max, k, k, rank, world, keys=keys, stream=stream)
        allreduce_min_(keys, group)
    return keys


def plan_step(planner, req, slo, k_max: int, rank: int, world: int, keys, plans=None, group=None, stream=None):
    """One step of the sharded hot path: keys of this rank's shards (with the exchange of
    ``search_sharded``) -> decode this rank's slice.  Returns (keys, plans of the slice,
    (lo, hi))."""
    search_sharded(planner, req, slo, k_max, rank, world, keys, group, stream)
    lo, hi = request_slice(int(slo.numel()), rank, world)
    plans = planner.plan_decode(req[lo:hi], slo[lo:hi], keys[lo:hi], k_max, out=plans, stream=stream)
    return keys, plans, (lo, hi)


def plan_step_host(planner, h_req, h_slo, d_req, d_slo, k_max: int, rank: int, world: int, keys, plans, h_out,
                   group=None):
    """End-to-end step through the public API with host buffers: H2D of the batch,
    the sharded step, D2H of this rank's plans, synchronise."""
    import torch
    d_req.copy_(h_req, non_blocking=True)
    d_slo.copy_(h_slo, non_blocking=True)
    plan_step(planner, d_req, d_slo, k_max, rank, world, keys, plans, group)
    h_out.copy_(plans.view(-1), non_blocking=True)
    torch.cuda.current_stream().synchronize()
    return h_out


def segment_tasks(chain_len: np.ndarray, k_max: int) -> list[int]:
    """Number of (request, cut mask) tasks of each stage count k = 1..k_max."""
    from math import comb
    out = []
    for k in range(1, k_max + 1):
        tab = np.array([comb(m - 1, k - 1) if m >= k else 0 for m in range(33)], dtype=np.int64)
        out.append(int(tab[chain_len].sum()))
    return out
