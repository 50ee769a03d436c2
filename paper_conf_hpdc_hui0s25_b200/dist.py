"""N-GPU path of the search: one process per GPU, torch.distributed NCCL.

Every rank stages the same tables and holds the whole request batch.  For each stage
count k the flattened (request, cut mask) task list is split into `world` equal
contiguous ranges (``task_shard``, the same integer formula the search kernel uses), so
shards are equal in candidates even with skewed chain lengths.  Each rank writes the
minimum key of its range per request; one ``all_reduce(keys, MIN)`` over NCCL combines
them (valid keys < INT64_MAX, the "none" sentinel, so MIN is exact and order-free).
Each rank then decodes its own contiguous slice of the requests (``request_slice``).
"""
from __future__ import annotations

import numpy as np


def task_shard(T: int, rank: int, world: int) -> tuple[int, int]:
    """[lo, hi) of a segment of T tasks owned by `rank` (floor(T*g/G) boundaries)."""
    return T * rank // world, T * (rank + 1) // world


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


def plan_step(planner, req, slo, k_max: int, rank: int, world: int, keys, plans=None, group=None, stream=None):
    """One step of the sharded hot path: keys of this rank's shard -> all_reduce(MIN) ->
    decode this rank's slice.  Returns (keys, plans of the slice, (lo, hi))."""
    planner.plan_keys(req, slo, k_max, rank, world, keys=keys, stream=stream)
    allreduce_min_(keys, group)
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
