"""N-GPU path of the search: one process per GPU, torch.distributed (NCCL
on GPUs, gloo in the CPU tests).  Every rank stages the same tables and holds the whole
request batch.  Two ways to split it, both bit-identical to one GPU:

``shard="requests"`` (default for batches with many requests, the C5 case): requests are
independent against the snapshot (R13), so rank g plans the contiguous request slice
``request_slice(R, g, G)`` -- every segment, its own keys, its own decode -- with no
data-path collective.  The request order of a batch is arrival order (Azure-shaped,
functions drawn i.i.d.), so equal request counts are equal in candidates to within the
sampling noise of R/G requests (C5 at 8 ranks: DESIGN.md §7 measures the spread).
Pruning is per request, so a shard prunes exactly as one GPU does.

``shard="candidates"`` (few requests with huge candidate sets): for each stage count k the
flattened (request, cut mask) task list is cut into equal pieces dealt round-robin to the
ranks one warp-sized chunk of 32 pieces at a time (``task_shard``, the same integer
formula the search kernel uses); each rank writes the minimum key of its pieces per
request and ``all_reduce(keys, MIN)`` over NCCL combines them after every segment, so the
next (heavier) segment prunes against the best key of all shards of the earlier ones
(valid keys < INT64_MAX, the "none" sentinel: MIN is exact and order-free).  Each rank
then decodes its own slice of the requests.
"""
from __future__ import annotations

import numpy as np

MIN_REQUESTS_PER_RANK = 64  # below this a request shard is too lumpy: use candidate shards


def task_shard(T: int, rank: int, world: int, chunks_per_rank: int, grain: int = 32) -> list[tuple[int, int]]:
    """[lo, hi) pieces of a segment of T tasks owned by `rank`: the list is cut into
    NC = world * chunks_per_rank chunks of `grain` (the warp) equal contiguous pieces
    (floor(T*u/(NC*grain)) boundaries) and rank g owns chunks j*world + g (the rule of
    k_plan_search, where chunks_per_rank = warps per launch x kDyn -- fewer for short
    segments, whose pieces are clamped to a minimum length -- and the rank's warps grab its
    chunks dynamically)."""
    NT = world * chunks_per_rank * grain
    us = [(j * world + rank) * grain + i for j in range(chunks_per_rank) for i in range(grain)]
    return [(T * u // NT, T * (u + 1) // NT) for u in us]


def request_slice(R: int, rank: int, world: int) -> tuple[int, int]:
    """[lo, hi) of the requests `rank` owns (request shards) / decodes (candidate shards)."""
    return R * rank // world, R * (rank + 1) // world


def choose_shard(R: int, world: int) -> str:
    return "requests" if world == 1 or R >= MIN_REQUESTS_PER_RANK * world else "candidates"


def allreduce_min_(keys, group=None):
    """In-place element-wise MIN of int64 keys over the process group (NCCL on GPUs,
    gloo in the CPU tests)."""
    import torch.distributed as dist
    if dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(keys, op=dist.ReduceOp.MIN, group=group)
    return keys


def search_sharded(planner, req, slo, k_max: int, rank: int, world: int, keys, group=None, stream=None):
    """Candidate shards: keys of the whole batch on every rank: for k = 1..K, shard
    segment k -> all_reduce(MIN).  Each segment then prunes against the best key of every
    earlier segment over all shards, as on one GPU.  One GPU: one ffs_plan_keys."""
    if world == 1:
        planner.plan_keys(req, slo, k_max, rank, world, keys=keys, stream=stream)
        return keys
    for k in range(1, k_max + 1):
        planner.plan_keys_range(req, slo, k_max, k, k, rank, world, keys=keys, stream=stream)
        allreduce_min_(keys, group)
    return keys


def plan_step(planner, req, slo, k_max: int, rank: int, world: int, keys, plans=None, group=None, stream=None,
              shard: str | None = None):
    """One step of the sharded hot path; returns (keys, plans of this rank's slice,
    (lo, hi)).  Request shards: keys[lo:hi] and the plans of [lo, hi) from this rank
    alone.  Candidate shards: keys of the whole batch (exchange per segment), then decode
    of [lo, hi)."""
    R = int(slo.numel())
    shard = shard or choose_shard(R, world)
    lo, hi = request_slice(R, rank, world)
    if shard == "requests":
        if hi > lo:
            planner.plan_keys(req[lo:hi], slo[lo:hi], k_max, keys=keys[lo:hi], stream=stream)
    elif shard == "candidates":
        search_sharded(planner, req, slo, k_max, rank, world, keys, group, stream)
    else:
        raise ValueError(f"shard={shard!r}")
    if hi > lo:
        plans = planner.plan_decode(req[lo:hi], slo[lo:hi], keys[lo:hi], k_max, out=plans, stream=stream)
    return keys, plans, (lo, hi)


def plan_step_host(planner, h_req, h_slo, d_req, d_slo, k_max: int, rank: int, world: int, keys, plans, h_out,
                   group=None, shard: str | None = None):
    """End-to-end step through the public API with host buffers: H2D of the batch rows the
    rank needs (its slice for request shards, all of it for candidate shards), the sharded
    step, D2H of this rank's plans, synchronise."""
    import torch
    R = int(h_slo.numel())
    shard = shard or choose_shard(R, world)
    lo, hi = request_slice(R, rank, world)
    a, b = (lo, hi) if shard == "requests" else (0, R)
    d_req[a:b].copy_(h_req[a:b], non_blocking=True)
    d_slo[a:b].copy_(h_slo[a:b], non_blocking=True)
    plan_step(planner, d_req, d_slo, k_max, rank, world, keys, plans, group, shard=shard)
    h_out.copy_(plans.view(-1), non_blocking=True)
    torch.cuda.current_stream().synchronize()
    return h_out


def capture_graph(step):
    """A rank's whole step (count + scan, every segment, decode: ~12 library calls)
    captured once into a CUDA graph; ``g.replay()`` then issues it as one launch.  The
    library allocates its scratch on the first call, so `step` is run once on the capture
    stream before capturing.  Only collective-free steps (request shards) are captured."""
    import torch
    side = torch.cuda.Stream()
    side.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(side):
        step()
    torch.cuda.current_stream().wait_stream(side)
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        step()
    return g


def h2d_bytes(R: int, rank: int, world: int, shard: str, row_bytes: int = 12) -> int:
    lo, hi = request_slice(R, rank, world)
    return (hi - lo if shard == "requests" else R) * row_bytes


def segment_tasks(chain_len: np.ndarray, k_max: int) -> list[int]:
    """Number of (request, cut mask) tasks of each stage count k = 1..k_max."""
    from math import comb
    out = []
    for k in range(1, k_max + 1):
        tab = np.array([comb(m - 1, k - 1) if m >= k else 0 for m in range(33)], dtype=np.int64)
        out.append(int(tab[chain_len].sum()))
    return out
