"""The N-GPU path's host logic at world_size 2 over gloo on CPU:
request shards (no collective) and task-range shards with all_reduce(MIN) of int64 keys
(INT64_MAX sentinel), decode slices.  The CUDA shard kernel is replaced by an independent CPU emulation of the same
task split (tests/helpers.candidate_keys); the GPU kernel's own sharding is checked
bit-exactly in tests/test_gpu_parity.py::test_sharding_invariance."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_hpdc_hui0s25_b200 import dist as D

KEY_NONE = np.iinfo(np.int64).max
CHUNKS, GRAIN = 3, 2  # emulated chunks per rank (warps x kDyn) and pieces per chunk (warp)


def emulated_shard_keys(prob, rank, world, k_first=1, k_last=None):
    """Per-request minimum key over the tasks of `rank` in stage-count segments
    k_first..k_last (default: all)."""
    from helpers import candidate_keys
    cands = [candidate_keys(prob, r) for r in range(prob.R)]
    keys = np.full(prob.R, KEY_NONE, dtype=np.int64)
    for k in range(k_first, (k_last or prob.k_max) + 1):
        tasks = [(r, rk) for r in range(prob.R) for rk in sorted({c[1] for c in cands[r] if c[0] == k})]
        mine = {t for lo, hi in D.task_shard(len(tasks), rank, world, CHUNKS, GRAIN) for t in tasks[lo:hi]}
        for r in range(prob.R):
            for kk, rk, key in cands[r]:
                if kk == k and key is not None and (r, rk) in mine:
                    keys[r] = min(keys[r], key)
    return keys


class FakePlanner:
    """Stands in for ffs.Planner on CPU: plan_keys = emulated shard, decode = keys.  The
    fake request rows carry the request index in their first four bytes, so a call on a
    slice of the batch knows which requests it holds."""

    def __init__(self, prob):
        self.prob = prob
        self.calls = []

    def plan_keys(self, req, slo, k_max, rank=0, world=1, keys=None, stream=None):
        self.calls.append((1, k_max, int(req.shape[0])))
        idx = req[:, :4].contiguous().view(torch.int32).view(-1).numpy()
        sub = self.prob.subset(idx)
        keys.copy_(torch.from_numpy(emulated_shard_keys(sub, rank, world)))
        return keys

    def plan_keys_range(self, req, slo, k_max, k_first, k_last, rank, world, keys=None, stream=None):
        """ffs_plan_keys_range contract: k_first == 1 overwrites, later ranges min-combine."""
        self.calls.append((k_first, k_last))
        part = torch.from_numpy(emulated_shard_keys(self.prob, rank, world, k_first, k_last))
        keys.copy_(part if k_first == 1 else torch.minimum(keys, part))
        return keys

    def plan_decode(self, req, slo, keys, k_max, out=None, stream=None):
        return keys.clone()


def _worker(rank, world, port, q, shard):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import sys
        sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
        from test_oracle_pins import random_tiny
        prob = random_tiny(1007)
        R = prob.R
        keys = torch.full((R,), KEY_NONE, dtype=torch.int64)
        req = torch.zeros((R, 8), dtype=torch.uint8)
        req[:, :4] = torch.arange(R, dtype=torch.int32).view(-1, 1).view(torch.uint8).view(R, 4)
        slo = torch.zeros(R, dtype=torch.int32)
        fp = FakePlanner(prob)
        keys, plans, (lo, hi) = D.plan_step(fp, req, slo, prob.k_max, rank, world, keys, shard=shard)
        if shard == "candidates":  # one sharded range per segment, an exchange after each
            assert fp.calls == [(k, k) for k in range(1, prob.k_max + 1)]
        else:  # one whole search of the rank's own request slice, no collective
            assert fp.calls == [(1, prob.k_max, hi - lo)]
        # sentinel survives MIN, and a MIN of partial minima is the global minimum
        t = torch.tensor([KEY_NONE, 5, KEY_NONE], dtype=torch.int64) if rank == 0 else \
            torch.tensor([KEY_NONE, KEY_NONE, 3], dtype=torch.int64)
        D.allreduce_min_(t)
        q.put((rank, keys.numpy().tolist(), (lo, hi), plans.numpy().tolist(), t.tolist()))
    finally:
        dist.destroy_process_group()


def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.parametrize("world,shard", [(2, "candidates"), (2, "requests")])
def test_sharded_step_matches_oracle_over_gloo(world, shard):
    import oracle
    from test_oracle_pins import random_tiny
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q, shard)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=120) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    prob = random_tiny(1007)
    o = oracle.plan(prob)
    slices = []
    for rank, keys, (lo, hi), plans, t in res:
        if shard == "candidates":
            assert keys == o["key"].tolist()      # all_reduce(MIN) of the shards = global argmin
        else:
            assert keys[lo:hi] == o["key"][lo:hi].tolist()  # the rank's own requests, complete
        assert plans == o["key"][lo:hi].tolist()  # each rank decodes its own slice
        assert t == [KEY_NONE, 5, 3]
        slices.append((lo, hi))
    assert slices[0][0] == 0 and slices[-1][1] == prob.R and all(a[1] == b[0] for a, b in zip(slices, slices[1:]))



def test_shard_partitions_are_exact():
    for T in (0, 1, 7, 1000, 2**41 + 3):
        for world in (1, 2, 3, 8):
            for chunks, grain in ((1, 1), (3, 2), (1184 * 8, 32)):
                pieces = sorted(p for g in range(world) for p in D.task_shard(T, g, world, chunks, grain))
                assert pieces[0][0] == 0 and pieces[-1][1] == T  # exact cover, no overlap
                assert all(x[1] == y[0] for x, y in zip(pieces, pieces[1:]))
                sizes = [sum(h - l for l, h in D.task_shard(T, g, world, chunks, grain)) for g in range(world)]
                assert max(sizes) - min(sizes) <= chunks * grain  # pieces within 1 of each other


def test_emulated_shards_cover_every_candidate():
    """The union over shards of the emulated per-shard minima is the global minimum."""
    import oracle
    from test_oracle_pins import random_tiny
    prob = random_tiny(1011)
    o = oracle.plan(prob)
    for world in (2, 3, 5):
        parts = np.stack([emulated_shard_keys(prob, g, world) for g in range(world)])
        np.testing.assert_array_equal(parts.min(axis=0), o["key"])


def test_request_slices_partition_and_choice():
    for R in (0, 1, 7, 1000, 1 << 20):
        for world in (1, 2, 3, 8):
            sl = [D.request_slice(R, g, world) for g in range(world)]
            assert sl[0][0] == 0 and sl[-1][1] == R and all(a[1] == b[0] for a, b in zip(sl, sl[1:]))
            assert max(h - l for l, h in sl) - min(h - l for l, h in sl) <= 1
    assert D.choose_shard(1 << 20, 8) == "requests" and D.choose_shard(100, 8) == "candidates"
    assert D.choose_shard(5, 1) == "requests"
    assert D.h2d_bytes(1000, 1, 4, "requests") == 250 * 12 and D.h2d_bytes(1000, 1, 4, "candidates") == 12000
