"""C5 at full size (1,048,576 requests) in the launch configuration bench.py times, checked
against the oracle on the stratified sample SURVEY §8(d) prescribes for C5: every 16th
request, the requests straddling a task-chunk boundary of the KS = 4 split at world 1 and
world 8 (candidate shards) and the request-shard boundaries at world 8, and a 10,000-request
slice of the infeasible ones; plus the bounded (production) and exhaustive modes agreeing on
all 1,048,576 keys.  About 3 minutes of oracle time on the GPU box's host cores."""
from math import comb

import numpy as np
import pytest
import torch

import oracle
from paper_conf_hpdc_hui0s25_b200 import dist as D, workload as W
from test_gpu_parity import assert_plans_equal

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def F():
    from paper_conf_hpdc_hui0s25_b200 import ffs
    return ffs


def chunk_straddlers(prob, sms, world, ks=4, warps_per_sm=16, kdyn=64, limit=1000):
    """Requests whose KS-segment task range contains a chunk boundary of the search
    kernel's task split in exhaustive mode (every request enumerated; NC = sms x 16 warps x
    kdyn x world chunks of 32 pieces, at least 1 task per piece for KS = 4), at world 1 or 8
    (candidate shards).  Evenly spaced subset."""
    n = prob.chain_len()[prob.req["func"]].astype(np.int64)
    tab = np.array([comb(m - 1, ks - 1) if m >= ks else 0 for m in range(33)], np.int64)
    pre = np.concatenate([[0], np.cumsum(tab[n])])
    T = int(pre[-1])
    NC = sms * warps_per_sm * kdyn * world
    want = T // 32
    if want < NC:
        NC = max(world, -(-want // world) * world)
    NT = NC * 32
    u = np.arange(1, NC, dtype=np.int64) * 32  # chunk boundaries (in pieces)
    Tq, Tr = T // NT, T % NT
    b = Tq * u + (Tr * u) // NT
    r = np.searchsorted(pre, b, side="right") - 1  # request holding task b
    inside = b > pre[r]                             # boundary strictly inside the request
    r = np.unique(r[inside])
    return r[np.linspace(0, len(r) - 1, min(limit, len(r))).astype(np.int64)] if len(r) else r


def test_c5_stratified(F):
    prob = W.config5()
    pl = F.Planner(0)
    pl.stage(prob)
    req, slo = F.to_device(prob)
    K = prob.k_max
    keys = pl.plan_keys(req, slo, K)
    p = F.plans_to_numpy(pl.plan_decode(req, slo, keys, K))
    pl.set_search_mode(F.SEARCH_EXHAUSTIVE)
    ex = pl.plan_keys(req, slo, K).cpu().numpy()
    pl.set_search_mode(F.SEARCH_BOUNDED)
    np.testing.assert_array_equal(ex, keys.cpu().numpy())
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    R = prob.R
    shard_b = np.array([x for g in range(1, 8) for lo in [D.request_slice(R, g, 8)[0]] for x in (lo - 1, lo)])
    infeas = np.flatnonzero(p["status"] == 1)
    assert len(infeas) >= 10_000
    parts = {"every_16th": np.arange(0, R, 16),
             "chunk_straddlers_world1": chunk_straddlers(prob, sms, 1),
             "chunk_straddlers_world8": chunk_straddlers(prob, sms, 8),
             "request_shard_boundaries_world8": shard_b,
             "infeasible": infeas[np.linspace(0, len(infeas) - 1, 10_000).astype(np.int64)]}
    assert all(len(v) for v in parts.values()), {k: len(v) for k, v in parts.items()}
    idx = np.unique(np.concatenate(list(parts.values())))
    o = oracle.plan(prob.subset(idx), checks=False)
    assert_plans_equal(p, o, idx)
    print({k: len(v) for k, v in parts.items()}, "checked", len(idx))
    pl.close()
