"""A rank's step captured into a CUDA graph (dist.capture_graph, used by bench.py's
production leg and tools/shard_emulation.py) replays to the same keys and plans as the
eager calls, in both search modes, on a request shard of C3."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("mode", ["bounded", "exhaustive"])
def test_graph_replay_matches_eager(mode):
    import torch
    from paper_conf_hpdc_hui0s25_b200 import dist, ffs, workload as W
    prob = W.config3()
    pl = ffs.Planner(0)
    pl.stage(prob)
    pl.set_search_mode(ffs.SEARCH_BOUNDED if mode == "bounded" else ffs.SEARCH_EXHAUSTIVE)
    req, slo = ffs.to_device(prob)
    R, K = prob.R, prob.k_max
    lo, hi = dist.request_slice(R, 1, 4)  # one rank's slice: graph over sliced views
    keys = torch.empty(R, dtype=torch.int64, device="cuda")
    plans = torch.empty((R, 80), dtype=torch.uint8, device="cuda")

    def step():
        pl.plan_keys(req[lo:hi], slo[lo:hi], K, keys=keys[lo:hi])
        pl.plan_decode(req[lo:hi], slo[lo:hi], keys[lo:hi], K, out=plans[lo:hi])

    step()
    torch.cuda.synchronize()
    k_ref, p_ref = keys[lo:hi].clone(), plans[lo:hi].clone()
    g = dist.capture_graph(step)
    for _ in range(2):
        keys.fill_(0)
        plans.fill_(0)
        g.replay()
        torch.cuda.synchronize()
        assert torch.equal(keys[lo:hi], k_ref)
        assert torch.equal(plans[lo:hi], p_ref)
    assert int((keys[:lo] != 0).sum()) == 0  # nothing outside the slice was written
    assert np.any(k_ref.cpu().numpy() != np.iinfo(np.int64).max)
    pl.close()
