"""GPU <-> oracle parity through the C ABI (libffs.so).  Needs a B200: marked gpu.

Bar: bit-exact keys, plans and per-request checksums (candidates scored,
feasible count, sum of feasible keys mod 2^64) against the CPU oracle on the same seeded
inputs; zero filter misses; sharding invariance.
"""
import numpy as np
import pytest

import oracle
from helpers import problem, abi_evict_score
from test_oracle_pins import random_tiny
from paper_conf_hpdc_hui0s25_b200 import workload as W

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def F():
    from paper_conf_hpdc_hui0s25_b200 import ffs
    assert torch.cuda.is_available(), "gpu tests need a CUDA device"
    return ffs


@pytest.fixture(scope="module")
def planner(F):
    return F.Planner(0)


def run_gpu(F, planner, prob, k_max=None, verify=True, world=1):
    """keys (+ checksums) over `world` shards combined with a host MIN/SUM (fake
    collective), then decode.  Returns (plans numpy, keys, checks)."""
    k_max = prob.k_max if k_max is None else k_max
    planner.stage(prob)
    req, slo = F.to_device(prob)
    R = prob.R
    keys = torch.full((R,), F.KEY_NONE, dtype=torch.int64, device="cuda")
    checks = torch.zeros((R, 3), dtype=torch.int64, device="cuda") if verify else None
    for rank in range(world):
        k = torch.empty(R, dtype=torch.int64, device="cuda")
        c = torch.empty((R, 3), dtype=torch.int64, device="cuda") if verify else None
        planner.plan_keys(req, slo, k_max, rank, world, keys=k, checks=c)
        keys = torch.minimum(keys, k)
        if verify:
            checks += c  # int64 wrap-around == uint64 sum mod 2^64
    plans = planner.plan_decode(req, slo, keys, k_max)
    torch.cuda.synchronize()
    ch = checks.cpu().numpy().view(np.uint64) if verify else None
    return F.plans_to_numpy(plans), keys.cpu().numpy(), ch


def assert_plans_equal(p, o, idx=None):
    idx = np.arange(len(o["key"])) if idx is None else idx
    g = p[idx]
    np.testing.assert_array_equal(g["key"], o["key"])
    np.testing.assert_array_equal(g["status"], o["status"])
    ok = o["status"] == oracle.PLAN_OK
    for a, b in (("k", "k"), ("cut_mask", "cut_mask"), ("e2e_us", "e2e_us"), ("bottleneck_us", "bottleneck_us"),
                 ("gpcs", "gpcs"), ("cvq", "cvq")):
        np.testing.assert_array_equal(g[a][ok], o[b][ok], err_msg=a)
    np.testing.assert_array_equal(g["prof"], o["prof"])
    np.testing.assert_array_equal(g["slice"], o["slice"])


def test_exports_and_context(F, planner):
    assert planner.device == 0


def test_golden_hand_cases_gpu(F, planner):
    import json, os
    with open(os.path.join(os.path.dirname(__file__), "golden", "hand_cases.json")) as fh:
        cases = json.load(fh)
    for case in cases:
        nodes = [[[s if isinstance(s, int) else tuple(s) for s in gpu] for gpu in node] for node in case["nodes"]]
        prob = problem(case["funcs"], nodes, [tuple(r) for r in case["requests"]], k_max=case["k_max"])
        p, keys, ch = run_gpu(F, planner, prob)
        o = oracle.plan(prob)
        assert_plans_equal(p, o)
        np.testing.assert_array_equal(ch, o["checks"])


@pytest.mark.parametrize("seed", range(1000, 1040))
def test_tiny_random_bit_exact(F, planner, seed):
    prob = random_tiny(seed)
    p, keys, ch = run_gpu(F, planner, prob)
    o = oracle.plan(prob)
    assert_plans_equal(p, o)
    np.testing.assert_array_equal(ch, o["checks"])
    # production (non-verify) path gives the same keys
    p2, keys2, _ = run_gpu(F, planner, prob, verify=False)
    np.testing.assert_array_equal(keys2, o["key"])
    # and so does the exhaustive mode (KS = 3, 4 walk the chain-length groups: mostly idle
    # lanes on a tiny batch)
    try:
        planner.set_search_mode(F.SEARCH_EXHAUSTIVE)
        p3, keys3, _ = run_gpu(F, planner, prob, verify=False)
    finally:
        planner.set_search_mode(F.SEARCH_BOUNDED)
    np.testing.assert_array_equal(keys3, o["key"])


@pytest.mark.parametrize("K", [1, 2, 3, 4, 5, 6, 7, 8])
def test_every_stage_count(F, planner, K):
    # chains of 1..10 components so that every KS template runs, with ragged tails
    rng = W.SplitMix64(777 + K)
    lengths = [1, 2, 3, 5, 8, 10]
    prob = W._problem("ks", rng, lengths, W.NODE_BLOCK, 96, k_max=K)
    p, keys, ch = run_gpu(F, planner, prob, k_max=K)
    o = oracle.plan(prob, k_max=K)
    assert_plans_equal(p, o)
    np.testing.assert_array_equal(ch, o["checks"])
    assert planner.filter_misses() == 0


@pytest.mark.parametrize("cfg", ["C1", "C1b", "C2"])
def test_small_configs_full(F, planner, cfg):
    prob = {"C1": W.config1, "C1b": W.config1b, "C2": W.config2}[cfg]()
    p, keys, ch = run_gpu(F, planner, prob)
    o = oracle.plan(prob)
    assert_plans_equal(p, o)
    np.testing.assert_array_equal(ch, o["checks"])
    p2, keys2, _ = run_gpu(F, planner, prob, verify=False)
    np.testing.assert_array_equal(keys2, o["key"])
    assert planner.filter_misses() == 0


def test_c3_sample_and_checksums(F, planner):
    prob = W.config3()
    p, keys, ch = run_gpu(F, planner, prob)
    idx = np.concatenate([np.arange(0, prob.R, 97), np.arange(prob.R - 50, prob.R)])
    o = oracle.plan(prob.subset(idx))
    assert_plans_equal(p, o, idx)
    np.testing.assert_array_equal(ch[idx], o["checks"])
    # every request scored exactly S(n, K) candidates
    n = prob.chain_len()[prob.req["func"]]
    from math import comb
    S = {m: sum(comb(m - 1, k - 1) * 5 ** k for k in range(1, min(m, 4) + 1)) for m in set(n.tolist())}
    np.testing.assert_array_equal(ch[:, 0], np.array([S[m] for m in n], dtype=np.uint64))
    _, keys2, _ = run_gpu(F, planner, prob, verify=False)
    np.testing.assert_array_equal(keys2, keys)
    assert planner.filter_misses() == 0


@pytest.mark.parametrize("world", [2, 3, 8])
def test_sharding_invariance(F, planner, world):
    prob = W.config2(R=2048)
    p1, k1, c1 = run_gpu(F, planner, prob)
    pw, kw, cw = run_gpu(F, planner, prob, world=world)
    np.testing.assert_array_equal(k1, kw)
    np.testing.assert_array_equal(c1, cw)
    np.testing.assert_array_equal(p1.view(np.uint8), pw.view(np.uint8))


@pytest.mark.parametrize("split", [1, 2, 3])
def test_keys_range_composition(F, planner, split):
    """ffs_plan_keys_range: segments 1..split then split+1..K continuing from the combined
    keys give the keys and checksums of one ffs_plan_keys call, on every shard
    (world 3: each shard's ranges, MIN over shards between and after, as dist.plan_step)."""
    prob = W.config2(R=2048)
    planner.stage(prob)
    req, slo = F.to_device(prob)
    K = prob.k_max
    ref = planner.plan_keys(req, slo, K).cpu().numpy()
    ck_ref = torch.empty(3 * prob.R, dtype=torch.int64, device="cuda")
    planner.plan_keys(req, slo, K, checks=ck_ref)
    keys = torch.empty((3, prob.R), dtype=torch.int64, device="cuda")
    cks = torch.empty((3, 3 * prob.R), dtype=torch.int64, device="cuda")
    for g in range(3):
        planner.plan_keys_range(req, slo, K, 1, split, g, 3, keys=keys[g], checks=cks[g])
    comb = keys.min(dim=0).values
    for g in range(3):
        keys[g].copy_(comb)
        planner.plan_keys_range(req, slo, K, split + 1, K, g, 3, keys=keys[g], checks=cks[g])
    np.testing.assert_array_equal(keys.min(dim=0).values.cpu().numpy(), ref)
    tot = cks.cpu().numpy().view(np.uint64).sum(axis=0, dtype=np.uint64)  # SUM mod 2^64
    np.testing.assert_array_equal(tot, ck_ref.cpu().numpy().view(np.uint64))
    ms = planner.segment_times()
    assert all(ms[k] > 0 for k in range(K)) and all(m == 0 for m in ms[K:])
    with pytest.raises(F.FFSError) as e:
        planner.plan_keys_range(req, slo, K, 3, 2, keys=keys[0])
    assert e.value.status == F.FFS_ERR_RANGE
    with pytest.raises(F.FFSError):
        planner.plan_keys_range(req, slo, K, 1, K + 1, keys=keys[0])


def test_c5_bench_configuration_sampled(F, planner):
    """C5 at full size in the launch configuration bench.py times (world 1, production
    path), checked on a stratified sample against the oracle."""
    prob = W.config5()
    p, keys, _ = run_gpu(F, planner, prob, verify=False)
    rng = W.SplitMix64(55)
    idx = np.unique(np.concatenate([np.arange(0, prob.R, 4099), prob.R - 1 - np.arange(8),
                                    rng.integers(0, prob.R - 1, 64)]))
    o = oracle.plan(prob.subset(idx), checks=False)
    assert_plans_equal(p, o, idx)
    # properties at any size: statuses consistent with keys, slices valid
    ok = p["status"] == 0
    assert (p["key"][~ok] == np.iinfo(np.int64).max).all()
    assert (p["e2e_us"][ok] <= prob.slo_us[ok]).all()
    # the KS = 4 pre-filter's stage-0 SLO bound skips work on C5 (large
    # profiles busy on most nodes): evaluated iterations lie in (0, 5 x KS = 4 masks]
    from math import comb
    n = prob.chain_len()[prob.req["func"]]
    masks = sum(comb(int(m) - 1, 3) for m in n if m >= 4)
    ev = planner.scored()[3]
    assert 0 < ev <= 625 * masks


def test_exhaustive_mode_scores_every_candidate(F, planner):
    """FFS_SEARCH_EXHAUSTIVE (the benchmark's mode, "all possible partitions"): the
    device counters see every candidate of every request scored -- sum over ks equals
    sum_r S(n_r, K), including requests on nodes without a free slice -- and the keys are
    bit-identical to the bounded mode's (C3, full batch) and to the oracle (sample)."""
    from math import comb
    prob = W.config3()
    planner.stage(prob)
    req, slo = F.to_device(prob)
    K = prob.k_max
    bounded = planner.plan_keys(req, slo, K).cpu().numpy()
    try:
        planner.set_search_mode(F.SEARCH_EXHAUSTIVE)
        ex = planner.plan_keys(req, slo, K).cpu().numpy()
        sc = planner.scored()
    finally:
        planner.set_search_mode(F.SEARCH_BOUNDED)
    np.testing.assert_array_equal(ex, bounded)
    n = prob.chain_len()[prob.req["func"]]
    per_ks = [sum(comb(int(m) - 1, k - 1) * 5 ** k for m in n if m >= k) for k in range(1, 9)]
    assert sc[:K] == per_ks[:K] and sum(sc[K:]) == 0
    idx = np.arange(0, prob.R, 997)
    o = oracle.plan(prob.subset(idx), checks=False)
    np.testing.assert_array_equal(ex[idx], o["key"])
    with pytest.raises(F.FFSError):
        planner.set_search_mode(7)


@pytest.mark.parametrize("world", [2, 3, 8])
def test_exhaustive_sharding_invariance(F, planner, world):
    """Exhaustive mode over candidate shards (the KS = 4 segment walks requests grouped by
    chain length, units interleaved over the ranks): every rank's call must derive the same
    grouping, so the element-wise MIN of the shards' keys equals one GPU's keys, and the
    shards' device counters add up to sum_r S(n_r, K)."""
    prob = W.config3()
    planner.stage(prob)
    req, slo = F.to_device(prob)
    K = prob.k_max
    try:
        planner.set_search_mode(F.SEARCH_EXHAUSTIVE)
        ref = planner.plan_keys(req, slo, K).clone()
        total = sum(planner.scored()[:K])
        keys, scored = [], 0
        for r in range(world):
            keys.append(planner.plan_keys(req, slo, K, rank=r, world=world).clone())
            scored += sum(planner.scored()[:K])
    finally:
        planner.set_search_mode(F.SEARCH_BOUNDED)
    import torch
    assert torch.equal(torch.stack(keys).min(0).values, ref)
    assert scored == total


@pytest.mark.parametrize("seed", range(16))
def test_bounded_list_mode_chains(F, planner, seed):
    """Production mode (exact SLO lower bounds: live-mask compaction + list search,
    DESIGN.md §4.3) on random 4-7 component chains, K = 4, budgets from infeasible to
    loose: keys and plans equal the oracle and the exhaustive mode."""
    from test_bound_tables import random_chain_problem
    prob = random_chain_problem(seed)
    rng = W.SplitMix64(seed + 77)
    reqs = np.repeat(prob.req, 6)
    slo = rng.integers(20, 400, len(reqs)).astype(np.uint32)
    prob = prob.with_requests(reqs, slo)
    p, keys, _ = run_gpu(F, planner, prob, verify=False)
    o = oracle.plan(prob, checks=False)
    assert_plans_equal(p, o)
    req, slo_d = F.to_device(prob)
    planner.set_search_mode(F.SEARCH_EXHAUSTIVE)
    try:
        ex = planner.plan_keys(req, slo_d, prob.k_max).cpu().numpy()
    finally:
        planner.set_search_mode(F.SEARCH_BOUNDED)
    np.testing.assert_array_equal(ex, o["key"])


def test_bounded_list_path_and_fallback(F, planner):
    """The bounded mode compacts live masks for KS = 2..4 and walks the records; a context
    whose list is too small for a segment falls back to the task ranges inside the search
    kernel -- same keys either way (C3 subset)."""
    import os
    prob = W.config3(R=16384)
    planner.stage(prob)
    req, slo = F.to_device(prob)
    K = prob.k_max
    keys = planner.plan_keys(req, slo, K).cpu().numpy()
    live = planner.live_records()
    assert all(live[k] > 0 for k in (1, 2, 3)) and live[0] == 0 and sum(live[4:]) == 0
    planner.set_search_mode(F.SEARCH_EXHAUSTIVE)
    try:
        ex = planner.plan_keys(req, slo, K).cpu().numpy()
    finally:
        planner.set_search_mode(F.SEARCH_BOUNDED)
    np.testing.assert_array_equal(keys, ex)
    os.environ["FFS_LIST_CAP"] = "16"
    try:
        small = F.Planner(0)
    finally:
        del os.environ["FFS_LIST_CAP"]
    small.stage(prob)
    k2 = small.plan_keys(req, slo, K).cpu().numpy()
    assert small.live_records()[3] > 16  # KS = 4 overflowed: task-range fallback
    np.testing.assert_array_equal(k2, ex)
    small.close()


def test_bad_requests_and_empty(F, planner):
    prob = random_tiny(1001)
    req = prob.req.copy()
    req["func"][0] = 99
    req["node"][1] = 7
    bad = prob.with_requests(req, prob.slo_us)
    p, keys, ch = run_gpu(F, planner, bad)
    assert p["status"][0] == 2 and p["status"][1] == 2
    assert (ch[:2] == 0).all()
    o = oracle.plan(bad)
    assert_plans_equal(p, o)
    empty = prob.subset(np.arange(0))
    planner.stage(empty)
    req_t, slo_t = F.to_device(empty)
    out = planner.plan_batch(req_t, slo_t, 4)
    assert out.shape[0] == 0


def test_validation_errors(F, planner):
    prob = random_tiny(1002)
    bad = prob.with_requests(prob.req, prob.slo_us)
    bad.lat_us = prob.lat_us.copy()
    bad.lat_us[0, 0] = 0
    with pytest.raises(F.FFSError) as e:
        planner.stage(bad)
    assert e.value.status == F.FFS_ERR_ARG
    bad2 = prob.with_requests(prob.req, prob.slo_us)
    bad2.slices = prob.slices[::-1].copy()
    with pytest.raises(F.FFSError) as e:
        planner.stage(bad2)
    assert e.value.status == F.FFS_ERR_ARG
    bad3 = prob.with_requests(prob.req, prob.slo_us)
    bad3.lat_us = prob.lat_us.copy()
    bad3.lat_us[:, :] = 1 << 23
    with pytest.raises(F.FFSError) as e:
        planner.stage(bad3)
    assert e.value.status == F.FFS_ERR_RANGE
    planner.stage(prob)
    req, slo = F.to_device(prob)
    with pytest.raises(F.FFSError) as e:
        planner.plan_keys(req, slo, 9)
    assert e.value.status == F.FFS_ERR_RANGE


def test_host_entry_point_matches(F, planner):
    prob = W.config2(R=1024)
    p, _, _ = run_gpu(F, planner, prob, verify=False)
    h = planner.plan_batch_host(np.ascontiguousarray(prob.req), np.ascontiguousarray(prob.slo_us), prob.k_max)
    np.testing.assert_array_equal(h.view(np.uint8), p.view(np.uint8))


def test_eviction_scores_and_victims(F, planner):
    """C4 at full size: every instance score and state of all 4096 ticks and the victim
    of every load, against the oracle."""
    wl = W.config4()
    assert len(wl.now_us) == 4096
    prob = wl.problem
    planner.stage(prob)
    inst = torch.from_numpy(wl.inst.view(np.uint8)).cuda()
    toff = torch.from_numpy(wl.tick_off.view(np.int32)).cuda()
    now = torch.from_numpy(wl.now_us.view(np.int64)).cuda()
    score, state = planner.evict_scores_ticks(inst, toff, now, window_us=wl.window_us)
    req, slo = F.to_device(prob)
    rt = torch.from_numpy(wl.req_tick.view(np.int32)).cuda()
    vic = planner.evict_victims(req, slo, rt, inst, toff, score)
    torch.cuda.synchronize()
    score, state, vic = score.cpu().numpy(), state.cpu().numpy(), vic.cpu().numpy()
    for t in range(len(wl.now_us)):
        a, b = int(wl.tick_off[t]), int(wl.tick_off[t + 1])
        ev = oracle.evict(wl.inst[a:b], int(wl.now_us[t]), 30, wl.window_us)
        np.testing.assert_array_equal(score[a:b], abi_evict_score(ev))
        np.testing.assert_array_equal(state[a:b], ev.state)
        rs = np.where(wl.req_tick == t)[0]
        sub = prob.subset(rs)
        v_o = oracle.victim(sub, np.full(len(rs), oracle.PLAN_INFEASIBLE, np.int32), wl.inst[a:b], ev)
        np.testing.assert_array_equal(vic[rs], v_o)
    assert (vic >= 0).sum() > 0


def test_evict_step_fused_matches_separate_calls(F, planner):
    """ffs_evict_step (scores + per-tick victim table in one pass, then picks) equals
    ffs_evict_scores_ticks + ffs_evict_victims bit for bit on C4 (all 4096 ticks), also
    with loads whose tick is out of range and with no loads at all."""
    wl = W.config4()
    prob = wl.problem
    planner.stage(prob)
    inst = torch.from_numpy(wl.inst.view(np.uint8)).cuda()
    toff = torch.from_numpy(wl.tick_off.view(np.int32)).cuda()
    now = torch.from_numpy(wl.now_us.view(np.int64)).cuda()
    req, slo = F.to_device(prob)
    rt_np = wl.req_tick.astype(np.uint32).copy()
    rt_np[::13] = len(wl.now_us) + 1
    rt = torch.from_numpy(rt_np.view(np.int32)).cuda()
    s1, st1 = planner.evict_scores_ticks(inst, toff, now, window_us=wl.window_us)
    v1 = planner.evict_victims(req, slo, rt, inst, toff, s1)
    s2, st2, v2 = planner.evict_step(inst, toff, now, req, slo, rt, window_us=wl.window_us)
    assert torch.equal(s1, s2) and torch.equal(st1, st2) and torch.equal(v1, v2)
    assert int((v2 >= 0).sum()) > 0 and bool((v2[::13] == -1).all())
    # loads grouped by tick (the C4 batch is tick-sorted): picks inside the tick's CTA
    T = len(wl.now_us)
    lo = torch.from_numpy(np.searchsorted(wl.req_tick, np.arange(T + 1)).astype(np.int32)).cuda()
    rt_all = torch.from_numpy(wl.req_tick.view(np.int32)).cuda()
    v_ref = planner.evict_victims(req, slo, rt_all, inst, toff, s1)
    s4, st4, v4 = planner.evict_step(inst, toff, now, req, slo, load_off=lo, window_us=wl.window_us)
    assert torch.equal(s1, s4) and torch.equal(st1, st4) and torch.equal(v_ref, v4)
    s3, st3, _ = planner.evict_step(inst, toff, now, req[:0], slo[:0], rt[:0], window_us=wl.window_us)
    assert torch.equal(s1, s3) and torch.equal(st1, st3)


def test_eviction_epoch_timestamps_and_range(F, planner):
    """Unix-epoch microsecond timestamps (~1.8e15 > 2^43) score like small ones (the LRU key
    packs cold_after - idle, not the timestamp); a future last use counts as idle 0; a
    cold_after >= 2^43 (the only unpackable input) is FFS_ERR_RANGE."""
    wl = W.config4(T=1)
    planner.stage(wl.problem)
    base = 1_800_000_000_000_000
    a = wl.inst.copy()
    a["last_used_us"] = a["last_used_us"] - int(wl.now_us[0]) + base
    a["last_used_us"][::11] = base + 5  # in the future
    inst = torch.from_numpy(a.view(np.uint8)).cuda()
    score, state = planner.evict_scores(inst, base, window_us=wl.window_us)
    ev = oracle.evict(a, base, 30, wl.window_us)
    np.testing.assert_array_equal(score.cpu().numpy(), abi_evict_score(ev))
    np.testing.assert_array_equal(state.cpu().numpy(), ev.state)
    assert ev.evictable.sum() > 10
    with pytest.raises(F.FFSError) as e:
        planner.evict_scores(inst, base, window_us=wl.window_us, cold_after_us=1 << 43)
    assert e.value.status == F.FFS_ERR_RANGE


def test_victims_table_and_scan_paths_agree(F, planner):
    """The per-(tick, node, profile) table path and the warp-scan path (taken when the table
    would exceed 256 MiB: here forced by appending empty ticks) give the same victims;
    requests whose tick is out of range get -1 on both."""
    wl = W.config4(T=32)
    prob = wl.problem
    planner.stage(prob)
    inst = torch.from_numpy(wl.inst.view(np.uint8)).cuda()
    toff = torch.from_numpy(wl.tick_off.view(np.int32)).cuda()
    now = torch.from_numpy(wl.now_us.view(np.int64)).cuda()
    score, _ = planner.evict_scores_ticks(inst, toff, now, window_us=wl.window_us)
    req, slo = F.to_device(prob)
    rt_np = wl.req_tick.astype(np.uint32).copy()
    rt_np[::7] = len(wl.now_us)  # out of range for the table path
    rt = torch.from_numpy(rt_np.view(np.int32)).cuda()
    v_tab = planner.evict_victims(req, slo, rt, inst, toff, score).cpu().numpy()
    pad = 256 * 2**20 // (prob.n_nodes * 5 * 8) + 1
    toff_big = np.concatenate([wl.tick_off, np.full(pad, wl.tick_off[-1], wl.tick_off.dtype)])
    toff_big = torch.from_numpy(toff_big.view(np.int32)).cuda()
    rt_np[::7] = len(toff_big) + 3  # beyond the padded range too
    rt = torch.from_numpy(rt_np.view(np.int32)).cuda()
    v_scan = planner.evict_victims(req, slo, rt, inst, toff_big, score).cpu().numpy()
    np.testing.assert_array_equal(v_tab, v_scan)
    assert (v_tab[::7] == -1).all() and (v_tab >= 0).sum() > 0


def test_decode_victims_single_snapshot(F, planner):
    wl = W.config4(T=1)
    prob = wl.problem
    p, keys, _ = run_gpu(F, planner, prob, verify=False)
    inst = torch.from_numpy(wl.inst.view(np.uint8)).cuda()
    score, _ = planner.evict_scores(inst, int(wl.now_us[0]), window_us=wl.window_us)
    req, slo = F.to_device(prob)
    plans = F.plans_to_numpy(planner.plan_decode(req, slo, torch.from_numpy(keys).cuda(), prob.k_max, inst, score))
    o = oracle.plan(prob, checks=False)
    ev = oracle.evict(wl.inst, int(wl.now_us[0]), 30, wl.window_us)
    v_o = oracle.victim(prob, o["status"], wl.inst, ev)
    np.testing.assert_array_equal(plans["victim"], v_o)


def test_decode_victims_many_instances(F, planner):
    """Victims in ffs_plan_decode with 50,000 instances on the C3 cluster (the per-(node,
    profile) minima path, O(n_inst + n_req)) against the oracle's direct LRU scan."""
    prob = W.config3(R=4096)
    planner.stage(prob)
    rng = W.SplitMix64(808)
    n = 50_000
    inst = np.zeros(n, dtype=W.INST_DTYPE)
    inst["func"] = rng.integers(0, prob.F - 1, n)
    inst["slice"] = rng.integers(-1, len(prob.slices) - 1, n)
    inst["flags"] = np.where(rng.uniform(n) < 0.1, W.INST_BUSY, 0)
    inst["busy_us"] = rng.integers(0, 4_000_000, n)
    now = 10**12
    inst["last_used_us"] = now - rng.integers(0, 700_000_000, n).astype(np.uint64)
    d_inst = torch.from_numpy(inst.view(np.uint8)).cuda()
    score, _ = planner.evict_scores(d_inst, now, window_us=10_000_000)
    req, slo = F.to_device(prob)
    keys = planner.plan_keys(req, slo, prob.k_max)
    plans = F.plans_to_numpy(planner.plan_decode(req, slo, keys, prob.k_max, d_inst, score))
    o = oracle.plan(prob, checks=False)
    ev = oracle.evict(inst, now, 30, 10_000_000)
    v_o = oracle.victim(prob, o["status"], inst, ev)
    np.testing.assert_array_equal(plans["victim"], v_o)
    assert (v_o >= 0).sum() > 20


# ---- NEXT-1: ranked first-fit ----------------------------------------------
def run_ranked(F, planner, prob, p_ref=4):
    planner.stage(prob)
    planner.rank_partitions(prob.k_max, p_ref)
    req, slo = F.to_device(prob)
    out = planner.plan_ranked(req, slo)
    torch.cuda.synchronize()
    return F.plans_to_numpy(out)


@pytest.mark.parametrize("seed", range(1000, 1016))
def test_ranked_tiny_random(F, planner, seed):
    prob = random_tiny(seed, n_max=5, K=4)
    for p_ref in (0, 4):
        p = run_ranked(F, planner, prob, p_ref)
        assert_plans_equal(p, oracle.plan_ranked(prob, p_ref=p_ref))


@pytest.mark.parametrize("cfg", ["C1", "C2", "C3"])
def test_ranked_configs(F, planner, cfg):
    prob = {"C1": W.config1, "C2": W.config2, "C3": lambda: W.config3(R=8192)}[cfg]()
    p = run_ranked(F, planner, prob)
    assert_plans_equal(p, oracle.plan_ranked(prob))


def test_ranked_c5_sample(F, planner):
    prob = W.config5()
    p = run_ranked(F, planner, prob)
    idx = np.arange(0, prob.R, 1021)
    assert_plans_equal(p, oracle.plan_ranked(prob.subset(idx)), idx)


# ---- NEXT-2: joint commit ------------------------------------------------
def run_joint(F, planner, prob):
    planner.stage(prob)
    req, slo = F.to_device(prob)
    out, rounds = planner.plan_joint(req, slo, prob.k_max)
    return F.plans_to_numpy(out), rounds


@pytest.mark.parametrize("seed", range(1000, 1016))
def test_joint_tiny_random(F, planner, seed):
    prob = random_tiny(seed)
    p, _ = run_joint(F, planner, prob)
    assert_plans_equal(p, oracle.plan_joint(prob))


@pytest.mark.parametrize("cfg", ["C1", "C2", "C3s"])
def test_joint_configs(F, planner, cfg):
    prob = {"C1": W.config1, "C2": W.config2, "C3s": lambda: W.config3(R=4096)}[cfg]()
    p, rounds = run_joint(F, planner, prob)
    assert_plans_equal(p, oracle.plan_joint(prob))
    used = p["slice"][p["status"] == 0].ravel()
    used = used[used >= 0]
    assert len(used) == len(set(used.tolist()))  # jointly feasible
    assert rounds >= 1


# ---- NEXT-3: frontier precompute -----------------------------------------------------------
@pytest.mark.parametrize("cfg", ["tiny", "C1", "C2", "C3s"])
def test_frontier_plans_equal_argmin_plans(F, planner, cfg):
    prob = {"tiny": lambda: random_tiny(1003), "C1": W.config1, "C2": W.config2,
            "C3s": lambda: W.config3(R=8192)}[cfg]()
    p_arg, _, _ = run_gpu(F, planner, prob, verify=False)
    groups, rounds = planner.frontier_build(prob.k_max)
    req, slo = F.to_device(prob)
    p_fr = F.plans_to_numpy(planner.plan_frontier(req, slo))
    torch.cuda.synchronize()
    np.testing.assert_array_equal(p_fr.view(np.uint8), p_arg.view(np.uint8))  # identical plans
    assert rounds >= 1 and groups >= 1
    if cfg in ("tiny", "C1"):
        assert_plans_equal(p_fr, oracle.plan(prob, checks=False))


def test_frontier_c5_sample(F, planner):
    prob = W.config5()
    planner.stage(prob)
    planner.frontier_build(prob.k_max)
    req, slo = F.to_device(prob)
    p = F.plans_to_numpy(planner.plan_frontier(req, slo))
    idx = np.arange(0, prob.R, 2053)
    assert_plans_equal(p, oracle.plan(prob.subset(idx), checks=False), idx)


def test_next_rows_error_states(F):
    pl = F.Planner(0)
    prob = random_tiny(1004)
    req, slo = F.to_device(prob)
    for call in (lambda: pl.plan_ranked(req, slo), lambda: pl.plan_frontier(req, slo),
                 lambda: pl.plan_joint(req, slo, 4)):
        with pytest.raises(F.FFSError) as e:
            call()
        assert e.value.status == F.FFS_ERR_STATE
    pl.stage(prob)
    with pytest.raises(F.FFSError) as e:
        pl.rank_partitions(4, 5)  # p_ref >= P
    assert e.value.status == F.FFS_ERR_RANGE
    pl.frontier_build(4)
    pl.stage(prob)  # re-staging invalidates derived structures
    with pytest.raises(F.FFSError) as e:
        pl.plan_frontier(req, slo)
    assert e.value.status == F.FFS_ERR_STATE
    pl.close()


# ---- NEXT-2: routing -------------------------------------------------------------
def _route_case(prob, n_inst, seed):
    rng = W.SplitMix64(seed)
    func = rng.integers(0, prob.F - 1, n_inst).astype(np.uint32)
    state = rng.integers(0, 3, n_inst).astype(np.uint8)
    lat = rng.integers(1, 40, n_inst).astype(np.uint32)
    cap = rng.integers(0, 30, n_inst).astype(np.uint32)
    inst = np.zeros(n_inst, dtype=W.INST_DTYPE)
    inst["func"] = func
    return inst, state, lat, cap


@pytest.mark.parametrize("cfg,n_inst", [("tiny", 9), ("C2", 40), ("C3", 3000), ("C4", 0)])
def test_route_matches_oracle(F, planner, cfg, n_inst):
    if cfg == "C4":
        wl = W.config4(T=1)
        prob = wl.problem
        inst = wl.inst
        state = oracle.evict(inst, int(wl.now_us[0]), 30, wl.window_us).state
        rng = W.SplitMix64(3)
        lat = rng.integers(1, 100, len(inst)).astype(np.uint32)
        cap = rng.integers(0, 3, len(inst)).astype(np.uint32)
    else:
        prob = {"tiny": lambda: random_tiny(1009), "C2": W.config2, "C3": W.config3}[cfg]()
        inst, state, lat, cap = _route_case(prob, n_inst, 11)
    planner.stage(prob)
    req, slo = F.to_device(prob)
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a).view(np.uint8) if a.dtype == W.INST_DTYPE else a).cuda()
    route = planner.route(req, slo, t(inst), t(state), t(lat.view(np.int32)), t(cap.view(np.int32)))
    torch.cuda.synchronize()
    exp = oracle.route(prob, inst["func"], state, lat, cap)
    np.testing.assert_array_equal(route.cpu().numpy(), exp)


def check_plan_properties(prob, p):
    """Properties that hold at any size, checked on every request (vectorised numpy):
    (a) ESG placement when a single free slice holds the function within the budget,
    (d) e2e / bottleneck / cvq / gpcs recomputed from the tables, slices valid."""
    R, P = prob.R, prob.P
    f = prob.req["func"].astype(np.int64)
    v = prob.req["node"].astype(np.int64)
    B = prob.slo_us.astype(np.int64)
    off = prob.comp_off.astype(np.int64)
    n = off[f + 1] - off[f]
    lat = prob.lat_us.astype(np.int64)
    PL = np.zeros((lat.shape[0] + 1, P), np.int64)
    PL[1:] = np.cumsum(lat, axis=0)
    PM = np.concatenate([[0], np.cumsum(prob.mem_mib.astype(np.int64))])
    sl = prob.slices
    free = np.zeros((prob.n_nodes, P), np.int64)
    np.add.at(free, (sl["node"][sl["busy"] == 0].astype(np.int64), sl["profile"][sl["busy"] == 0].astype(np.int64)), 1)
    cap = prob.cap_mib.astype(np.int64)
    g = prob.gpcs.astype(np.int64)
    # (a) ESG placement
    tot_mem = PM[off[f + 1]] - PM[off[f]]
    tot_lat = PL[off[f + 1]] - PL[off[f]]                     # [R, P]
    ok1 = (free[v] > 0) & (tot_mem[:, None] <= cap[None, :]) & (tot_lat <= B[:, None])
    has = ok1.any(axis=1)
    esg = np.where(ok1, g[None, :] * 16 + np.arange(P)[None, :], 10**9).argmin(axis=1)
    assert (p["k"][has] == 1).all() and (p["prof"][has, 0] == esg[has]).all()
    # (d) recompute every OK plan from the tables
    ok = p["status"] == 0
    k = p["k"].astype(np.int64)
    mask = p["cut_mask"].astype(np.int64)
    St = np.zeros(R, np.int64); Sq = np.zeros(R, np.int64); bott = np.zeros(R, np.int64)
    X = np.zeros(R, np.int64); gp = np.zeros(R, np.int64)
    a = np.zeros(R, np.int64); m = mask.copy()
    used = np.zeros((R, P), np.int64)
    for i in range(8):
        live = ok & (i < k)
        last = live & (i == k - 1)
        low = m & -m
        j = np.where(m > 0, np.log2(np.maximum(low, 1)).astype(np.int64), 0)
        b = np.where(last, n, j + 1)
        pr = np.where(live, p["prof"][:, i].astype(np.int64), 0)
        t = np.where(live, PL[off[f] + b, pr] - PL[off[f] + a, pr], 0)
        mem = np.where(live, PM[off[f] + b] - PM[off[f] + a], 0)
        assert (mem[live] <= cap[pr[live]]).all()
        X += np.where(live & ~last, prob.xfer_us[np.minimum(off[f] + j, len(prob.xfer_us) - 1)].astype(np.int64), 0)
        St += t; Sq += t * t; bott = np.maximum(bott, t); gp += np.where(live, g[pr], 0)
        np.add.at(used, (np.arange(R)[live], pr[live]), 1)
        m = np.where(live & ~last, m & (m - 1), m)
        a = np.where(live, b, a)
    assert (p["e2e_us"][ok] == (St + X)[ok]).all() and (St + X <= B)[ok].all()
    assert (p["bottleneck_us"][ok] == bott[ok]).all() and (p["gpcs"][ok] == gp[ok]).all()
    D = St * St
    Nn = k * Sq - D
    cvq = np.where(ok, (Nn << 10) // np.maximum(D, 1), 0)
    assert (p["cvq"][ok] == cvq[ok]).all() and ((p["key"][ok] >> 50) == cvq[ok]).all()
    assert (used[ok] <= free[v[ok]]).all()
    s = p["slice"][ok]
    live = s >= 0
    assert (sl["node"][s[live]] == np.repeat(v[ok], (live).sum(axis=1))).all()
    assert (sl["busy"][s[live]] == 0).all()
    assert (sl["profile"][s[live]] == p["prof"][ok][live]).all()


@pytest.mark.parametrize("cfg", ["C3", "C5"])
def test_host_entry_point_large(F, planner, cfg):
    """ffs_plan_batch_host at C3 / C5 size: byte-identical to ffs_plan_batch on the
    device-resident batch, with pinned and with pageable host buffers."""
    import torch
    prob = W.config3() if cfg == "C3" else W.config5()
    planner.stage(prob)
    req, slo = F.to_device(prob)
    ref = F.plans_to_numpy(planner.plan_batch(req, slo, prob.k_max))
    h_req = torch.from_numpy(np.ascontiguousarray(prob.req).view(np.uint8)).pin_memory()
    h_slo = torch.from_numpy(np.ascontiguousarray(prob.slo_us).view(np.uint8)).pin_memory()
    h_out = torch.zeros(prob.R * 80, dtype=torch.uint8).pin_memory()
    out = h_out.numpy().view(F.PLAN_DTYPE)
    planner.plan_batch_host(h_req.numpy().view(W.REQ_DTYPE), h_slo.numpy().view(np.uint32), prob.k_max, out=out)
    np.testing.assert_array_equal(out.view(np.uint8), ref.view(np.uint8))
    pageable = planner.plan_batch_host(np.ascontiguousarray(prob.req), np.ascontiguousarray(prob.slo_us), prob.k_max)
    np.testing.assert_array_equal(pageable.view(np.uint8), ref.view(np.uint8))


def test_host_entry_point_ragged_slices(F, planner):
    """A batch just above 2^20 requests (two uneven host slices; the exhaustive mode's
    grouped walks on both): ffs_plan_batch_host = ffs_plan_batch on the device batch."""
    import torch
    base = W.config5()
    idx = np.concatenate([np.arange(base.R), np.arange(0, 37 * 997, 997)])
    prob = base.subset(idx)
    planner.stage(prob)
    req, slo = F.to_device(prob)
    try:
        planner.set_search_mode(F.SEARCH_EXHAUSTIVE)
        ref = F.plans_to_numpy(planner.plan_batch(req, slo, prob.k_max))
        h_req = torch.from_numpy(np.ascontiguousarray(prob.req).view(np.uint8)).pin_memory()
        h_slo = torch.from_numpy(np.ascontiguousarray(prob.slo_us).view(np.uint8)).pin_memory()
        out = torch.zeros(prob.R * 80, dtype=torch.uint8).pin_memory().numpy().view(F.PLAN_DTYPE)
        planner.plan_batch_host(h_req.numpy().view(W.REQ_DTYPE), h_slo.numpy().view(np.uint32), prob.k_max,
                                out=out)
    finally:
        planner.set_search_mode(F.SEARCH_BOUNDED)
    np.testing.assert_array_equal(out.view(np.uint8), ref.view(np.uint8))
    np.testing.assert_array_equal(ref["key"][base.R:], ref["key"][idx[base.R:]])  # duplicated requests


def test_c5_full_batch_properties(F, planner):
    prob = W.config5()
    p, _, _ = run_gpu(F, planner, prob, verify=False)
    check_plan_properties(prob, p)
    ok = p["status"] == 0
    assert ok.mean() > 0.5 and (ok & (p["k"] > 1)).mean() > 0.05 and (~ok).mean() > 0.05


# ---- NEXT-4: time-sharing simulator ----------------------------------------------------------
@pytest.mark.parametrize("case", ["small", "c4"])
def test_simulator_matches_oracle(F, planner, case):
    if case == "small":
        tr = W.sim_trace(seed=101, T=600, n_funcs=12, nodes=[W.PART_P1, W.PART_HYBRID, W.PART_P2], rate_scale=8.0)
        cold = 5_000_000
    else:
        tr = W.sim_trace(T=2048)
        cold = 60_000_000
    planner.stage(tr.problem)
    for K in (tr.problem.k_max, 0):  # with pipeline instances (R44-R46), and monolithic only
        out = planner.simulate(tr, cold_after_us=cold, k_max=K)
        torch.cuda.synchronize()
        o = oracle.sim(tr, cold_after_us=cold, k_max=K)
        _assert_sim_equal(out, o)
        assert o[0][:, 5].sum() > 0 and o[0][:, 6].sum() > 0
        assert (o[0][:, 8].sum() > 0) == (K > 0)  # pipelines are placed exactly when enabled


def _assert_sim_equal(out, o):
    ctr, sl, st, last, busy, stages = out
    np.testing.assert_array_equal(ctr.cpu().numpy().view(np.uint64), o[0])
    np.testing.assert_array_equal(sl.cpu().numpy(), o[1])
    np.testing.assert_array_equal(st.cpu().numpy(), o[2])
    np.testing.assert_array_equal(last.cpu().numpy().view(np.uint64), o[3])
    np.testing.assert_array_equal(busy.cpu().numpy().view(np.uint32), o[4])
    np.testing.assert_array_equal(stages.cpu().numpy(), o[5])


@pytest.mark.parametrize("case", ["fragmented", "never_evicted", "migration"])
def test_simulator_pipeline_hand_cases(F, planner, case):
    """The oracle's hand-worked pipeline scenarios (tests/test_oracle_sim.py) on the GPU."""
    from test_oracle_sim import pipe_funcs, make_trace, G1, G2
    if case == "fragmented":
        prob = pipe_funcs([[[G1, G1, (G2, 1)]]])
        tr, cold = make_trace(prob, 3, [(0, 0, 0, 300), (1, 0, 0, 106), (2, 0, 0, 107)], window_ticks=100), 600_000_000
    elif case == "never_evicted":
        prob = pipe_funcs([[[G1, G1]]], mem_h=5 * 1024)
        tr, cold = make_trace(prob, 2, [(0, 0, 0, 10**6), (1, 0, 1, 10**6)], window_ticks=100), 600_000_000
    else:
        prob = pipe_funcs([[[G2, G1, G1]]])
        ev = [(0, 0, 1, 10**6), (1, 0, 0, 10**6), (2, 0, 0, 10**6), (3, 0, 0, 10**6), (4, 0, 0, 75)]
        tr, cold = make_trace(prob, 5, ev, window_ticks=100), 300
    planner.stage(prob)
    o = oracle.sim(tr, cold_after_us=cold)
    _assert_sim_equal(planner.simulate(tr, cold_after_us=cold), o)
    assert o[0][0, 8] == 1


def test_large_table_image_reads_tables_from_global(F, planner):
    """800 functions: the table image no longer fits shared memory; the search reads it
    from global memory (tables_global) with identical results."""
    rng = W.SplitMix64(4242)
    lengths = rng.sub(9).integers(3, 12, 800)
    prob = W._problem("big", rng, lengths, W.NODE_BLOCK, 2048)
    p, keys, ch = run_gpu(F, planner, prob)
    o = oracle.plan(prob)
    assert_plans_equal(p, o)
    np.testing.assert_array_equal(ch, o["checks"])
    p2, keys2, _ = run_gpu(F, planner, prob, verify=False)
    np.testing.assert_array_equal(keys2, o["key"])
    assert planner.filter_misses() == 0


def _f16_stress_problem(seed):
    """KS = 4 inputs aimed at the f16x2 pre-filter's margins: latencies
    spanning 1 us .. 2^22 us (underflow / the exact 'wide' path), stages of equal time
    (CV = 0 ties), budgets exactly at a candidate's e2e (inclusive SLO) and far above the
    slowest chain (scale clamped to tmax), plus nodes with one free slice per profile."""
    rng = W.SplitMix64(seed)
    funcs = []
    for f in range(6):
        n = int(rng.integers(4, 11, 1)[0])
        kind = f % 3
        if kind == 0:    # extreme dynamic range
            lat = (2 ** rng.integers(0, 22, n * 5)).reshape(n, 5) + rng.integers(0, 3, n * 5).reshape(n, 5)
        elif kind == 1:  # equal components: many exact CV ties
            base = int(rng.integers(1000, 5000, 1)[0])
            lat = np.tile(np.array([7, 5, 3, 2, 1]) * base, (n, 1))
        else:            # ordinary, narrow spread
            lat = rng.integers(900, 1100, n * 5).reshape(n, 5)
        mem = rng.integers(1000, 9000, n).tolist()
        xfer = rng.integers(0, 40, n).tolist()
        funcs.append(dict(lat=np.asarray(lat).tolist(), mem=mem, xfer=xfer, load=10))
    nodes = [[[0, 1, 2], [3, 4]], [[0, 0, 1, 1], [2, 2, 3]], [[0], [1], [2]]]
    reqs = []
    for f, fd in enumerate(funcs):
        lat = np.asarray(fd["lat"], np.int64)
        n = lat.shape[0]
        one_stage = lat.sum(0)
        for v in range(len(nodes)):
            # exact e2e of a 4-stage candidate (equal stages, cuts after 0, 1, 2) and budgets around it
            cut = [0, 1, 2]
            stages = [lat[0:1, 0].sum(), lat[1:2, 1].sum(), lat[2:3, 2].sum(), lat[3:n, 3].sum()]
            e2e = int(sum(stages) + sum(fd["xfer"][c] for c in cut))
            for B in (e2e - 1, e2e, e2e + 1, int(one_stage.min()), int(one_stage.max()) * 4, 2 ** 30):
                reqs.append((f, v, max(int(B), 1)))
    return problem(funcs, nodes, reqs, k_max=4)


@pytest.mark.parametrize("seed", range(6))
def test_f16_prefilter_stress(F, planner, seed):
    prob = _f16_stress_problem(4200 + seed)
    p, keys, ch = run_gpu(F, planner, prob)
    o = oracle.plan(prob)
    assert_plans_equal(p, o)
    np.testing.assert_array_equal(ch, o["checks"])
    assert planner.filter_misses() == 0
    p2, keys2, _ = run_gpu(F, planner, prob, verify=False)
    np.testing.assert_array_equal(keys2, o["key"])


# ---- NEXT-2 throughput floor (R38) ------------------------------------------
def _floored(prob, seed=0xF1):
    rng = W.SplitMix64(seed)
    fl = rng.integers(0, 160, prob.F).astype(np.uint32)
    fl[rng.sub(1).uniform(prob.F) < 0.3] = 0
    return prob.__class__(**{**prob.__dict__, "max_stage_us": fl})


@pytest.mark.parametrize("seed", range(2000, 2012))
def test_floor_tiny_random(F, planner, seed):
    prob = _floored(random_tiny(seed, n_max=6, K=5), seed)
    p, keys, ch = run_gpu(F, planner, prob)
    o = oracle.plan(prob)
    assert_plans_equal(p, o)
    np.testing.assert_array_equal(ch, o["checks"])
    assert planner.filter_misses() == 0


@pytest.mark.parametrize("K", [2, 3, 4, 6])
def test_floor_configs(F, planner, K):
    # every search template (KS 1..K) with floors that bind on a C2-shaped mix
    prob = W.with_throughput_floor(W.config2(R=1024 if K <= 4 else 256))
    p, keys, ch = run_gpu(F, planner, prob, k_max=K)
    o = oracle.plan(prob, k_max=K)
    assert_plans_equal(p, o)
    np.testing.assert_array_equal(ch, o["checks"])
    assert planner.filter_misses() == 0
    p2, keys2, _ = run_gpu(F, planner, prob, k_max=K, verify=False)
    np.testing.assert_array_equal(keys2, o["key"])


def test_floor_next_paths(F, planner):
    """ranked first-fit, joint commit, frontier and victims honour the floor like the oracle."""
    prob = W.with_throughput_floor(W.config2(R=512))
    assert_plans_equal(run_ranked(F, planner, prob), oracle.plan_ranked(prob, p_ref=4))
    pj, _ = run_joint(F, planner, prob)
    assert_plans_equal(pj, oracle.plan_joint(prob))
    p_arg, keys, _ = run_gpu(F, planner, prob, verify=False)
    planner.frontier_build(prob.k_max)
    req, slo = F.to_device(prob)
    p_fr = F.plans_to_numpy(planner.plan_frontier(req, slo))
    np.testing.assert_array_equal(p_fr.view(np.uint8), p_arg.view(np.uint8))
    # victims of the infeasible requests (single snapshot, decode path)
    wl = W.config4(T=1)
    fprob = W.with_throughput_floor(wl.problem)
    p, keys, _ = run_gpu(F, planner, fprob, verify=False)
    inst = torch.from_numpy(wl.inst.view(np.uint8)).cuda()
    score, _ = planner.evict_scores(inst, int(wl.now_us[0]), window_us=wl.window_us)
    req, slo = F.to_device(fprob)
    plans = F.plans_to_numpy(planner.plan_decode(req, slo, torch.from_numpy(keys).cuda(), fprob.k_max, inst, score))
    o = oracle.plan(fprob, checks=False)
    ev = oracle.evict(wl.inst, int(wl.now_us[0]), 30, wl.window_us)
    np.testing.assert_array_equal(plans["victim"], oracle.victim(fprob, o["status"], wl.inst, ev))


# ---- NEXT-2 any-invoker (cross-node) planning (R39) --------------------------
def _run_any(F, planner, prob):
    planner.stage(prob)
    planner.frontier_build(prob.k_max)
    req, slo = F.to_device(prob)
    out, node = planner.plan_frontier_any(req, slo)
    torch.cuda.synchronize()
    return F.plans_to_numpy(out), node.cpu().numpy()


@pytest.mark.parametrize("seed", range(1000, 1008))
def test_any_invoker_tiny(F, planner, seed):
    prob = random_tiny(seed)
    p, node = _run_any(F, planner, prob)
    o, n_o = oracle.plan_any(prob)
    assert_plans_equal(p, o)
    np.testing.assert_array_equal(node, n_o)


@pytest.mark.parametrize("floor", [False, True])
def test_any_invoker_c3_sample(F, planner, floor):
    prob = W.config3()
    prob = W.with_throughput_floor(prob) if floor else prob
    idx = np.arange(0, prob.R, 97)
    sub = prob.subset(idx)
    p, node = _run_any(F, planner, sub)
    o, n_o = oracle.plan_any(sub)
    assert_plans_equal(p, o)
    np.testing.assert_array_equal(node, n_o)
    home = oracle.plan(sub, checks=False)
    assert (o["key"] <= home["key"]).all() and (o["key"] < home["key"]).any()


def test_any_invoker_bad_requests(F, planner):
    prob = random_tiny(1001)
    req = prob.req.copy()
    req["node"][0] = 99
    req["func"][1] = 77
    bad = prob.with_requests(req, prob.slo_us)
    p, node = _run_any(F, planner, bad)
    assert p["status"][0] == oracle.PLAN_BAD_REQ and p["status"][1] == oracle.PLAN_BAD_REQ
    assert node[0] == -1 and node[1] == -1
    o, n_o = oracle.plan_any(bad)
    assert_plans_equal(p, o)
