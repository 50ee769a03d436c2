"""north_star invariants (a)-(d) and the extra invariants of SURVEY §8(c), checked on the
oracle over seeded synthetic tables (CPU only).  Each check uses an independent routine
(ESG placement, min-e2e dynamic programme, exact rationals), not the oracle's own code.
"""
from functools import lru_cache
from fractions import Fraction
import statistics

import numpy as np
import pytest

import oracle
from helpers import KEY_NONE
from paper_conf_hpdc_hui0s25_b200 import workload as W

SEEDS = range(1000, 1012)


def small_problem(seed, R=48, n_lo=1, n_hi=9, nodes=None):
    rng = W.SplitMix64(seed)
    lengths = rng.sub(9).integers(n_lo, n_hi, 8)
    parts = nodes if nodes is not None else W.NODE_BLOCK
    return W._problem(f"inv{seed}", rng, lengths, parts, R)


def free_counts(prob, v):
    sl = prob.slices
    return [int(((sl["node"] == v) & (sl["busy"] == 0) & (sl["profile"] == p)).sum()) for p in range(prob.P)]


def esg_place(prob, r):
    """ESG-style monolithic placement: the most resource-efficient (fewest GPCs)
    free slice that holds the whole function and meets the SLO; lowest profile id on ties."""
    f, v, B = int(prob.req["func"][r]), int(prob.req["node"][r]), int(prob.slo_us[r])
    a, b = int(prob.comp_off[f]), int(prob.comp_off[f + 1])
    free = free_counts(prob, v)
    best = None
    for p in range(prob.P):
        if free[p] and int(prob.mem_mib[a:b].sum()) <= int(prob.cap_mib[p]) and int(prob.lat_us[a:b, p].sum()) <= B:
            if best is None or int(prob.gpcs[p]) < int(prob.gpcs[best]):
                best = p
    return best


@pytest.mark.parametrize("seed", SEEDS)
def test_a_one_stage_reproduces_esg_placement(seed):
    prob = small_problem(seed)
    o = oracle.plan(prob)
    o1 = oracle.plan(prob, k_max=1)
    for r in range(prob.R):
        p = esg_place(prob, r)
        if p is not None:
            assert o["k"][r] == 1 and o["prof"][r, 0] == p
        # with K = 1 the planner IS the monolithic placement, feasible or not
        assert (o1["status"][r] == oracle.PLAN_OK) == (p is not None)
        if p is not None:
            assert o1["prof"][r, 0] == p


@pytest.mark.parametrize("seed", SEEDS)
def test_b_freeing_a_slice_never_worsens(seed):
    prob = small_problem(seed, R=24)
    o = oracle.plan(prob)
    rng = W.SplitMix64(seed + 77)
    busy = np.where(prob.slices["busy"] == 1)[0]
    for trial in range(3):
        s = int(busy[int(rng.integers(0, len(busy) - 1, 1)[0])])
        p2 = prob.with_requests(prob.req, prob.slo_us)
        p2.slices = prob.slices.copy()
        p2.slices["busy"][s] = 0
        o2 = oracle.plan(p2)
        assert (o2["key"] <= o["key"]).all()


def min_e2e_dp(prob, r, K):
    """Independent min-e2e over chains with per-stage memory and per-profile free counts
    (dynamic programme over (next component, profile usage, stages used))."""
    f, v = int(prob.req["func"][r]), int(prob.req["node"][r])
    a, b = int(prob.comp_off[f]), int(prob.comp_off[f + 1])
    n, P = b - a, prob.P
    lat = prob.lat_us[a:b].astype(int).tolist()
    mem = prob.mem_mib[a:b].astype(int).tolist()
    xfer = prob.xfer_us[a:b].astype(int).tolist()
    free = tuple(free_counts(prob, v))
    cap = [int(c) for c in prob.cap_mib]
    INF = float("inf")

    @lru_cache(maxsize=None)
    def go(c, used, s):
        if c == n:
            return 0
        if s == K:
            return INF
        best = INF
        for e in range(c + 1, n + 1):
            m = sum(mem[c:e])
            for p in range(P):
                if used[p] >= free[p] or m > cap[p]:
                    continue
                u = list(used); u[p] += 1
                t = sum(lat[i][p] for i in range(c, e)) + (xfer[e - 1] if e < n else 0)
                best = min(best, t + go(e, tuple(u), s + 1))
        return best
    return go(0, tuple([0] * P), 0)


@pytest.mark.parametrize("seed", SEEDS)
def test_c_infeasible_iff_no_chain_fits(seed):
    prob = small_problem(seed)
    o = oracle.plan(prob)
    for r in range(prob.R):
        dp = min_e2e_dp(prob, r, prob.k_max)
        assert (o["status"][r] == oracle.PLAN_INFEASIBLE) == (dp > int(prob.slo_us[r]))
        # quick necessary conditions of SURVEY §8(c)
        f, v = int(prob.req["func"][r]), int(prob.req["node"][r])
        a, b = int(prob.comp_off[f]), int(prob.comp_off[f + 1])
        free = free_counts(prob, v)
        caps = [int(prob.cap_mib[p]) for p in range(prob.P) if free[p]]
        if not caps or int(prob.mem_mib[a:b].max()) > max(caps):
            assert o["status"][r] == oracle.PLAN_INFEASIBLE


@pytest.mark.parametrize("seed", SEEDS)
def test_d_throughput_is_inverse_bottleneck(seed):
    prob = small_problem(seed)
    o = oracle.plan(prob)
    for r in np.where(o["status"] == oracle.PLAN_OK)[0]:
        f = int(prob.req["func"][r])
        a, b = int(prob.comp_off[f]), int(prob.comp_off[f + 1])
        k, mask = int(o["k"][r]), int(o["cut_mask"][r])
        bounds = [0] + [j + 1 for j in range(b - a - 1) if mask >> j & 1] + [b - a]
        assert len(bounds) == k + 1
        t = [int(prob.lat_us[a + bounds[i]:a + bounds[i + 1], o["prof"][r, i]].sum()) for i in range(k)]
        x = sum(int(prob.xfer_us[a + j]) for j in range(b - a - 1) if mask >> j & 1)
        assert o["bottleneck_us"][r] == max(t)
        assert o["e2e_us"][r] == sum(t) + x <= prob.slo_us[r]
        tf = [Fraction(v) for v in t]
        assert o["cvq"][r] == int(statistics.pvariance(tf) / statistics.mean(tf) ** 2 * 1024)
        thr = Fraction(10 ** 6, max(t))  # requests/s of the pipeline = 1 / bottleneck stage
        assert thr == Fraction(10 ** 6, int(o["bottleneck_us"][r]))
        # bound slices: in the request's node, free, of the stage's profile, distinct
        s = o["slice"][r, :k]
        assert len(set(s.tolist())) == k and (s >= 0).all()
        assert (prob.slices["node"][s] == prob.req["node"][r]).all() and (prob.slices["busy"][s] == 0).all()
        assert (prob.slices["profile"][s] == o["prof"][r, :k]).all()


@pytest.mark.parametrize("seed", SEEDS[:6])
def test_monotone_in_budget_and_kmax(seed):
    prob = small_problem(seed)
    o = oracle.plan(prob)
    looser = prob.with_requests(prob.req, (prob.slo_us.astype(np.int64) * 5 // 4).astype(np.uint32))
    assert (oracle.plan(looser)["key"] <= o["key"]).all()
    prev = None
    for K in (1, 2, 3, 4):
        k = oracle.plan(prob, k_max=K)["key"]
        if prev is not None:
            assert (k <= prev).all()
        prev = k


@pytest.mark.parametrize("seed", SEEDS[:6])
def test_scaling_latencies_keeps_the_plan(seed):
    prob = small_problem(seed)
    o = oracle.plan(prob)
    p3 = prob.with_requests(prob.req, prob.slo_us)
    p3.lat_us = prob.lat_us * 3
    p3.xfer_us = prob.xfer_us * 3
    p3.slo_us = (prob.slo_us.astype(np.int64) * 3).clip(0, 2**32 - 1).astype(np.uint32)
    keep = prob.slo_us.astype(np.int64) * 3 < 2**32
    o3 = oracle.plan(p3)
    assert (o3["key"][keep] == o["key"][keep]).all()


def test_permuting_requests_permutes_plans():
    prob = small_problem(1234)
    o = oracle.plan(prob)
    perm = np.argsort(W.SplitMix64(9).u64(prob.R))
    op = oracle.plan(prob.subset(perm))
    for name in ("key", "status", "k", "cut_mask", "e2e_us", "prof", "slice"):
        assert (op[name] == o[name][perm]).all()


def test_single_thread_equals_multi_thread():
    prob = small_problem(4321)
    a = oracle.plan(prob, threads=1)
    b = oracle.plan(prob, threads=5)
    for name in a:
        assert (a[name] == b[name]).all()


def test_generator_mix_acceptance_c2():
    """SURVEY §8(d) acceptance on the C2 draw: >=10% multi-stage, >=5% infeasible,
    >=20% 1-stage winners (so parity is not trivially satisfied)."""
    prob = W.config2()
    o = oracle.plan(prob, checks=False)
    ok = o["status"] == oracle.PLAN_OK
    assert (ok & (o["k"] > 1)).mean() >= 0.10
    assert (o["status"] == oracle.PLAN_INFEASIBLE).mean() >= 0.05
    assert (ok & (o["k"] == 1)).mean() >= 0.20
