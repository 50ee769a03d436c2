"""Pins of the NEXT-1 oracle (offline CV ranking + first-fit walk): an
independent Python reading (Fractions, itertools, sorted()) and a hand-worked case."""
import statistics
from fractions import Fraction

import numpy as np
import pytest

import oracle
from helpers import problem
from test_oracle_pins import random_tiny
from paper_conf_hpdc_hui0s25_b200 import workload as W

G1, G2, G3, G4, G7 = range(5)
GB = 1024


def ranked_brute(prob, r, p_ref=None):
    P = prob.P
    p_ref = int(np.argmax(prob.gpcs)) if p_ref is None else p_ref
    f, v, B = int(prob.req["func"][r]), int(prob.req["node"][r]), int(prob.slo_us[r])
    a, b = int(prob.comp_off[f]), int(prob.comp_off[f + 1])
    n = b - a
    lat = prob.lat_us[a:b].astype(int).tolist()
    mem = prob.mem_mib[a:b].astype(int).tolist()
    xfer = prob.xfer_us[a:b].astype(int).tolist()
    cap = [int(c) for c in prob.cap_mib]
    g = [int(x) for x in prob.gpcs]
    sl = prob.slices
    free = [int(((sl["node"] == v) & (sl["busy"] == 0) & (sl["profile"] == p)).sum()) for p in range(P)]
    fl = getattr(prob, "max_stage_us", None)
    floor = 0 if fl is None else int(fl[f])  # R38 throughput floor

    def fast_enough(lo, hi, p):
        return floor == 0 or sum(lat[c][p] for c in range(lo, hi)) <= floor

    parts = []
    for mask in range(1 << (n - 1)):
        k = bin(mask).count("1") + 1
        if k > prob.k_max:
            continue
        bounds = [0] + [j + 1 for j in range(n - 1) if mask >> j & 1] + [n]
        t = [Fraction(sum(lat[c][p_ref] for c in range(bounds[i], bounds[i + 1]))) for i in range(k)]
        cvq = int(statistics.pvariance(t) / statistics.mean(t) ** 2 * 1024)
        parts.append((cvq, k, mask, bounds))
    parts.sort()
    order = sorted(range(P), key=lambda p: (cap[p], g[p], p))
    for pos, (cvq_ref, k, mask, bounds) in enumerate(parts):
        m = [sum(mem[bounds[i]:bounds[i + 1]]) for i in range(k)]
        left = list(free)
        prof = [None] * k
        for s in sorted(range(k), key=lambda i: (-m[i], i)):
            for p in order:
                if left[p] > 0 and m[s] <= cap[p] and fast_enough(bounds[s], bounds[s + 1], p):
                    prof[s] = p
                    left[p] -= 1
                    break
        if None in prof:
            continue
        t = [sum(lat[c][prof[i]] for c in range(bounds[i], bounds[i + 1])) for i in range(k)]
        e2e = sum(t) + sum(xfer[j] for j in range(n - 1) if mask >> j & 1)
        if e2e > B:
            continue
        return dict(key=pos, k=k, mask=mask, prof=prof, e2e=e2e)
    return None


@pytest.mark.parametrize("seed", range(1000, 1030))
def test_ranked_matches_independent_reading(seed):
    prob = random_tiny(seed, n_max=5, K=4)
    o = oracle.plan_ranked(prob, threads=2)
    for r in range(prob.R):
        exp = ranked_brute(prob, r)
        if exp is None:
            assert o["status"][r] == oracle.PLAN_INFEASIBLE
            continue
        assert o["status"][r] == oracle.PLAN_OK
        assert o["key"][r] == exp["key"] and o["k"][r] == exp["k"] and o["cut_mask"][r] == exp["mask"]
        assert list(o["prof"][r, :exp["k"]]) == exp["prof"] and o["e2e_us"][r] == exp["e2e"]


@pytest.mark.parametrize("seed", range(3000, 3020))
def test_ranked_with_floor_matches_independent_reading(seed):
    prob = random_tiny(seed, n_max=5, K=4)
    rng = W.SplitMix64(seed ^ 0xF1)
    fl = rng.integers(0, 160, prob.F).astype(np.uint32)
    prob = prob.__class__(**{**prob.__dict__, "max_stage_us": fl})
    o = oracle.plan_ranked(prob, threads=2)
    for r in range(prob.R):
        exp = ranked_brute(prob, r)
        if exp is None:
            assert o["status"][r] == oracle.PLAN_INFEASIBLE
            continue
        assert o["status"][r] == oracle.PLAN_OK
        assert o["key"][r] == exp["key"] and o["k"][r] == exp["k"] and o["cut_mask"][r] == exp["mask"]
        assert list(o["prof"][r, :exp["k"]]) == exp["prof"] and o["e2e_us"][r] == exp["e2e"]


def test_ranked_hand_case():
    # Reference (7g) stage times of the partitions (components 10, 10, 20 us on 7g):
    #   rank 0: [c0 c1 c2]    (40)          cvq 0, k=1
    #   rank 1: [c0 c1 | c2]  (20, 20)      cvq 0, k=2
    #   rank 2: [c0|c1|c2]    (10, 10, 20)  CV^2 = 1/8 -> cvq 128
    #   rank 3: [c0 | c1 c2]  (10, 30)      CV^2 = 1/4 -> cvq 256
    # Memory 12 + 12 + 6 GB.  Free {2g, 1g}: 30 GB and 24 GB fit no free slice, the
    # 3-stage split needs two slices >= 12 GB, [12 | 18] needs two 2g -> INFEASIBLE.
    # Free {2g, 2g, 1g}: rank 2 is supported with (2g, 2g, 1g):
    #   e2e = 30 (c0 on 2g) + 30 (c1 on 2g) + 80 (c2 on 1g) + 2 cuts x 100 = 340.
    lat = [[40, 30, 25, 20, 10], [40, 30, 25, 20, 10], [80, 60, 50, 40, 20]]
    f = dict(lat=lat, mem=[12 * GB, 12 * GB, 6 * GB], xfer=[100, 100, 0])
    p1 = problem([f], [[[G2, G1]]], [(0, 0, 10**6)], k_max=3)
    o = oracle.plan_ranked(p1)
    assert o["status"][0] == oracle.PLAN_INFEASIBLE
    p2 = problem([f], [[[G2, G2, G1]]], [(0, 0, 10**6), (0, 0, 339)], k_max=3)
    o = oracle.plan_ranked(p2)
    assert o["status"][0] == oracle.PLAN_OK and o["k"][0] == 3 and o["cut_mask"][0] == 0b11
    assert list(o["prof"][0, :3]) == [G2, G2, G1] and list(o["slice"][0, :3]) == [0, 1, 2]
    assert o["key"][0] == 2 and o["e2e_us"][0] == 340
    # budget 339: rank 2 misses the SLO (340); rank 3 [c0 | c1 c2] = 12 | 18 GB takes the
    # two 2g slices: e2e = 30 + (30 + 60) + 100 = 220 <= 339 -> chosen
    assert o["status"][1] == oracle.PLAN_OK and o["key"][1] == 3 and o["cut_mask"][1] == 0b01
    assert list(o["prof"][1, :2]) == [G2, G2] and o["e2e_us"][1] == 220


def test_ranked_rank0_is_the_smallest_monolithic_fit():
    # rank 0 is the 1-stage partition (CV = 0).  When the smallest-capacity free profile
    # that holds the whole function meets the SLO, the walk stops there (k = 1 on it).
    prob = W.config2(R=256)
    o = oracle.plan_ranked(prob)
    sl = prob.slices
    hits = 0
    for r in range(prob.R):
        f, v, B = int(prob.req["func"][r]), int(prob.req["node"][r]), int(prob.slo_us[r])
        a, b = int(prob.comp_off[f]), int(prob.comp_off[f + 1])
        mem = int(prob.mem_mib[a:b].sum())
        fits = [p for p in range(prob.P)
                if ((sl["node"] == v) & (sl["busy"] == 0) & (sl["profile"] == p)).any() and mem <= prob.cap_mib[p]]
        if not fits:
            continue
        p = min(fits, key=lambda q: (int(prob.cap_mib[q]), int(prob.gpcs[q]), q))
        if int(prob.lat_us[a:b, p].sum()) <= B:
            hits += 1
            assert o["k"][r] == 1 and o["prof"][r, 0] == p and o["key"][r] == 0
    assert hits > 0
