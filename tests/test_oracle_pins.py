"""Pins of the CPU oracle against things other than itself (CPU only).

Hand enumerations, the paper's worked scenarios (Fig. 1, Fig. 4 P:186,
Table 5, Eq. 1), closed forms for the candidate count and an
independent Python brute force (tests/helpers.brute_plan).
"""
import json
import os
from fractions import Fraction
from math import comb
import statistics

import numpy as np
import pytest

import oracle
from helpers import problem, pack_key, brute_plan, KEY_NONE
from paper_conf_hpdc_hui0s25_b200 import workload as W

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
G1, G2, G3, G4, G7 = range(5)
GB = 1024


def flat(lat_by_profile, n):
    """n components, every component with the same per-profile latency list."""
    return [list(lat_by_profile) for _ in range(n)]


def test_n1_five_candidates_by_hand():
    # one component; 1g too small for 15000 MiB; 3g not free; budget excludes 2g
    f = dict(lat=[[50, 40, 30, 20, 10]], mem=[15000])
    prob = problem([f], [[[G1, G2, G4]]], [(0, 0, 35), (0, 0, 50), (0, 0, 5)])
    o = oracle.plan(prob)
    # budget 35: 2g (40us) misses the SLO, 4g (20us) is the only feasible one, idx 3
    assert o["key"][0] == pack_key(0, 1, 4, 3)
    assert list(o["checks"][0]) == [5, 1, pack_key(0, 1, 4, 3)]
    # budget 50: 2g (idx 1, 2 GPCs) and 4g (idx 3, 4 GPCs) feasible -> fewest GPCs
    assert o["key"][1] == pack_key(0, 1, 2, 1)
    assert list(o["checks"][1]) == [5, 2, pack_key(0, 1, 2, 1) + pack_key(0, 1, 4, 3)]
    # budget 5: nothing meets the SLO
    assert o["status"][2] == oracle.PLAN_INFEASIBLE and o["key"][2] == KEY_NONE
    assert list(o["checks"][2]) == [5, 0, 0]
    assert o["slice"][1, 0] == 1 and o["prof"][1, 0] == G2 and o["slice"][1, 1] == -1


def test_n2_k2_thirty_candidates_by_hand():
    # 8000 + 8000 MiB: the whole function (16000) does not fit 1g; each component does.
    # Only two 1g slices are free -> the single feasible candidate is (1g,1g) with the cut.
    # t = (10, 30): mean 20, population std 10, CV = 0.5, CV^2 = 1/4 -> cvq = 256 (Eq. 1).
    f = dict(lat=[[10] * 5, [30] * 5], mem=[8000, 8000], xfer=[5, 0])
    prob = problem([f], [[[G1, G1]]], [(0, 0, 45), (0, 0, 44)], k_max=2)
    o = oracle.plan(prob)
    # idx: k=1 occupies 0..4; k=2 mask 1 (rank 0), seq p1*5+p2 = 0 -> idx 5
    assert o["key"][0] == pack_key(256, 2, 2, 5)
    assert list(o["checks"][0]) == [30, 1, pack_key(256, 2, 2, 5)]
    assert o["e2e_us"][0] == 45 and o["bottleneck_us"][0] == 30 and o["cvq"][0] == 256
    assert o["cut_mask"][0] == 1 and list(o["prof"][0, :2]) == [G1, G1] and list(o["slice"][0, :2]) == [0, 1]
    # e2e = 10 + 30 + 5 = 45 > 44: infeasible (inclusive SLO, R8)
    assert o["status"][1] == oracle.PLAN_INFEASIBLE and list(o["checks"][1]) == [30, 0, 0]


def test_eq1_worked_example_cvq_170():
    # Each component 8000 MiB: any two together exceed 1g, only 1g slices free, so the
    # only feasible plan is three 1g stages with t = (10, 20, 30).
    f = dict(lat=[[10] * 5, [20] * 5, [30] * 5], mem=[8000] * 3, xfer=[1, 1, 0])
    prob = problem([f], [[[G1, G1, G1]]], [(0, 0, 1000)], k_max=3)
    o = oracle.plan(prob)
    t = [Fraction(10), Fraction(20), Fraction(30)]
    cv2 = statistics.pvariance(t) / statistics.mean(t) ** 2
    assert cv2 == Fraction(1, 6)
    assert o["cvq"][0] == int(cv2 * 1024) == 170
    assert o["k"][0] == 3 and o["cut_mask"][0] == 0b11 and o["e2e_us"][0] == 62


def test_fig1_instance_D_two_stage_on_fragmented_slices():
    # GPU-1 = [1.1 free 2g, 1.2 busy (instance A), 1.3 free 1g]; GPU-2 fully
    # busy.  Instance D (3 x 10 GB) fits no single free slice; it becomes a 2g-20GB stage
    # and a 1g-10GB stage on slices 1.1 and 1.3.
    comp = [100, 60, 45, 40, 25]
    f = dict(lat=flat(comp, 3), mem=[10 * GB] * 3, xfer=[500, 500, 0])
    gpu1 = [G2, (G4, 1), G1]
    gpu2 = [(G4, 1), (G2, 1), (G1, 1)]
    prob = problem([f], [[gpu1, gpu2]], [(0, 0, 10**6)])
    o = oracle.plan(prob)
    # stage order from the key: (1g, 2g) with the cut after component 0 (t = 100, 120)
    # ties on CV with (2g, 1g) cut after component 1 and wins on the canonical index
    assert o["status"][0] == oracle.PLAN_OK and o["k"][0] == 2
    assert list(o["prof"][0, :2]) == [G1, G2] and o["cut_mask"][0] == 0b01
    assert list(o["slice"][0, :2]) == [2, 0]
    # a free 3g makes it a 1-stage plan on 3g (30 GB <= 40 GB)
    prob2 = problem([f], [[[G3, G2, G1]]], [(0, 0, 10**6)])
    o2 = oracle.plan(prob2)
    assert o2["k"][0] == 1 and o2["prof"][0, 0] == G3


def test_fig4c_35_plus_10_on_3g_and_1g():
    # P:186 Fig. 4(c): the 45 GB instance becomes 3g.40gb + 1g.10gb
    f = dict(lat=flat([90, 50, 40, 30, 20], 2), mem=[35 * GB, 10 * GB], xfer=[700, 0])
    prob = problem([f], [[[G3, (G4, 1)], [G1, (G7, 1)]]], [(0, 0, 10**6)])
    o = oracle.plan(prob)
    assert o["k"][0] == 2 and list(o["prof"][0, :2]) == [G3, G1] and o["cut_mask"][0] == 1
    assert list(o["slice"][0, :2]) == [0, 2]


def test_fig4d_15_10_10_on_two_2g():
    # P:186 Fig. 4(d): two 2g.20gb slices; 15 | 10+10 is the only split that fits
    f = dict(lat=flat([90, 50, 40, 30, 20], 3), mem=[15 * GB, 10 * GB, 10 * GB], xfer=[700, 700, 0])
    prob = problem([f], [[[G2], [G2]]], [(0, 0, 10**6)])
    o = oracle.plan(prob)
    assert o["k"][0] == 2 and list(o["prof"][0, :2]) == [G2, G2] and o["cut_mask"][0] == 0b01
    assert list(o["slice"][0, :2]) == [0, 1]


def test_table5_medium_variant_needs_pipeline_on_1g():
    # Table 5: medium = baseline >= 2g, FluidFaaS >= 1g
    f = dict(lat=flat([60, 40, 35, 30, 20], 4), mem=[5 * GB, 4 * GB, 5 * GB, 4 * GB], xfer=[300] * 3 + [0])
    loose, tight = 10**6, 4 * 60
    prob = problem([f], [[[G1] * 7]], [(0, 0, loose), (0, 0, tight)])
    o = oracle.plan(prob, k_max=1)
    assert (o["status"] == oracle.PLAN_INFEASIBLE).all()  # monolithic: no slice holds 18 GB
    o = oracle.plan(prob, k_max=4)
    assert o["status"][0] == oracle.PLAN_OK and o["k"][0] >= 2
    assert o["status"][1] == oracle.PLAN_INFEASIBLE  # cuts add transfer beyond 4 x 60 us


@pytest.mark.parametrize("n", range(1, 9))
def test_candidate_count_closed_form(n):
    # 2^(n-1) consecutive partitions; with P profiles per stage and K >= n the
    # count is sum_k C(n-1,k-1) P^k = P (P+1)^(n-1)
    f = dict(lat=flat([5, 4, 3, 2, 1], n), mem=[1] * n)
    prob = problem([f], [[[G1]]], [(0, 0, 0)], k_max=8)
    o = oracle.plan(prob)
    assert o["checks"][0, 0] == 5 * 6 ** (n - 1)
    for K in (1, 2, 3):
        o = oracle.plan(prob, k_max=K)
        assert o["checks"][0, 0] == sum(comb(n - 1, k - 1) * 5 ** k for k in range(1, min(n, K) + 1))
    assert sum(comb(n - 1, k - 1) for k in range(1, n + 1)) == 2 ** (n - 1)


def random_tiny(seed, n_max=4, K=3):
    rng = W.SplitMix64(seed)
    F = 3
    funcs = []
    for _ in range(F):
        n = int(rng.integers(1, n_max, 1)[0])
        lat = rng.integers(1, 60, n * 5).reshape(n, 5).tolist()
        mem = rng.integers(1000, 25000, n).tolist()
        xfer = rng.integers(0, 30, n).tolist()
        funcs.append(dict(lat=lat, mem=mem, xfer=xfer, load=int(rng.integers(0, 50, 1)[0])))
    nodes = []
    for _ in range(2):
        gpus = [[int(p) for p in rng.integers(0, 4, int(rng.integers(1, 3, 1)[0]))] for _ in range(2)]
        nodes.append(gpus)
    reqs = [(int(rng.integers(0, F - 1, 1)[0]), int(rng.integers(0, 1, 1)[0]), int(rng.integers(20, 250, 1)[0]))
            for _ in range(6)]
    return problem(funcs, nodes, reqs, k_max=K)


@pytest.mark.parametrize("seed", range(1000, 1040))
def test_oracle_matches_independent_brute_force(seed):
    prob = random_tiny(seed)
    o = oracle.plan(prob, threads=2)
    for r in range(prob.R):
        best, scored, nfeas, ksum, c = brute_plan(prob, r)
        assert o["key"][r] == best
        assert list(o["checks"][r]) == [scored, nfeas, ksum]
        if c is not None:
            assert o["k"][r] == c["k"] and o["cut_mask"][r] == c["mask"] and o["e2e_us"][r] == c["e2e"]
            assert list(o["prof"][r, :c["k"]]) == c["prof"] and o["bottleneck_us"][r] == max(c["t"])
            assert o["gpcs"][r] == c["gpcs"] and o["cvq"][r] == c["cvq"]


def test_golden_hand_cases():
    """tests/golden/hand_cases.json: hand-derived plans, each with its citation."""
    with open(os.path.join(GOLDEN, "hand_cases.json")) as fh:
        cases = json.load(fh)
    for case in cases:
        nodes = [[[s if isinstance(s, int) else tuple(s) for s in gpu] for gpu in node] for node in case["nodes"]]
        prob = problem(case["funcs"], nodes, [tuple(r) for r in case["requests"]], k_max=case["k_max"])
        o = oracle.plan(prob)
        for r, exp in enumerate(case["expect"]):
            if exp is None:
                assert o["status"][r] == oracle.PLAN_INFEASIBLE, case["cite"]
                continue
            assert o["status"][r] == oracle.PLAN_OK, case["cite"]
            assert o["k"][r] == exp["k"], case["cite"]
            assert o["cut_mask"][r] == exp["mask"], case["cite"]
            assert list(o["prof"][r, :exp["k"]]) == exp["prof"], case["cite"]
            assert o["e2e_us"][r] == exp["e2e"], case["cite"]
            assert o["cvq"][r] == exp["cvq"], case["cite"]
            if "slice" in exp:
                assert list(o["slice"][r, :exp["k"]]) == exp["slice"], case["cite"]
