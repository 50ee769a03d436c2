"""Pins of the NEXT-2 routing oracle: a hand case and an independent Python walk."""
import numpy as np
import pytest

import oracle
from helpers import problem
from test_oracle_pins import random_tiny
from paper_conf_hpdc_hui0s25_b200 import workload as W

HOT, TS, WARM, COLD = oracle.ST_EXCL_HOT, oracle.ST_TIME_SHARING, oracle.ST_WARM, oracle.ST_COLD


def route_brute(prob, func, state, lat, cap):
    out = np.full(prob.R, -1, np.int32)
    for f in range(prob.F):
        a, b = int(prob.comp_off[f]), int(prob.comp_off[f + 1])
        fast = int(prob.lat_us[a:b].astype(np.int64).sum(axis=0).min())
        reqs = sorted((int(prob.slo_us[r]) - int(prob.load_us[f]) - fast, r) for r in range(prob.R)
                      if prob.req["func"][r] == f)
        hot = sorted((int(lat[i]), i) for i in range(len(func)) if func[i] == f and state[i] == HOT)
        ts = next((i for i in range(len(func)) if func[i] == f and state[i] in (TS, WARM)), -1)
        slots = [i for _, i in hot for _ in range(int(cap[i]))]
        for j, (_, r) in enumerate(reqs):
            out[r] = slots[j] if j < len(slots) else ts
    return out


def test_route_hand_case():
    # one function, 5 requests with budgets 500, 100, 300, 400, 200 (load 0, fastest 10):
    # urgency order = r1, r4, r2, r3, r0.  Hot instances: #1 (lat 30, cap 2), #0 (lat 20,
    # cap 1); #2 time-sharing, #3 cold.  Order: #0 takes r1; #1 takes r4, r2; rest -> #2.
    f = dict(lat=[[10, 10, 10, 10, 10]], mem=[1000])
    prob = problem([f], [[[0]]], [(0, 0, 500), (0, 0, 100), (0, 0, 300), (0, 0, 400), (0, 0, 200)])
    route = oracle.route(prob, [0, 0, 0, 0], [HOT, HOT, TS, COLD], [20, 30, 0, 0], [1, 2, 0, 0])
    assert route.tolist() == [2, 0, 1, 2, 1]
    # without a time-sharing instance the overflow has nowhere to go
    route = oracle.route(prob, [0, 0, 0], [HOT, HOT, COLD], [20, 30, 0], [1, 2, 0])
    assert route.tolist() == [-1, 0, 1, -1, 1]


@pytest.mark.parametrize("seed", range(1000, 1012))
def test_route_matches_independent_walk(seed):
    prob = random_tiny(seed)
    rng = W.SplitMix64(seed + 5)
    n = 9
    func = rng.integers(0, prob.F - 1, n).astype(np.uint32)
    state = rng.integers(0, 3, n).astype(np.uint8)
    lat = rng.integers(1, 5, n).astype(np.uint32)  # ties on latency -> index order
    cap = rng.integers(0, 3, n).astype(np.uint32)
    np.testing.assert_array_equal(oracle.route(prob, func, state, lat, cap), route_brute(prob, func, state, lat, cap))
