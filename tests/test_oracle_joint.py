"""Pins of the NEXT-2 oracle (joint commit in adjusted-deadline order):
an independent Python walk on top of tests/helpers.brute_plan, and the properties a
jointly committed batch must have."""
import numpy as np
import pytest

import oracle
from helpers import brute_plan
from test_oracle_pins import random_tiny
from test_oracle_invariants import small_problem


def adjusted(prob, r):
    f = int(prob.req["func"][r])
    a, b = int(prob.comp_off[f]), int(prob.comp_off[f + 1])
    fast = int(prob.lat_us[a:b].astype(np.int64).sum(axis=0).min())
    return int(prob.slo_us[r]) - int(prob.load_us[f]) - fast


def joint_brute(prob):
    p = prob.with_requests(prob.req, prob.slo_us)
    p.slices = prob.slices.copy()
    order = sorted(range(prob.R), key=lambda r: (int(prob.req["node"][r]), adjusted(prob, r), r))
    out = {}
    for r in order:
        best, _, _, _, c = brute_plan(p, r)
        if c is None:
            out[r] = None
            continue
        v = int(prob.req["node"][r])
        taken = []
        for prof in c["prof"]:
            s = next(i for i in range(len(p.slices))
                     if p.slices["node"][i] == v and not p.slices["busy"][i] and p.slices["profile"][i] == prof
                     and i not in taken)
            taken.append(s)
        for s in taken:
            p.slices["busy"][s] = 1
        out[r] = (best, taken)
    return out


@pytest.mark.parametrize("seed", range(1000, 1025))
def test_joint_matches_independent_walk(seed):
    prob = random_tiny(seed)
    o = oracle.plan_joint(prob)
    exp = joint_brute(prob)
    for r in range(prob.R):
        if exp[r] is None:
            assert o["status"][r] == oracle.PLAN_INFEASIBLE
        else:
            assert o["key"][r] == exp[r][0]
            assert list(o["slice"][r, :len(exp[r][1])]) == exp[r][1]


@pytest.mark.parametrize("seed", range(1000, 1006))
def test_joint_batch_is_jointly_feasible_and_never_better(seed):
    prob = small_problem(seed, R=64)
    j = oracle.plan_joint(prob)
    ind = oracle.plan(prob, checks=False)
    used = [s for r in range(prob.R) if j["status"][r] == oracle.PLAN_OK for s in j["slice"][r, :j["k"][r]]]
    assert len(used) == len(set(used))                      # no slice served twice
    assert (prob.slices["busy"][used] == 0).all()            # only initially free slices
    assert (j["key"] >= ind["key"]).all()                    # consuming slices never improves a plan
    # the first request of every node (in adjusted-deadline order) is planned as alone
    first = {}
    for r in sorted(range(prob.R), key=lambda r: (int(prob.req["node"][r]), adjusted(prob, r), r)):
        first.setdefault(int(prob.req["node"][r]), r)
    for r in first.values():
        assert j["key"][r] == ind["key"][r]
