"""Oracle pins for the NEXT-2 throughput floor (R38): every stage of a plan of
function f runs in at most max_stage_us[f] (= 10^6 / lambda_f, an instance sized for the
function's load); 0 = no floor.  Pinned by a hand case, the independent Python brute
force (helpers.brute_plan), and invariants (no floor == floor 0 == an unreachable floor;
monotone in the floor; every plan's bottleneck within its floor)."""
import numpy as np
import pytest

import oracle
from helpers import KEY_NONE, brute_plan, pack_key, problem
from test_oracle_pins import random_tiny
from paper_conf_hpdc_hui0s25_b200 import workload as W


def _hand():
    row = [1000, 600, 450, 400, 300]  # one component, us on 1g, 2g, 3g, 4g, 7g
    fn = dict(lat=[row, row], mem=[1000, 1000], xfer=[100, 0], load=10)
    nodes = [[[0, 0, 2]], [[0, 0]]]   # node 0: 1g, 1g, 3g free; node 1: 1g, 1g free
    reqs = [(0, 0, 10000), (1, 0, 10000), (1, 1, 10000), (2, 1, 10000), (0, 1, 10000)]
    prob = problem([fn, fn, fn], nodes, reqs, k_max=4)
    return prob.__class__(**{**prob.__dict__, "max_stage_us": np.array([0, 1000, 999], np.uint32)})


def test_floor_hand_case():
    """Worked by hand (R38 + R1):
    f0 (no floor), node 0: 1-stage on 1g (2000 us), key (cvq 0, k 1, gpcs 1, idx 0).
    f1 (floor 1000), node 0: 1g (2000) and 2g (1200) exceed the floor, 3g (900) meets it; the
      2-stage (1g, 1g) also meets it but k = 2 ranks after k = 1: 3g, idx 2, gpcs 3.
    f1, node 1 (two 1g): only the 2-stage (1g, 1g), cut after component 0, stages 1000 /
      1000 us (CV 0), idx = offk(2) + 0 = 5, gpcs 2, e2e 2100.
    f2 (floor 999), node 1: the 1000 us stages exceed it: INFEASIBLE.
    f0, node 1: 1-stage on 1g again."""
    prob = _hand()
    o = oracle.plan(prob)
    exp = [pack_key(0, 1, 1, 0), pack_key(0, 1, 3, 2), pack_key(0, 2, 2, 5), KEY_NONE, pack_key(0, 1, 1, 0)]
    assert o["key"].tolist() == exp
    assert o["status"].tolist() == [0, 0, 0, 1, 0]
    assert o["cut_mask"][2] == 1 and o["e2e_us"][2] == 2100 and o["bottleneck_us"][2] == 1000
    assert list(o["prof"][1, :1]) == [2] and list(o["prof"][2, :2]) == [0, 0]


def _tiny_with_floor(seed):
    prob = random_tiny(seed)
    rng = W.SplitMix64(seed ^ 0xF1)
    # floors from "none" through binding to "nothing fits"
    fl = rng.integers(0, 160, prob.F).astype(np.uint32)
    fl[rng.sub(1).uniform(prob.F) < 0.3] = 0
    return prob.__class__(**{**prob.__dict__, "max_stage_us": fl})


@pytest.mark.parametrize("seed", range(2000, 2030))
def test_floor_matches_independent_brute_force(seed):
    prob = _tiny_with_floor(seed)
    o = oracle.plan(prob, threads=2)
    for r in range(prob.R):
        best, scored, nfeas, ksum, c = brute_plan(prob, r)
        assert o["key"][r] == best
        assert list(o["checks"][r]) == [scored, nfeas, ksum]


def test_floor_zero_and_unreachable_equal_no_floor():
    prob = W.config2(R=256)
    base = oracle.plan(prob)
    zero = oracle.plan(prob.__class__(**{**prob.__dict__, "max_stage_us": np.zeros(prob.F, np.uint32)}))
    big = oracle.plan(prob.__class__(**{**prob.__dict__, "max_stage_us": np.full(prob.F, 1 << 30, np.uint32)}))
    for o in (zero, big):
        np.testing.assert_array_equal(o["key"], base["key"])
        np.testing.assert_array_equal(o["checks"], base["checks"])


def test_floor_monotone_and_respected():
    prob = W.with_throughput_floor(W.config2(R=384))
    fl = prob.max_stage_us
    o = oracle.plan(prob)
    ok = o["status"] == oracle.PLAN_OK
    f = prob.req["func"]
    lim = np.where(fl[f] == 0, np.iinfo(np.uint32).max, fl[f])
    assert (o["bottleneck_us"][ok] <= lim[ok]).all()
    # a looser floor never raises the key (it only admits candidates)
    looser = prob.__class__(**{**prob.__dict__, "max_stage_us": np.where(fl == 0, 0, fl * 2).astype(np.uint32)})
    o2 = oracle.plan(looser)
    assert (o2["key"] <= o["key"]).all()
    # the floor binds on this mix: some requests need a pipeline or a larger slice for it
    base = oracle.plan(prob.__class__(**{**prob.__dict__, "max_stage_us": None}))
    assert (o["key"] != base["key"]).mean() > 0.05


def test_floor_victims_and_ranked_respect_it():
    prob = W.with_throughput_floor(W.config2(R=256))
    fl = prob.max_stage_us
    f = prob.req["func"]
    lim = np.where(fl[f] == 0, np.iinfo(np.uint32).max, fl[f])
    r = oracle.plan_ranked(prob)
    ok = r["status"] == oracle.PLAN_OK
    assert (r["bottleneck_us"][ok] <= lim[ok]).all()
    # time-share victims: the monolithic instance on the victim's slice meets the floor
    o = oracle.plan(prob)
    rng = np.random.default_rng(3)
    n_inst = 64
    inst = np.zeros(n_inst, dtype=W.INST_DTYPE)
    inst["func"] = rng.integers(0, prob.F, n_inst)
    inst["slice"] = rng.integers(0, len(prob.slices), n_inst)
    inst["last_used_us"] = rng.integers(0, 1 << 30, n_inst)
    ev = oracle.evict(inst, 1 << 31, 30, 10_000_000)
    vic = oracle.victim(prob, o["status"], inst, ev)
    for q in np.nonzero(vic >= 0)[0]:
        p = int(prob.slices["profile"][inst["slice"][vic[q]]])
        a, b = int(prob.comp_off[f[q]]), int(prob.comp_off[f[q] + 1])
        assert int(prob.lat_us[a:b, p].sum()) <= lim[q]
