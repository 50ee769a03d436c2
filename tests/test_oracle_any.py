"""Oracle pins for NEXT-2 any-invoker (cross-node) planning (R39): the plan of a
request is the argmin over nodes of its per-node plan; ties prefer the home node, then the
lowest node id.  Pinned by a hand case and by properties against per-node oracle plans."""
import numpy as np

import oracle
from helpers import KEY_NONE, pack_key, problem
from test_oracle_pins import random_tiny
from paper_conf_hpdc_hui0s25_b200 import workload as W


def test_any_hand_case():
    """One 2-component function (each component 1000 us on 1g .. 300 us on 7g, 1000 MiB).
    node 0: nothing free; node 1: one 1g free; node 2: one 3g free; node 3: one 1g free.
    r0 home 0, B 3000: node 0 has no plan; 1-stage on 1g (key (0,1,1,0)) on nodes 1 and 3,
       3g (key (0,1,3,2)) on node 2 -> the 1g plan, lowest node id among the tie: node 1.
    r1 home 3, same budget: the same key on nodes 1 and 3 -> the home node 3.
    r2 home 1, B 1000: 1g (2000 us) misses the budget, 3g (900 us) meets it -> node 2.
    r3 home 0, B 800: nothing meets it anywhere -> INFEASIBLE, node -1."""
    row = [1000, 600, 450, 400, 300]
    fn = dict(lat=[row, row], mem=[1000, 1000], xfer=[100, 0], load=10)
    nodes = [[[(0, 1)]], [[0]], [[2]], [[0]]]
    reqs = [(0, 0, 3000), (0, 3, 3000), (0, 1, 1000), (0, 0, 800)]
    prob = problem([fn], nodes, reqs, k_max=2)
    o, node = oracle.plan_any(prob)
    assert o["key"].tolist() == [pack_key(0, 1, 1, 0), pack_key(0, 1, 1, 0), pack_key(0, 1, 3, 2), KEY_NONE]
    assert node.tolist() == [1, 3, 2, -1]
    sl = prob.slices
    assert sl["node"][o["slice"][0, 0]] == 1 and sl["node"][o["slice"][1, 0]] == 3
    assert sl["node"][o["slice"][2, 0]] == 2


def _check_properties(prob):
    o, node = oracle.plan_any(prob)
    per = []
    for v in range(prob.n_nodes):
        req = prob.req.copy()
        req["node"] = v
        per.append(oracle.plan(prob.with_requests(req, prob.slo_us), checks=False)["key"])
    per = np.stack(per)                      # [nodes, R]
    np.testing.assert_array_equal(o["key"], per.min(0))
    home = oracle.plan(prob, checks=False)
    assert (o["key"] <= home["key"]).all()   # never worse than the home invoker
    ok = o["status"] == oracle.PLAN_OK
    assert ((node >= 0) == ok).all()
    for r in np.nonzero(ok)[0]:
        tied = np.nonzero(per[:, r] == o["key"][r])[0]
        h = int(prob.req["node"][r])
        assert node[r] == (h if h in tied else tied.min())
        s = o["slice"][r, :o["k"][r]]
        assert (prob.slices["node"][s] == node[r]).all() and len(set(s.tolist())) == len(s)
        assert not prob.slices["busy"][s].any()


def test_any_properties_tiny():
    for seed in range(1000, 1012):
        _check_properties(random_tiny(seed))


def test_any_properties_c3_sample():
    prob = W.config3(R=1024)
    _check_properties(prob.subset(np.arange(0, prob.R, 16)))
