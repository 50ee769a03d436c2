"""NEXT-1 DAG stages on the GPU (ffs_dag_stage / ffs_plan_dag, R40-R43)
against the CPU oracle (oracle_plan_dag) through the C ABI: bit-exact keys, plans, bound
slices and per-request checksums.  Needs a B200: marked gpu."""
import numpy as np
import pytest

import oracle
from helpers import problem
from test_oracle_dag import chain_problem, random_dag
from paper_conf_hpdc_hui0s25_b200 import workload as W

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")

FIELDS = ("key", "status", "k", "cut_mask", "split_mask", "e2e_us", "bottleneck_us", "gpcs", "cvq", "n_slots")


@pytest.fixture(scope="module")
def F():
    from paper_conf_hpdc_hui0s25_b200 import ffs
    assert torch.cuda.is_available(), "gpu tests need a CUDA device"
    return ffs


@pytest.fixture(scope="module")
def planner(F):
    return F.Planner(0)


def run_dag(F, planner, prob, dag, k_max=None):
    """Verify mode (checksums) and production mode (cvq pre-test before the division):
    both must give the same plans."""
    k_max = prob.k_max if k_max is None else k_max
    planner.stage(prob)
    planner.stage_dag(dag, k_max)
    req, slo = F.to_device(prob)
    checks = torch.zeros((prob.R, 3), dtype=torch.int64, device="cuda")
    out = planner.plan_dag(req, slo, checks=checks)
    prod = planner.plan_dag(req, slo)
    torch.cuda.synchronize()
    assert torch.equal(out, prod), "production and verify mode differ"
    return F.dag_plans_to_numpy(out), checks.cpu().numpy().view(np.uint64)


def assert_dag_equal(g, o, checks=None, idx=None):
    sel = slice(None) if idx is None else idx
    for f in FIELDS:
        assert np.array_equal(g[f], o[f][sel].astype(g[f].dtype)), f
    assert np.array_equal(g["prof"], o["prof"][sel]) and np.array_equal(g["slice"], o["slice"][sel])
    if checks is not None:
        assert np.array_equal(checks, o["checks"][sel])


def hand5(budget, free):
    """The oracle's hand case (test_oracle_dag.hand) on the P = 5 build: only `free` 1g
    slices exist on the node, profile 0 carries the hand latencies."""
    lat = [[10, 9, 8, 7, 6], [10, 9, 8, 7, 6], [15, 14, 13, 12, 11], [10, 9, 8, 7, 6]]
    prob = problem([dict(lat=lat, mem=[10, 10, 10, 10], xfer=[1, 2, 3, 0])], [[[0] * free]],
                   [(0, 0, budget)], k_max=3)
    return prob, W.dag_table([[[1], [1, 1], [1]]])


def test_dag_hand_case(F, planner):
    for budget, free in ((41, 4), (40, 4), (41, 3), (1000, 4)):
        prob, d = hand5(budget, free)
        g, c = run_dag(F, planner, prob, d)
        o = oracle.plan_dag(prob, d)
        assert_dag_equal(g, o, c)
        if (budget, free) == (41, 4):  # the split stage: 10 | max(10, 15) | 10, 4 slices
            assert g["status"][0] == 0 and g["split_mask"][0] == 0b010 and g["e2e_us"][0] == 41
            assert g["n_slots"][0] == 4 and list(g["slice"][0, :4]) == [0, 1, 2, 3]
        else:
            assert g["status"][0] == (0 if budget == 1000 else 1)


@pytest.mark.parametrize("seed", range(2000, 2012))
def test_dag_random_tiny(F, planner, seed):
    prob, d = random_dag(seed, K=2 if seed % 3 == 0 else 3, nb_max=4 if seed % 3 == 0 else 2)
    g, c = run_dag(F, planner, prob, d)
    assert_dag_equal(g, oracle.plan_dag(prob, d), c)


@pytest.mark.parametrize("cfg", [2, 3])
def test_chain_dag_reproduces_the_chain_search(F, planner, cfg):
    """A DAG of one-component units: the keys and plans of ffs_plan_batch."""
    prob = chain_problem(cfg)
    g, c = run_dag(F, planner, prob, W.chain_dag(prob))
    o = oracle.plan(prob)
    for f in ("key", "status", "k", "cut_mask", "e2e_us", "bottleneck_us", "gpcs", "cvq"):
        assert np.array_equal(g[f], o[f].astype(g[f].dtype)), f
    assert np.array_equal(g["prof"], o["prof"]) and np.array_equal(g["slice"], o["slice"])
    assert np.array_equal(c, o["checks"])
    planner.stage(prob)
    req, slo = F.to_device(prob)
    chain = F.plans_to_numpy(planner.plan_batch(req, slo, prob.k_max))
    assert np.array_equal(chain["key"], g["key"])


def test_dag_config_full_parity(F, planner):
    prob, d = W.dag_config(R=4096)
    g, c = run_dag(F, planner, prob, d)
    o = oracle.plan_dag(prob, d)
    assert (o["split_mask"] > 0).sum() > 50 and (o["status"] == 1).any()
    assert_dag_equal(g, o, c)


def test_dag_config_bench_size_sample(F, planner):
    """The bench workload (R = 65536): sampled requests against the oracle."""
    prob, d = W.dag_config()
    g, c = run_dag(F, planner, prob, d)
    idx = np.arange(0, prob.R, 97)
    o = oracle.plan_dag(prob.subset(idx), d)
    assert_dag_equal(g[idx], o, c[idx])


def test_dag_with_floors_and_three_branches(F, planner):
    prob, d = W.dag_config(R=1024, F=12, branches=(2, 3), p_block=0.5, k_max=2)
    prob = W.with_throughput_floor(prob)
    g, c = run_dag(F, planner, prob, d, k_max=2)
    assert_dag_equal(g, oracle.plan_dag(prob, d, k_max=2), c)


def test_dag_bad_requests_and_errors(F, planner):
    prob, d = W.dag_config(R=64, F=6)
    req = prob.req.copy()
    req["func"][3] = prob.F
    req["node"][5] = prob.n_nodes
    p2 = prob.with_requests(req, prob.slo_us)
    g, _ = run_dag(F, planner, p2, d)
    assert g["status"][3] == 2 and g["status"][5] == 2 and g["key"][3] == F.KEY_NONE
    assert_dag_equal(g, oracle.plan_dag(p2, d))
    planner.stage(prob)
    with pytest.raises(F.FFSError):  # staging new tables drops the DAG
        rq, sl = F.to_device(prob)
        planner.plan_dag(rq, sl)
    bad = W.DagTable(d.unit_off[:-1].copy(), d.unit_nb, d.unit_bend)
    with pytest.raises(F.FFSError):
        planner.stage_dag(bad, 4)
    with pytest.raises(F.FFSError):  # 4 stages x 4 branches > 8 slices
        p3, d3 = W.dag_config(R=8, F=4, branches=(4, 4), p_block=1.0)
        planner.stage(p3)
        planner.stage_dag(d3, 4)


# ---- R48 conditional units (App 3, Table 4) --------------------------------------
def app3_5(budget, mem, branch_y, k_max):
    """test_oracle_dag.app3_like on the P = 5 build: four free 4g.40gb slices; mem MiB per
    component (12000: the whole function does not fit one slice, [D, X|Y] does)."""
    lat = [[10] * 5, [20] * 5] + ([[15] * 5] if branch_y else []) + [[30] * 5]
    xfer = [1, 2] + ([3] if branch_y else []) + [0]
    f = dict(lat=lat, mem=[mem] * len(lat), xfer=xfer)
    prob = problem([f], [[[3] * 4]], [(0, 0, budget)], k_max=k_max)
    return prob, W.dag_table([[[1], W.Cond([1, branch_y]), [1]]])


@pytest.mark.parametrize("budget,mem,branch_y,k_max", [(1000, 1000, 1, 2), (1000, 12000, 1, 2), (62, 12000, 1, 2),
                                                        (1000, 1000, 1, 3), (1000, 12000, 0, 2)])
def test_dag_conditional_units_hand(F, planner, budget, mem, branch_y, k_max):
    prob, d = app3_5(budget, mem, branch_y, k_max)
    g, c = run_dag(F, planner, prob, d)
    o = oracle.plan_dag(prob, d)
    assert_dag_equal(g, o, c)
    assert (g["split_mask"] == 0).all()


@pytest.mark.parametrize("seed", range(2030, 2040))
def test_dag_random_tiny_conditional(F, planner, seed):
    prob, d = random_dag(seed, K=2 if seed % 3 == 0 else 3, nb_max=4 if seed % 3 == 0 else 2, p_cond=0.4)
    assert d.unit_cond is not None
    g, c = run_dag(F, planner, prob, d)
    assert_dag_equal(g, oracle.plan_dag(prob, d), c)


def test_dag_config_with_conditional_units(F, planner):
    """The CD recipe with App-3-like conditional units ("super resolution | pass")."""
    prob, d = W.dag_config(R=4096, p_cond=0.2)
    assert d.unit_cond is not None and d.unit_cond.sum() > 0
    g, c = run_dag(F, planner, prob, d)
    o = oracle.plan_dag(prob, d)
    assert_dag_equal(g, o, c)
    assert (o["status"] == 0).mean() > 0.3
