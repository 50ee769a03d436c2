"""Pins of the NEXT-1 DAG-stage oracle (oracle_plan_dag, R40-R43; "If a
stage involves multiple MIGs running in parallel, we use the maximum execution time among
them", P:430 two-branch DAG): reduction to the chain oracle, a hand-worked case, an
independent Python brute force (Fractions, itertools over compositions and option
tuples) and plan invariants."""
import itertools
import statistics
from fractions import Fraction

import numpy as np
import pytest

import oracle
from helpers import pack_key, problem
from paper_conf_hpdc_hui0s25_b200 import workload as W


def dag_of(shapes):
    return W.dag_table(shapes)


# ---- the chain is the DAG of one-component units ----------------------------------
def chain_problem(cfg):
    if cfg == 2:
        return W.config2(R=1024)
    # C3-shaped (8 nodes, 20 functions) with chains of at most 16 components (= units)
    rng = W.SplitMix64(0xDA6 + cfg)
    return W._problem("C3-16", rng, rng.sub(9).integers(3, 16, 20), W.NODE_BLOCK, 256)


@pytest.mark.parametrize("cfg", [2, 3])
def test_chain_dag_equals_chain_oracle(cfg):
    prob = chain_problem(cfg)
    a = oracle.plan(prob)
    b = oracle.plan_dag(prob, W.chain_dag(prob))
    for f in ("key", "status", "k", "cut_mask", "e2e_us", "bottleneck_us", "gpcs", "cvq"):
        assert np.array_equal(a[f], b[f]), f
    assert np.array_equal(a["checks"], b["checks"])
    assert np.array_equal(a["prof"], b["prof"][:, :8]) and np.array_equal(a["slice"], b["slice"][:, :8])
    assert (b["split_mask"] == 0).all()
    assert np.array_equal(b["n_slots"], np.where(a["status"] == 0, a["k"], 0))


# ---- hand-worked case ------------------------------------------------------------
def hand(budget, free=4):
    """Units [A], [B | C], [D] on one profile (1 GPC, 100 MiB): lat A=10, B=10, C=15,
    D=10; xfer A=1, B=2, C=3.  Candidates (R43 order): idx 0 k=1 (45); idx 1 k=2 cut
    after A (10 | 35, e2e 46); idx 2 cut after the block (35 | 10, e2e 45 + 2 + 3 = 50);
    idx 3 k=3 single (10 | 25 | 10, e2e 51); idx 4 k=3 split (10 | max(10, 15) | 10,
    e2e 35 + 1 + 5 = 41, 4 slices, CV^2 = (3*425 - 35^2)/35^2 = 50/1225 -> cvq 41)."""
    prob = problem([dict(lat=[[10], [10], [15], [10]], mem=[10, 10, 10, 10], xfer=[1, 2, 3, 0])],
                   [[[0] * free]], [(0, 0, budget)], k_max=3, gpcs=[1], cap=[100])
    return prob, dag_of([[[1], [1, 1], [1]]])


def test_hand_split_stage_takes_the_max_and_pays_both_transfers():
    prob, d = hand(41)
    o = oracle.plan_dag(prob, d)
    assert o["status"][0] == 0
    assert o["key"][0] == pack_key(41, 3, 4, 4)
    assert o["split_mask"][0] == 0b010 and o["cut_mask"][0] == 0b11 and o["n_slots"][0] == 4
    assert o["e2e_us"][0] == 41 and o["bottleneck_us"][0] == 15 and o["gpcs"][0] == 4
    assert list(o["slice"][0, :4]) == [0, 1, 2, 3]
    assert list(o["checks"][0]) == [5, 1, o["key"][0]]


def test_hand_budget_and_free_slices():
    # 40 < 41: R42 (both branch outputs move) makes it infeasible; a last-branch-only
    # reading would give e2e 38
    assert oracle.plan_dag(*hand(40))["status"][0] == 1
    # the split stage needs 4 slices
    assert oracle.plan_dag(*hand(41, free=3))["status"][0] == 1
    # a generous budget: the 1-stage plan (CV 0) wins
    o = oracle.plan_dag(*hand(1000))
    assert o["key"][0] == pack_key(0, 1, 1, 0) and o["e2e_us"][0] == 45


# ---- independent brute force ----------------------------------------------------
def brute_dag(prob, dag, r):
    P, K = prob.P, prob.k_max
    f, v, B = int(prob.req["func"][r]), int(prob.req["node"][r]), int(prob.slo_us[r])
    base = int(prob.comp_off[f])
    units = dag.units(f)
    m = len(units)
    cu = [False] * m if dag.unit_cond is None else \
        [bool(dag.unit_cond[int(dag.unit_off[f]) + u]) for u in range(m)]  # R48 conditional units
    lat = lambda c, p: int(prob.lat_us[base + c, p])  # noqa: E731
    mem = lambda c: int(prob.mem_mib[base + c])  # noqa: E731
    xf = lambda c: int(prob.xfer_us[base + c])  # noqa: E731
    sl = prob.slices
    free = [int(((sl["node"] == v) & (sl["busy"] == 0) & (sl["profile"] == p)).sum()) for p in range(P)]
    fl = getattr(prob, "max_stage_us", None)
    floor = 0 if fl is None else int(fl[f])
    best, idx, nfeas, ksum = None, 0, 0, 0
    for k in range(1, min(K, m) + 1):
        # compositions of the unit list into k runs, cut masks ascending
        cuts_list = sorted(itertools.combinations(range(m - 1), k - 1), key=lambda cs: sum(1 << c for c in cs))
        for cuts in cuts_list:
            bounds = [0] + [c + 1 for c in cuts] + [m]
            stages = [units[bounds[i]:bounds[i + 1]] for i in range(k)]
            conds = [cu[bounds[i]:bounds[i + 1]] for i in range(k)]
            opts = []
            for st, cs in zip(stages, conds):
                o = [("one", (p,)) for p in range(P)]
                if len(st) == 1 and len(st[0]) >= 2 and not cs[0]:
                    o += [("split", ps) for ps in itertools.product(range(P), repeat=len(st[0]))]
                opts.append(o)

            def cut_cost(u):  # R42; R48: the output of the alternative that ran (worst case)
                xs = [xf(e - 1) if e > a else (xf(units[u][0][0] - 1) if units[u][0][0] > 0 else 0)
                      for (a, e) in units[u]]
                return max(xs) if cu[u] else sum(xs)
            xfer = sum(cut_cost(c) for c in cuts)
            for choice in itertools.product(*opts):
                t, used, ok = [], [0] * P, True
                for st, cs, (kind, ps) in zip(stages, conds, choice):
                    comps = [c for u in st for (a, e) in u for c in range(a, e)]
                    if kind == "one":
                        p = ps[0]
                        # a unit's time: its components in sequence, or its slowest alternative
                        t.append(sum(max(sum(lat(c, p) for c in range(a, e)) for (a, e) in u) if cnd
                                     else sum(lat(c, p) for (a, e) in u for c in range(a, e))
                                     for u, cnd in zip(st, cs)))
                        ok &= sum(mem(c) for c in comps) <= int(prob.cap_mib[p])
                        used[p] += 1
                    else:
                        bt = []
                        for (a, e), p in zip(st[0], ps):
                            bt.append(sum(lat(c, p) for c in range(a, e)))
                            ok &= sum(mem(c) for c in range(a, e)) <= int(prob.cap_mib[p])
                            used[p] += 1
                        t.append(max(bt))
                gp = sum(int(prob.gpcs[p]) for (_, ps) in choice for p in ps)
                ok &= all(u <= fr for u, fr in zip(used, free))
                ok &= floor == 0 or max(t) <= floor
                ok &= sum(t) + xfer <= B
                if ok:
                    tf = [Fraction(x) for x in t]
                    cvq = int(statistics.pvariance(tf) / statistics.mean(tf) ** 2 * 1024)
                    key = pack_key(cvq, k, gp, idx)
                    nfeas += 1
                    ksum = (ksum + key) % (1 << 64)
                    if best is None or key < best[0]:
                        split = sum(1 << s for s, (kind, _) in enumerate(choice) if kind == "split")
                        best = (key, sum(1 << c for c in cuts), split, sum(t) + xfer, max(t),
                                [p for (_, ps) in choice for p in ps])
                idx += 1
    return best, idx, nfeas, ksum


def random_dag(seed, K=3, nb_max=3, p_cond=0.0):
    rng = W.SplitMix64(seed)
    c_rng = rng.sub(5)
    shapes, funcs = [], []
    for _ in range(3):
        m = int(rng.integers(1, 4, 1)[0])
        units = []
        for _ in range(m):
            if float(rng.uniform(1)[0]) < 0.5:
                units.append([int(x) for x in rng.integers(1, 2, int(rng.integers(2, nb_max, 1)[0]))])
            else:
                units.append([1])
            if p_cond and float(c_rng.uniform(1)[0]) < p_cond:  # R48: alternatives, maybe a "pass"
                units[-1] = W.Cond([int(c_rng.integers(1, 2, 1)[0]), int(c_rng.integers(0, 1, 1)[0])])
        n = sum(sum(u) for u in units)
        shapes.append(units)
        funcs.append(dict(lat=rng.integers(1, 60, n * 5).reshape(n, 5).tolist(),
                          mem=rng.integers(1000, 25000, n).tolist(), xfer=rng.integers(0, 30, n).tolist()))
    nodes = [[[int(p) for p in rng.integers(0, 4, int(rng.integers(1, 4, 1)[0]))] for _ in range(2)]
             for _ in range(2)]
    reqs = [(int(rng.integers(0, 2, 1)[0]), int(rng.integers(0, 1, 1)[0]), int(rng.integers(20, 300, 1)[0]))
            for _ in range(6)]
    return problem(funcs, nodes, reqs, k_max=K), dag_of(shapes)


@pytest.mark.parametrize("seed", range(2000, 2040))
def test_dag_oracle_matches_independent_brute_force(seed):
    prob, d = random_dag(seed, K=2 if seed % 3 == 0 else 3, nb_max=4 if seed % 3 == 0 else 2,
                         p_cond=0.4 if seed >= 2030 else 0.0)
    if seed >= 2030:
        assert d.unit_cond is not None
    o = oracle.plan_dag(prob, d, threads=2)
    for r in range(prob.R):
        best, scored, nfeas, ksum = brute_dag(prob, d, r)
        assert list(o["checks"][r]) == [scored, nfeas, ksum]
        if best is None:
            assert o["status"][r] in (1, 2) and o["key"][r] == oracle.KEY_NONE
            continue
        key, cut, split, e2e, bott, prof = best
        assert o["key"][r] == key and o["cut_mask"][r] == cut and o["split_mask"][r] == split
        assert o["e2e_us"][r] == e2e and o["bottleneck_us"][r] == bott
        assert list(o["prof"][r, :len(prof)]) == prof and o["n_slots"][r] == len(prof)


# ---- invariants -------------------------------------------------------------------
def test_dag_freeing_a_slice_never_worsens_and_plans_are_valid():
    prob, d = W.dag_config(R=256, F=8)
    o = oracle.plan_dag(prob, d)
    assert (o["status"] == 0).any() and (o["split_mask"] > 0).any()
    sl = prob.slices
    for r in np.flatnonzero(o["status"] == 0)[:60]:
        n = int(o["n_slots"][r])
        s = o["slice"][r, :n]
        assert len(set(s.tolist())) == n and (s >= 0).all()
        assert (sl["busy"][s] == 0).all() and (sl["node"][s] == prob.req["node"][r]).all()
        assert (sl["profile"][s] == o["prof"][r, :n]).all()
        assert o["e2e_us"][r] <= prob.slo_us[r]
    busy = prob.slices["busy"].copy()
    idx = np.flatnonzero(busy == 1)[::3]
    freed = prob.with_requests(prob.req, prob.slo_us)
    freed.slices = prob.slices.copy()
    freed.slices["busy"][idx] = 0
    o2 = oracle.plan_dag(freed, d)
    assert (o2["key"] <= o["key"]).all()


def test_dag_table_validation():
    prob, d = hand(41)
    bad = W.DagTable(d.unit_off.copy(), d.unit_nb.copy(), d.unit_bend.copy())
    bad.unit_bend[1, 1] = 2  # branch ends must increase
    with pytest.raises(ValueError):
        oracle.plan_dag(prob, bad)
    bad = W.DagTable(d.unit_off.copy(), d.unit_nb.copy(), d.unit_bend.copy())
    bad.unit_bend[2, 0] = 3  # units must cover the chain
    with pytest.raises(ValueError):
        oracle.plan_dag(prob, bad)
    # k_max * slices per stage * max gpcs must stay below 64 (6-bit key field)
    p2, d2 = W.dag_config(R=8, F=4, branches=(4, 4), p_block=1.0)
    with pytest.raises(ValueError):
        oracle.plan_dag(p2, d2, k_max=4)


# ---- R48 conditional units (App 3, Table 4) --------------------------------------
def app3_like(budget, cap=100, k_max=2, branch_y=1):
    """Units [D], Cond[X | Y] (Y empty when branch_y = 0: "pass"), [E] on one profile:
    lat D=10, X=20, Y=15, E=30; mem 10 each; xfer D=1, X=2, Y=3."""
    lat = [[10], [20]] + ([[15]] if branch_y else []) + [[30]]
    xfer = [1, 2] + ([3] if branch_y else []) + [0]
    f = dict(lat=lat, mem=[10] * len(lat), xfer=xfer)
    prob = problem([f], [[[0] * 4]], [(0, 0, budget)], k_max=k_max, gpcs=[1], cap=[cap])
    return prob, W.dag_table([[[1], W.Cond([1, branch_y]), [1]]])


def test_conditional_unit_takes_the_slowest_alternative():
    # one slice: 10 + max(20, 15) + 30 = 60 (a fork/join block on one slice would be 75)
    o = oracle.plan_dag(*app3_like(1000))
    assert o["status"][0] == 0 and o["key"][0] == pack_key(0, 1, 1, 0) and o["e2e_us"][0] == 60
    # every alternative is hosted: memory 40 > cap 35 makes the one-stage plan infeasible
    o = oracle.plan_dag(*app3_like(1000, cap=35))
    # cut after the conditional unit: [D, X|Y] = 30 | [E] = 30 (CV 0), the cut moves the
    # output of whichever alternative ran: max(2, 3) = 3 -> e2e 63
    assert o["key"][0] == pack_key(0, 2, 2, 2) and o["e2e_us"][0] == 63 and o["cut_mask"][0] == 0b10
    # budget 62: that plan misses the SLO; the cut after D (10 | 50, cvq 455, e2e 61) wins
    o = oracle.plan_dag(*app3_like(62, cap=35))
    assert o["key"][0] == pack_key(455, 2, 2, 1) and o["e2e_us"][0] == 61


def test_conditional_unit_is_never_split_and_pass_moves_the_previous_output():
    # k_max 3: the mask with the conditional unit alone in a stage has 1 option (P = 1),
    # not P + P^2 = 2 as a fork/join block would: 1 + 2 + 1 candidates
    o = oracle.plan_dag(*app3_like(1000, k_max=3))
    assert o["checks"][0][0] == 4 and (o["split_mask"] == 0).all()
    # "pass" (empty alternative): one slice = 10 + max(20, 0) + 30; a cut after the unit
    # moves max(X's output 2, D's output passed through 1) = 2
    o = oracle.plan_dag(*app3_like(1000, cap=25, branch_y=0))
    assert o["e2e_us"][0] == 60 + 2 and o["cut_mask"][0] == 0b10
