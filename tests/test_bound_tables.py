"""The bounded mode's exact SLO lower bound ("live-mask compaction"),
restated in plain Python and checked against brute force -- CPU only.

For a request (function f, node v, budget B) and a cut mask with stage boundaries
0 = b0 < b1 < ... < bk = n, every candidate's end-to-end latency (P:339 stage times summed
+ transfer cost per cut, R5/R7) is >= LB = sum_s W(b_s, b_{s+1}) + sum_cuts X(b), where
W(i, j) = the fastest stage time of [i, j) over the profiles the node has at least one free
slice of, that hold the stage's memory (R6) and meet the floor (R38).  The kernels use the
same quantities through per-(function, availability) tables H0/Mt/T3 and the best-case
row / block bounds R2/R3; these tests pin that a mask with LB > B holds no feasible
candidate (so dropping it is exact) and that R2 / R3 never exceed the LB of any mask they
cover."""
import itertools

import pytest

from paper_conf_hpdc_hui0s25_b200 import workload as W
from helpers import problem

INF = float("inf")


def tables(prob, f, avail):
    a, b = int(prob.comp_off[f]), int(prob.comp_off[f + 1])
    n, P = b - a, prob.P
    lat = prob.lat_us[a:b].astype(int).tolist()
    mem = prob.mem_mib[a:b].astype(int).tolist()
    xf = prob.xfer_us[a:b].astype(int).tolist()
    fl = getattr(prob, "max_stage_us", None)
    floor = INF if fl is None or int(fl[f]) == 0 else int(fl[f])

    def Wf(i, j):
        best = INF
        for p in range(P):
            if not avail[p] or sum(mem[i:j]) > int(prob.cap_mib[p]):
                continue
            t = sum(lat[c][p] for c in range(i, j))
            if t <= floor:
                best = min(best, t)
        return best

    X = {j: xf[j - 1] for j in range(1, n)}
    H0 = {j: Wf(0, j) + X[j] for j in range(1, n)}
    T3 = {i: Wf(i, n) for i in range(1, n)}
    Mt = {(j, i): Wf(i, j) + X[j] for i in range(1, n) for j in range(i + 1, n)}
    R2 = {j: min([H0[i] + Mt[(j, i)] for i in range(1, j)], default=INF) for j in range(1, n)}
    R3 = {j: min([R2[i] + Mt[(j, i)] for i in range(2, j)], default=INF) for j in range(1, n)}
    return n, lat, mem, xf, floor, H0, T3, Mt, R2, R3


def lb(bounds, H0, T3, Mt):
    k = len(bounds) - 1
    if k == 2:
        return H0[bounds[1]] + T3[bounds[1]]
    v = H0[bounds[1]] + T3[bounds[k - 1]]
    for s in range(1, k - 1):
        v += Mt[(bounds[s + 1], bounds[s])]
    return v


def random_chain_problem(seed):
    rng = W.SplitMix64(seed)
    funcs = []
    for _ in range(2):
        n = int(rng.integers(4, 7, 1)[0])
        funcs.append(dict(lat=rng.integers(1, 80, n * 5).reshape(n, 5).tolist(),
                          mem=rng.integers(1000, 30000, n).tolist(),
                          xfer=rng.integers(0, 40, n).tolist(), load=0))
    nodes = [[[int(p) for p in rng.integers(0, 4, 3)], [(int(rng.integers(0, 4, 1)[0]), 1)]] for _ in range(2)]
    reqs = [(f, v, 10 ** 6) for f in range(2) for v in range(2)]
    return problem(funcs, nodes, reqs, k_max=4)


@pytest.mark.parametrize("seed", range(12))
def test_lower_bound_is_sound(seed):
    prob = random_chain_problem(seed)
    sl = prob.slices
    for r in range(prob.R):
        f, v = int(prob.req["func"][r]), int(prob.req["node"][r])
        free = [int(((sl["node"] == v) & (sl["busy"] == 0) & (sl["profile"] == p)).sum()) for p in range(prob.P)]
        avail = [x > 0 for x in free]
        n, lat, mem, xf, floor, H0, T3, Mt, R2, R3 = tables(prob, f, avail)
        for k in (2, 3, 4):
            for cuts in itertools.combinations(range(n - 1), k - 1):
                bounds = [0] + [j + 1 for j in cuts] + [n]
                L = lb(bounds, H0, T3, Mt)
                # every candidate that could be feasible under some budget has e2e >= LB
                best = INF
                for seq in itertools.product(range(prob.P), repeat=k):
                    st = [range(bounds[i], bounds[i + 1]) for i in range(k)]
                    t = [sum(lat[c][p] for c in s) for s, p in zip(st, seq)]
                    ok = all(sum(mem[c] for c in s) <= int(prob.cap_mib[p]) for s, p in zip(st, seq))
                    ok = ok and all(seq.count(p) <= free[p] for p in range(prob.P)) and max(t) <= floor
                    if ok:
                        best = min(best, sum(t) + sum(xf[j] for j in cuts))
                assert L <= best, (r, k, cuts, L, best)
                # the row / block bounds the compaction kernel tests first never exceed LB
                if k >= 3:
                    assert R2[bounds[2]] + (T3[bounds[2]] if k == 3 else
                                            Mt[(bounds[3], bounds[2])] + T3[bounds[3]]) <= L
                if k == 4:
                    assert R3[bounds[3]] + T3[bounds[3]] <= L


def test_lower_bound_is_tight_without_multiplicity():
    """With one free slice of every profile, a mask's LB is attained by the candidate that
    puts every stage on its fastest admissible profile when those profiles are distinct."""
    f = dict(lat=[[40, 30, 20, 15, 10], [50, 40, 30, 20, 10], [45, 35, 25, 15, 5]], mem=[100, 100, 100],
             xfer=[3, 4, 0], load=0)
    prob = problem([f], [[[0, 1, 2, 3, 4]]], [(0, 0, 1000)], k_max=3)
    n, lat, mem, xf, floor, H0, T3, Mt, R2, R3 = tables(prob, 0, [True] * 5)
    # mask with cuts after components 0 and 1: stages {0}, {1}, {2} -> 10 + 3 + 10 + 4 + 5
    assert lb([0, 1, 2, 3], H0, T3, Mt) == 10 + 3 + 10 + 4 + 5
