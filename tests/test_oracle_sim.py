"""Pins of the NEXT-4 time-sharing simulator oracle (Fig. 8; R31-R36):
hand-worked scenarios and an independent Python re-implementation on small traces."""
import numpy as np
import pytest

import oracle
from helpers import problem
from paper_conf_hpdc_hui0s25_b200 import workload as W

HOT, TS, WARM, COLD = oracle.ST_EXCL_HOT, oracle.ST_TIME_SHARING, oracle.ST_WARM, oracle.ST_COLD
G1, G2, G3, G4, G7 = range(5)


def make_trace(prob, T, events, window_ticks=4, tick_us=100, t0=1000):
    """events: list of (tick, node, func, budget)."""
    N = prob.n_nodes
    ev = sorted(events, key=lambda e: (e[1], e[0]))  # CSR by (node, tick), stable in input order
    off = np.zeros(N * T + 1, np.uint32)
    for t, v, f, b in ev:
        off[v * T + t + 1] += 1
    off = np.cumsum(off).astype(np.uint32)
    return W.SimTrace(problem=prob, req_off=off, req_func=np.array([e[2] for e in ev], np.uint32),
                      req_budget=np.array([e[3] for e in ev], np.uint32), T=T, tick_us=tick_us,
                      window_ticks=window_ticks, t0_us=t0)


def two_funcs(nodes):
    fa = dict(lat=[[50, 40, 30, 20, 10]], mem=[5000], load=100)
    fb = dict(lat=[[60, 50, 40, 30, 20]], mem=[5000], load=200)
    return problem([fa, fb], nodes, [(0, 0, 0)])


def test_eviction_reload_and_same_tick_protection():
    prob = two_funcs([[[G1]]])  # one node, one 1g slice
    # t0: A placed (reload 100 + exec 50 = 150 <= 200: hit); t1: B evicts A (A idle this
    # tick): 200 + 60 = 260 > 250 miss; t1: A again -> B was used in this tick -> unserved;
    # t2: A evicts B: 150 <= 150 hit
    tr = make_trace(prob, 3, [(0, 0, 0, 200), (1, 0, 1, 250), (1, 0, 0, 500), (2, 0, 0, 150)], window_ticks=100)
    ctr, fs, st, last, busy = oracle.sim(tr)
    # requests, served, hits, unserved, reloads, evictions, terminations, slice-ticks
    assert ctr[0].tolist() == [4, 3, 2, 1, 3, 2, 0, 3]
    assert fs[0].tolist() == [0, -1] and st[0].tolist() == [TS, WARM]
    assert last[0].tolist() == [1200, 1100] and busy[0].tolist() == [100, 60]


def test_hot_instances_are_exempt_and_cold_terminates():
    prob = two_funcs([[[G1]]])
    # window = 2 ticks of 100 us = 200 us; A busy 50 + 50 = 100 us >= 30% -> hot at t1 end;
    # in window 2 (t2, t3) B cannot evict A; A idle from t2: busy 0 -> time sharing again at
    # t3 end; t4: B evicts A.  cold_after = 350 us: B (last use t4 = 1400) is terminated at
    # the end of t8 (1800 - 1400 >= 350 -> first at t8: now 1800).
    ev = [(0, 0, 0, 10**6), (1, 0, 0, 10**6), (2, 0, 1, 10**6), (3, 0, 1, 10**6), (4, 0, 1, 10**6)]
    tr = make_trace(prob, 9, ev, window_ticks=2)
    ctr, fs, st, last, busy = oracle.sim(tr, cold_after_us=350)
    assert ctr[0].tolist()[:6] == [5, 3, 3, 2, 2, 1]
    # A: last use t1 = 1100 -> cold at the end of t5 (1500 - 1100 >= 350); B cold at t8
    assert ctr[0][6] == 2 and st[0].tolist() == [COLD, COLD]


def test_free_slice_preference_smallest_capacity():
    prob = two_funcs([[[G4, G2, G1]]])
    tr = make_trace(prob, 1, [(0, 0, 0, 10**6)])
    ctr, fs, st, last, busy = oracle.sim(tr)
    assert fs[0, 0] == 2  # the 1g slice (smallest capacity that holds 5000 MiB)


def sim_python(tr, thr=30, cold_after=600_000_000):
    """Independent re-implementation (plain Python)."""
    prob = tr.problem
    N, F, T = prob.n_nodes, prob.F, tr.T
    lat, mem, load = prob.lat_us.astype(int), prob.mem_mib.astype(int), prob.load_us.astype(int)
    off = prob.comp_off.astype(int)
    exe = [[int(lat[off[f]:off[f + 1], p].sum()) for p in range(prob.P)] for f in range(F)]
    mt = [int(mem[off[f]:off[f + 1]].sum()) for f in range(F)]
    sl = prob.slices
    cap, g = prob.cap_mib.astype(int), prob.gpcs.astype(int)
    out = []
    for v in range(N):
        slices = [s for s in range(len(sl)) if sl["node"][s] == v]
        res = {s: None for s in slices}
        inst = {}  # f -> dict(slice, last, busy, hot)
        c = [0] * 8
        for t in range(T):
            now = tr.t0_us + t * tr.tick_us
            for j in range(int(tr.req_off[v * T + t]), int(tr.req_off[v * T + t + 1])):
                f, B = int(tr.req_func[j]), int(tr.req_budget[j])
                c[0] += 1
                I = inst.setdefault(f, dict(slice=None, last=now, busy=0, hot=False))
                if I["slice"] is not None:
                    ex = exe[f][int(sl["profile"][I["slice"]])]
                    latency = ex
                else:
                    free = [s for s in slices if not sl["busy"][s] and res[s] is None
                            and mt[f] <= cap[sl["profile"][s]]]
                    tgt = min(free, key=lambda s: (cap[sl["profile"][s]], g[sl["profile"][s]], s)) if free else None
                    if tgt is None:
                        vic = [s for s in slices if res[s] is not None and res[s] != f
                               and not inst[res[s]]["hot"] and inst[res[s]]["last"] < now
                               and mt[f] <= cap[sl["profile"][s]]]
                        if vic:
                            tgt = min(vic, key=lambda s: (inst[res[s]]["last"], s))
                            inst[res[tgt]]["slice"] = None
                            res[tgt] = None
                            c[5] += 1
                    if tgt is None:
                        c[3] += 1
                        continue
                    res[tgt] = f
                    I["slice"] = tgt
                    c[4] += 1
                    ex = exe[f][int(sl["profile"][tgt])]
                    latency = load[f] + ex
                c[1] += 1
                c[2] += latency <= B
                I["busy"] += ex
                I["last"] = now
            c[7] += sum(1 for s in slices if res[s] is not None)
            if (t + 1) % tr.window_ticks == 0:
                for I in inst.values():
                    I["hot"] = I["busy"] * 100 >= thr * tr.window_ticks * tr.tick_us
                    I["busy"] = 0
            for f in list(inst):
                if now - inst[f]["last"] >= cold_after:
                    if inst[f]["slice"] is not None:
                        res[inst[f]["slice"]] = None
                    del inst[f]
                    c[6] += 1
        out.append(c)
    return np.array(out, np.uint64)


@pytest.mark.parametrize("seed", range(3))
def test_sim_matches_independent_python(seed):
    tr = W.sim_trace(seed=100 + seed, T=300, n_funcs=12, nodes=[W.PART_P1, W.PART_HYBRID], rate_scale=8.0)
    ctr, *_ = oracle.sim(tr, cold_after_us=5_000_000)
    np.testing.assert_array_equal(ctr, sim_python(tr, cold_after=5_000_000))
    assert ctr[:, 5].sum() > 0 and ctr[:, 6].sum() > 0  # evictions and terminations happen
