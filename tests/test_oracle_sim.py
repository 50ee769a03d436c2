"""Pins of the NEXT-4 time-sharing simulator oracle (Fig. 8; R31-R36,
R44-R46): hand-worked scenarios (eviction, hotness, cold, pipeline instances on fragmented
free slices, their eviction exemption, migration when a large slice frees) and an
independent Python re-implementation on small traces."""
import numpy as np
import pytest

import oracle
from helpers import problem, brute_plan
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
    ctr, fs, st, last, busy, k = oracle.sim(tr)
    # requests, served, hits, unserved, reloads, evictions, terminations, slice-ticks
    assert ctr[0].tolist()[:8] == [4, 3, 2, 1, 3, 2, 0, 3] and ctr[0].tolist()[8:] == [0, 0, 0, 0]
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
    ctr, fs, st, last, busy, k = oracle.sim(tr, cold_after_us=350)
    assert ctr[0].tolist()[:6] == [5, 3, 3, 2, 2, 1]
    # A: last use t1 = 1100 -> cold at the end of t5 (1500 - 1100 >= 350); B cold at t8
    assert ctr[0][6] == 2 and st[0].tolist() == [COLD, COLD]


def test_free_slice_preference_smallest_capacity():
    prob = two_funcs([[[G4, G2, G1]]])
    tr = make_trace(prob, 1, [(0, 0, 0, 10**6)])
    ctr, fs, st, last, busy, k = oracle.sim(tr)
    assert fs[0, 0] == 2  # the 1g slice (smallest capacity that holds 5000 MiB)
    assert k[0].tolist() == [1, 0]


def pipe_funcs(nodes, mem_h=15 * 1024):
    """F0: two 8 GiB components (16 GiB: no 1g slice holds it, two 1g do); F1 (H):
    one component of mem_h."""
    f0 = dict(lat=[[40, 30, 20, 15, 10], [60, 45, 30, 20, 10]], mem=[8 * 1024, 8 * 1024], xfer=[7, 0], load=100)
    f1 = dict(lat=[[50, 40, 30, 20, 10]], mem=[mem_h], load=200)
    return problem([f0, f1], nodes, [(0, 0, 0)])


def test_pipeline_instance_on_fragmented_slices():
    """No free slice holds F0, two free 1g slices do as a 2-stage pipeline:
    the argmin plan (1g, 1g), e2e = 40 + 7 + 60 = 107, latency = load + e2e = 207; later
    requests are served at e2e; the pipeline is exclusive hot."""
    prob = pipe_funcs([[[G1, G1, (G2, 1)]]])
    tr = make_trace(prob, 3, [(0, 0, 0, 300), (1, 0, 0, 106), (2, 0, 0, 107)], window_ticks=100)
    ctr, fs, st, last, busy, k = oracle.sim(tr)
    c = ctr[0].tolist()
    # requests, served, hits (207 <= 300, 107 > 106, 107 <= 107), unserved, reloads, evictions,
    # terminations, slice-ticks (2 per tick), pipelines, migrations, pipeline-served, pipe slice-ticks
    assert c == [3, 3, 2, 0, 1, 0, 0, 6, 1, 0, 3, 6]
    assert k[0].tolist() == [2, 0] and st[0, 0] == HOT and fs[0, 0] == 0
    assert busy[0, 0] == 3 * 107


def test_pipeline_is_never_evicted():
    """F1 (one 5 GiB component) arrives after F0's pipeline took both 1g slices: no free
    slice, no pipeline possible, and the pipeline's slices are not eviction victims."""
    prob = pipe_funcs([[[G1, G1]]], mem_h=5 * 1024)
    tr = make_trace(prob, 2, [(0, 0, 0, 10**6), (1, 0, 1, 10**6)], window_ticks=100)
    ctr, fs, st, last, busy, k = oracle.sim(tr)
    assert ctr[0].tolist()[:6] == [2, 1, 1, 1, 1, 0] and ctr[0][8] == 1
    assert k[0].tolist() == [2, 0] and st[0].tolist() == [HOT, WARM]  # F1 exists, never placed


def test_pipeline_migrates_when_a_large_slice_frees():
    """H (15 GiB) holds the 2g slice; F0 becomes a (1g, 1g) pipeline.  H goes cold (idle >=
    cold_after) at the end of tick 3, the 2g slice frees and F0 migrates to it: the
    pipeline's slices are released, the new instance loads (a reload) and serves t4 at the
    2g latency 30 + 45 = 75."""
    prob = pipe_funcs([[[(G2), G1, G1]]])
    ev = [(0, 0, 1, 10**6), (1, 0, 0, 10**6), (2, 0, 0, 10**6), (3, 0, 0, 10**6), (4, 0, 0, 75)]
    tr = make_trace(prob, 5, ev, window_ticks=100)
    ctr, fs, st, last, busy, k = oracle.sim(tr, cold_after_us=300)
    c = ctr[0].tolist()
    assert c[6] == 1 and c[8] == 1 and c[9] == 1  # H terminated, one pipeline, one migration
    assert c[4] == 3  # H placed, F0's pipeline, F0's migrated instance
    assert c[2] == 5 and c[10] == 3  # every request meets its budget; 3 served by the pipeline
    assert k[0].tolist() == [1, 0] and fs[0, 0] == 0 and st[0].tolist() == [TS, COLD]


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
        inst = {}  # f -> dict(slice, last, busy, hot, pipe (list of slices) or None, e2e)
        c = [0] * 12

        def free_fit(f):
            free = [s for s in slices if not sl["busy"][s] and res[s] is None and mt[f] <= cap[sl["profile"][s]]]
            return min(free, key=lambda s: (cap[sl["profile"][s]], g[sl["profile"][s]], s)) if free else None
        for t in range(T):
            now = tr.t0_us + t * tr.tick_us
            for j in range(int(tr.req_off[v * T + t]), int(tr.req_off[v * T + t + 1])):
                f, B = int(tr.req_func[j]), int(tr.req_budget[j])
                c[0] += 1
                I = inst.setdefault(f, dict(slice=None, last=now, busy=0, hot=False, pipe=None, e2e=0))
                if I["slice"] is not None:
                    ex = exe[f][int(sl["profile"][I["slice"]])]
                    latency = ex
                elif I["pipe"] is not None:
                    ex = latency = I["e2e"]
                    c[10] += 1
                else:
                    tgt = free_fit(f)
                    if tgt is None and any(not sl["busy"][s] and res[s] is None for s in slices):
                        # a pipeline over the free slices: the independent brute force's argmin
                        occ = sl.copy()
                        occ["busy"] = [1 if (sl["busy"][s] or res.get(s) is not None) else 0 for s in range(len(sl))]
                        sub = W.Problem(**{**prob.__dict__, "slices": occ}).with_requests(
                            np.array([(f, v)], dtype=W.REQ_DTYPE), np.array([B], np.uint32))
                        best, _, _, _, cand = brute_plan(sub, 0)
                        if cand is not None:
                            taken = []
                            for p in cand["prof"]:
                                x = min(s for s in slices if occ["busy"][s] == 0 and sl["profile"][s] == p
                                        and s not in taken)
                                taken.append(x)
                            for x in taken:
                                res[x] = f
                            I["pipe"], I["e2e"] = taken, cand["e2e"]
                            c[8] += 1
                            c[4] += 1
                            c[10] += 1
                            c[1] += 1
                            c[2] += load[f] + cand["e2e"] <= B
                            I["busy"] += cand["e2e"]
                            I["last"] = now
                            continue
                    if tgt is None:
                        vic = [s for s in slices if res[s] is not None and res[s] != f
                               and inst[res[s]]["pipe"] is None
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
            c[11] += sum(1 for s in slices if res[s] is not None and inst[res[s]]["pipe"] is not None)
            if (t + 1) % tr.window_ticks == 0:
                for I in inst.values():
                    I["hot"] = I["busy"] * 100 >= thr * tr.window_ticks * tr.tick_us
                    I["busy"] = 0
            for f in list(inst):
                if now - inst[f]["last"] >= cold_after:
                    if inst[f]["slice"] is not None:
                        res[inst[f]["slice"]] = None
                    for x in inst[f]["pipe"] or []:
                        res[x] = None
                    del inst[f]
                    c[6] += 1
            for f in sorted(inst):  # pipeline migration
                if inst[f]["pipe"] is None:
                    continue
                tgt = free_fit(f)
                if tgt is None:
                    continue
                for x in inst[f]["pipe"]:
                    res[x] = None
                inst[f]["pipe"] = None
                res[tgt] = f
                inst[f]["slice"] = tgt
                c[9] += 1
                c[4] += 1
        out.append(c)
    return np.array(out, np.uint64)


@pytest.mark.parametrize("seed", range(3))
def test_sim_matches_independent_python(seed):
    tr = W.sim_trace(seed=100 + seed, T=300, n_funcs=12, nodes=[W.PART_P1, W.PART_HYBRID], rate_scale=8.0)
    ctr, *_ = oracle.sim(tr, cold_after_us=5_000_000)
    np.testing.assert_array_equal(ctr, sim_python(tr, cold_after=5_000_000))
    assert ctr[:, 5].sum() > 0 and ctr[:, 6].sum() > 0  # evictions and terminations happen
    assert ctr[:, 8].sum() > 0  # pipelines happen
