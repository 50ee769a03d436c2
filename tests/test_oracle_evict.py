"""Pins of the eviction oracle (§5.3, Fig. 8) -- CPU only."""
import numpy as np

import oracle
from helpers import problem, KEY_NONE
from paper_conf_hpdc_hui0s25_b200 import workload as W

HOT, TS, WARM, COLD = oracle.ST_EXCL_HOT, oracle.ST_TIME_SHARING, oracle.ST_WARM, oracle.ST_COLD
WIN = 10_000_000
NOW = 5_000_000_000


def inst(rows):
    a = np.zeros(len(rows), dtype=W.INST_DTYPE)
    for i, (func, sl, flags, busy, last) in enumerate(rows):
        a[i]["func"], a[i]["slice"], a[i]["flags"], a[i]["busy_us"], a[i]["last_used_us"] = func, sl, flags, busy, last
    return a


def test_state_rules_fig8():
    rows = [
        (0, 3, 0, 2_999_999, NOW - 10),          # 29.99999% < 30% -> time sharing
        (0, 4, 0, 3_000_000, NOW - 10),          # exactly 30% -> exclusive hot ("exceeds")
        (1, 5, W.INST_PIPELINE, 0, NOW - 10),    # pipelines are exclusive hot
        (2, -1, 0, 0, NOW - 10),                 # evicted to CPU -> warm
        (3, 6, 0, 0, NOW - 600_000_000),         # 10 minutes without requests -> cold
        (3, 7, 0, 0, NOW - 599_999_999),         # just under 10 minutes
        (4, 8, W.INST_BUSY, 0, NOW - 10),        # serving right now: not evictable
        (5, -1, W.INST_PIPELINE, 9_000_000, NOW - 700_000_000),  # cold wins over everything
    ]
    ev = oracle.evict(inst(rows), NOW, 30, WIN, 600_000_000)
    assert ev.state.tolist() == [TS, HOT, HOT, WARM, COLD, TS, TS, COLD]
    assert ev.evictable.tolist() == [i in (0, 5) for i in range(len(rows))]
    assert ev.idle.tolist() == [NOW - r[4] for r in rows]


def test_epoch_timestamps_are_representable():
    # R20c: no packed key in the oracle -- Unix-epoch microseconds (~1.8e15 > 2^43) order
    # exactly like small ones; a last use in the future counts as idle 0 (R20b)
    T = 1_800_000_000_000_000
    rows = [(0, 1, 0, 0, T - 7), (1, 2, 0, 0, T - 9), (2, 3, 0, 0, T + 5)]
    ev = oracle.evict(inst(rows), T)
    assert ev.state.tolist() == [TS, TS, TS] and ev.evictable.all()
    assert ev.idle.tolist() == [7, 9, 0]


def test_lru_order_and_tie_break():
    # evict the least-recently-used time-sharing instance; equal last-use -> lower index
    rows = [(0, 1, 0, 0, NOW - 50), (1, 2, 0, 0, NOW - 500), (2, 3, 0, 0, NOW - 500), (3, 4, 0, 0, NOW - 5)]
    ev = oracle.evict(inst(rows), NOW)
    order = sorted(range(len(rows)), key=lambda i: (-int(ev.idle[i]), i))
    assert order == [1, 2, 0, 3]
    # the victim rule applies that order: every instance on one node whose slice fits
    G = 4
    f = dict(lat=[[100] * 5], mem=[1024], load=0)
    prob = problem([f], [[[(G, 1), (G, 1), (G, 1), (G, 1)]]], [(0, 0, 10_000)])
    v = oracle.victim(prob, np.array([oracle.PLAN_INFEASIBLE]), inst([(r[0], i, 0, 0, r[4]) for i, r in
                                                                    enumerate(rows)]), ev)
    assert v.tolist() == [1]


def test_victim_rules():
    # node 0: slices 0 (1g), 1 (2g), 2 (4g); node 1: slice 3 (7g); all occupied
    G1, G2, G4, G7 = 0, 1, 3, 4
    f = dict(lat=[[400, 300, 200, 150, 100]], mem=[15 * 1024], load=50)
    prob = problem([f], [[[(G1, 1), (G2, 1), (G4, 1)]], [[(G7, 1)]]],
                   [(0, 0, 400), (0, 0, 200), (0, 1, 1000), (0, 0, 400)])
    rows = [
        (7, 0, 0, 0, NOW - 900),   # 1g: 15 GB does not fit
        (8, 1, 0, 0, NOW - 500),   # 2g: 300 + 50 <= 400
        (9, 2, 0, 0, NOW - 100),   # 4g: 150 + 50 <= 400, more recently used
        (9, 3, 0, 0, NOW - 999),   # other node
    ]
    ev = oracle.evict(inst(rows), NOW)
    status = np.array([oracle.PLAN_INFEASIBLE, oracle.PLAN_INFEASIBLE, oracle.PLAN_INFEASIBLE, oracle.PLAN_OK])
    v = oracle.victim(prob, status, inst(rows), ev)
    # r0: LRU among {1, 2} -> 1;  r1: budget 200 leaves only 4g (150+50) -> 2;
    # r2: node 1 -> 3;  r3: has a free-slice plan -> no victim
    assert v.tolist() == [1, 2, 3, -1]


def test_c4_generator_snapshot_mix():
    wl = W.config4(T=8)
    t0, t1 = int(wl.tick_off[0]), int(wl.tick_off[1])
    ev = oracle.evict(wl.inst[t0:t1], int(wl.now_us[0]))
    counts = np.bincount(ev.state, minlength=4)
    assert (counts > 0).all(), counts  # every keep-alive state occurs
    assert ev.evictable.sum() > 10
