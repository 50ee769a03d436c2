"""Hand-built tiny problems and an independent pure-Python brute force (test-only).

``brute_plan`` is a second, independent reading of the definition used to pin the C
oracle: itertools enumeration, exact rational CV^2 through ``statistics.pvariance`` on
Fractions (Eq. 1, population std), no shared code with oracle/ffs_oracle.c.
"""
from __future__ import annotations

import itertools
import statistics
from fractions import Fraction

import numpy as np

from paper_conf_hpdc_hui0s25_b200 import workload as W

KEY_NONE = np.iinfo(np.int64).max


def problem(funcs, nodes, requests, k_max=4, gpcs=None, cap=None):
    """funcs: list of dicts {lat: [[...P] per component], mem: [...], xfer: [...], load: int}.
    nodes: list (per node) of GPUs, each GPU a list of slices in slice order; a slice is
    a profile id (free) or a tuple (profile id, 1) (busy).  requests: (func, node, budget)."""
    gpcs = W.PROFILE_GPCS.copy() if gpcs is None else np.asarray(gpcs, np.uint32)
    cap = W.PROFILE_CAP_MIB.copy() if cap is None else np.asarray(cap, np.uint32)
    lat, mem, xfer, load, off = [], [], [], [], [0]
    for f in funcs:
        lat += [list(r) for r in f["lat"]]
        mem += list(f["mem"])
        x = list(f.get("xfer", [0] * len(f["mem"])))
        xfer += x
        load.append(f.get("load", 0))
        off.append(off[-1] + len(f["mem"]))
    rows = []
    for v, gpus in enumerate(nodes):
        for g, gpu in enumerate(gpus):
            for s, item in enumerate(gpu):
                p, busy = (item, 0) if isinstance(item, int) else (item[0], item[1])
                rows.append((v, g, s, p, busy, 0, -1))
    slices = np.array(rows, dtype=W.SLICE_DTYPE)
    req = np.zeros(len(requests), dtype=W.REQ_DTYPE)
    req["func"] = [r[0] for r in requests]
    req["node"] = [r[1] for r in requests]
    slo = np.array([r[2] for r in requests], dtype=np.uint32)
    return W.Problem(name="hand", gpcs=gpcs, cap_mib=cap, comp_off=np.array(off, np.uint32),
                     lat_us=np.array(lat, np.uint32).reshape(-1, gpcs.shape[0]),
                     mem_mib=np.array(mem, np.uint32), xfer_us=np.array(xfer, np.uint32),
                     load_us=np.array(load, np.uint32), n_nodes=len(nodes), slices=slices,
                     req=req, slo_us=slo, k_max=k_max)


def pack_key(cvq, k, gpcs, idx):
    return (cvq << 50) | ((k - 1) << 47) | (gpcs << 41) | idx


def brute_plan(prob, r, k_max=None):
    """Independent brute force for request r.  Returns (best_key, n_scored, n_feasible,
    key_sum mod 2^64, best candidate dict or None)."""
    K = prob.k_max if k_max is None else k_max
    f, v, B = int(prob.req["func"][r]), int(prob.req["node"][r]), int(prob.slo_us[r])
    a, b = int(prob.comp_off[f]), int(prob.comp_off[f + 1])
    n, P = b - a, prob.P
    lat = prob.lat_us[a:b].astype(int).tolist()
    mem = prob.mem_mib[a:b].astype(int).tolist()
    xfer = prob.xfer_us[a:b].astype(int).tolist()
    sl = prob.slices
    free = [int(((sl["node"] == v) & (sl["busy"] == 0) & (sl["profile"] == p)).sum()) for p in range(P)]
    fl = getattr(prob, "max_stage_us", None)
    floor = 0 if fl is None else int(fl[f])
    best, best_c, idx, nfeas, ksum = KEY_NONE, None, 0, 0, 0
    for k in range(1, min(n, K) + 1):
        masks = sorted(m for m in range(1 << (n - 1)) if bin(m).count("1") == k - 1)
        for mask in masks:
            cuts = [j for j in range(n - 1) if mask >> j & 1]
            bounds = [0] + [j + 1 for j in cuts] + [n]
            stages = [range(bounds[i], bounds[i + 1]) for i in range(k)]
            for seq in itertools.product(range(P), repeat=k):
                t = [sum(lat[c][p] for c in st) for st, p in zip(stages, seq)]
                m = [sum(mem[c] for c in st) for st in stages]
                e2e = sum(t) + sum(xfer[j] for j in cuts)
                ok = all(mi <= int(prob.cap_mib[p]) for mi, p in zip(m, seq))
                ok = ok and all(seq.count(p) <= free[p] for p in range(P)) and e2e <= B
                ok = ok and (floor == 0 or max(t) <= floor)  # R38: throughput floor on the bottleneck
                if ok:
                    tf = [Fraction(x) for x in t]
                    cv2 = statistics.pvariance(tf) / statistics.mean(tf) ** 2
                    cvq = int(cv2 * 1024)  # floor of a non-negative rational
                    g = sum(int(prob.gpcs[p]) for p in seq)
                    key = pack_key(cvq, k, g, idx)
                    nfeas += 1
                    ksum = (ksum + key) % (1 << 64)
                    if key < best:
                        best = key
                        best_c = dict(k=k, mask=mask, prof=list(seq), t=t, e2e=e2e, gpcs=g, cvq=cvq)
                idx += 1
    return best, idx, nfeas, ksum, best_c


def candidate_keys(prob, r, k_max=None):
    """Every candidate of request r as (k, cut-mask rank, key or None), canonical order
    (independent enumeration; used to emulate shards of the task space)."""
    K = prob.k_max if k_max is None else k_max
    f, v, B = int(prob.req["func"][r]), int(prob.req["node"][r]), int(prob.slo_us[r])
    a, b = int(prob.comp_off[f]), int(prob.comp_off[f + 1])
    n, P = b - a, prob.P
    lat = prob.lat_us[a:b].astype(int).tolist()
    mem = prob.mem_mib[a:b].astype(int).tolist()
    xfer = prob.xfer_us[a:b].astype(int).tolist()
    sl = prob.slices
    free = [int(((sl["node"] == v) & (sl["busy"] == 0) & (sl["profile"] == p)).sum()) for p in range(P)]
    out, idx = [], 0
    for k in range(1, min(n, K) + 1):
        masks = sorted(m for m in range(1 << (n - 1)) if bin(m).count("1") == k - 1)
        for rank, mask in enumerate(masks):
            cuts = [j for j in range(n - 1) if mask >> j & 1]
            bounds = [0] + [j + 1 for j in cuts] + [n]
            stages = [range(bounds[i], bounds[i + 1]) for i in range(k)]
            for seq in itertools.product(range(P), repeat=k):
                t = [sum(lat[c][p] for c in st) for st, p in zip(stages, seq)]
                m = [sum(mem[c] for c in st) for st in stages]
                ok = all(mi <= int(prob.cap_mib[p]) for mi, p in zip(m, seq))
                ok = ok and all(seq.count(p) <= free[p] for p in range(P))
                ok = ok and sum(t) + sum(xfer[j] for j in cuts) <= B
                key = None
                if ok:
                    tf = [Fraction(x) for x in t]
                    cvq = int(statistics.pvariance(tf) / statistics.mean(tf) ** 2 * 1024)
                    key = pack_key(cvq, k, sum(int(prob.gpcs[p]) for p in seq), idx)
                out.append((k, rank, key))
                idx += 1
    return out


def abi_evict_score(ev, cold_after_us: int = 600_000_000) -> np.ndarray:
    """The ABI's documented LRU key (include/ffs.h, ffs_evict_scores) of an oracle.Evict:
    ((cold_after_us - idle) << 20) | index for an evictable instance, FFS_KEY_NONE
    otherwise -- smaller = less recently used, ties to the lower index."""
    n = len(ev.state)
    out = np.full(n, KEY_NONE, dtype=np.int64)
    i = np.flatnonzero(ev.evictable)
    out[i] = ((np.uint64(cold_after_us) - ev.idle[i].astype(np.uint64)) << np.uint64(20)).astype(np.int64) | i
    return out
