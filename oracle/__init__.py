"""CPU oracle for the FluidFaaS pipeline-construction search -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product path
(``paper_conf_hpdc_hui0s25_b200``) never imports it and shares no code with it.

``ffs_oracle.c`` holds the definitions (plan, bind, eviction score, victim), each
citing the paper passage it follows; this module only marshals numpy arrays to it.
The problem object is duck-typed (any object with the attributes of
``workload.Problem``), so this package imports nothing from the product tree.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import threading

import numpy as np
from typing import NamedTuple

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "ffs_oracle.c")
_LIB = os.path.join(_HERE, "libffs_oracle.so")
_lock = threading.Lock()
_lib = None

KEY_NONE = np.iinfo(np.int64).max
PLAN_OK, PLAN_INFEASIBLE, PLAN_BAD_REQ = 0, 1, 2
ST_EXCL_HOT, ST_TIME_SHARING, ST_WARM, ST_COLD = 0, 1, 2, 3


def build(force: bool = False) -> str:
    """Compile ffs_oracle.c with gcc (plain -O2, no fast-math)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-pthread", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


class _PlanArgs(C.Structure):
    _fields_ = [
        ("P", C.c_int), ("gpcs", C.c_void_p), ("cap_mib", C.c_void_p),
        ("F", C.c_int), ("comp_off", C.c_void_p), ("lat_us", C.c_void_p), ("mem_mib", C.c_void_p),
        ("xfer_us", C.c_void_p), ("load_us", C.c_void_p), ("max_stage_us", C.c_void_p),
        ("n_nodes", C.c_int), ("n_slices", C.c_int),
        ("sl_node", C.c_void_p), ("sl_gpu", C.c_void_p), ("sl_slice", C.c_void_p), ("sl_prof", C.c_void_p),
        ("sl_busy", C.c_void_p),
        ("R", C.c_int), ("req_func", C.c_void_p), ("req_node", C.c_void_p), ("req_slo_us", C.c_void_p),
        ("k_max", C.c_int),
        ("key", C.c_void_p), ("status", C.c_void_p), ("k", C.c_void_p), ("slice", C.c_void_p),
        ("cut_mask", C.c_void_p), ("e2e_us", C.c_void_p), ("bottleneck_us", C.c_void_p),
        ("gpcs_out", C.c_void_p), ("cvq", C.c_void_p), ("prof", C.c_void_p), ("checks", C.c_void_p),
    ]


class _DagArgs(C.Structure):
    _fields_ = [
        ("unit_off", C.c_void_p), ("unit_nb", C.c_void_p), ("unit_bend", C.c_void_p), ("unit_cond", C.c_void_p),
        ("key", C.c_void_p), ("status", C.c_void_p), ("k", C.c_void_p), ("slice", C.c_void_p),
        ("cut_mask", C.c_void_p), ("split_mask", C.c_void_p), ("e2e_us", C.c_void_p),
        ("bottleneck_us", C.c_void_p), ("gpcs_out", C.c_void_p), ("cvq", C.c_void_p), ("n_slots", C.c_void_p),
        ("prof", C.c_void_p), ("checks", C.c_void_p),
    ]


def lib():
    global _lib
    with _lock:
        if _lib is None:
            _lib = C.CDLL(build())
            _lib.oracle_plan.argtypes = [C.POINTER(_PlanArgs), C.c_int]
            _lib.oracle_plan.restype = C.c_int
            _lib.oracle_plan_ranked.argtypes = [C.POINTER(_PlanArgs), C.c_int, C.c_int]
            _lib.oracle_plan_ranked.restype = C.c_int
            _lib.oracle_plan_dag.argtypes = [C.POINTER(_PlanArgs), C.POINTER(_DagArgs), C.c_int]
            _lib.oracle_plan_dag.restype = C.c_int
            _lib.oracle_plan_joint.argtypes = [C.POINTER(_PlanArgs)]
            _lib.oracle_plan_joint.restype = C.c_int
            _lib.oracle_route.restype = C.c_int
            _lib.oracle_sim.restype = C.c_int
            _lib.oracle_evict.restype = None
            _lib.oracle_victim.restype = None
    return _lib


def _p(a):
    return a.ctypes.data_as(C.c_void_p)


def _c(a, dt):
    return np.ascontiguousarray(a, dtype=dt)


class _Held:
    """Keeps the contiguous copies alive while the C call runs."""

    def __init__(self, prob, k_max, with_checks):
        self.gpcs = _c(prob.gpcs, np.uint32)
        self.cap = _c(prob.cap_mib, np.uint32)
        self.comp_off = _c(prob.comp_off, np.uint32)
        self.lat = _c(prob.lat_us, np.uint32)
        self.mem = _c(prob.mem_mib, np.uint32)
        self.xfer = _c(prob.xfer_us, np.uint32)
        self.load = _c(prob.load_us, np.uint32)
        floor = getattr(prob, "max_stage_us", None)  # R38 throughput floor, optional
        self.floor = None if floor is None else _c(floor, np.uint32)
        sl = prob.slices
        self.sl_node = _c(sl["node"], np.uint16)
        self.sl_gpu = _c(sl["gpu"], np.uint8)
        self.sl_slice = _c(sl["slice"], np.uint8)
        self.sl_prof = _c(sl["profile"], np.uint8)
        self.sl_busy = _c(sl["busy"], np.uint8)
        self.func = _c(prob.req["func"], np.uint32)
        self.node = _c(prob.req["node"], np.uint32)
        self.slo = _c(prob.slo_us, np.uint32)
        R = self.func.shape[0]
        self.out = {
            "key": np.zeros(R, np.int64), "status": np.zeros(R, np.int32), "k": np.zeros(R, np.int32),
            "slice": np.zeros((R, 8), np.int32), "cut_mask": np.zeros(R, np.uint32),
            "e2e_us": np.zeros(R, np.uint32), "bottleneck_us": np.zeros(R, np.uint32),
            "gpcs": np.zeros(R, np.uint32), "cvq": np.zeros(R, np.uint32), "prof": np.zeros((R, 8), np.uint8),
        }
        if with_checks:
            self.out["checks"] = np.zeros((R, 3), np.uint64)
        o = self.out
        self.args = _PlanArgs(
            int(self.gpcs.shape[0]), _p(self.gpcs), _p(self.cap),
            int(self.comp_off.shape[0] - 1), _p(self.comp_off), _p(self.lat), _p(self.mem), _p(self.xfer),
            _p(self.load), None if self.floor is None else _p(self.floor), int(prob.n_nodes), int(self.sl_node.shape[0]),
            _p(self.sl_node), _p(self.sl_gpu), _p(self.sl_slice), _p(self.sl_prof), _p(self.sl_busy),
            int(R), _p(self.func), _p(self.node), _p(self.slo), int(k_max),
            _p(o["key"]), _p(o["status"]), _p(o["k"]), _p(o["slice"]), _p(o["cut_mask"]), _p(o["e2e_us"]),
            _p(o["bottleneck_us"]), _p(o["gpcs"]), _p(o["cvq"]), _p(o["prof"]),
            _p(o["checks"]) if with_checks else None)


def plan(prob, k_max: int | None = None, threads: int | None = None, checks: bool = True) -> dict:
    """Brute-force plan of every request of ``prob`` (see ffs_oracle.c: oracle_plan).

    Returns a dict of numpy arrays: key, status, k, cut_mask, e2e_us, bottleneck_us,
    gpcs, cvq, prof[R,8] (0xFF = unused), slice[R,8] (-1 = unused) and, when
    ``checks``, checks[R,3] = (candidates scored, feasible count, sum of feasible keys
    mod 2^64)."""
    k_max = int(prob.k_max if k_max is None else k_max)
    threads = os.cpu_count() if threads is None else threads
    h = _Held(prob, k_max, checks)
    rc = lib().oracle_plan(C.byref(h.args), int(threads))
    if rc != 0:
        raise ValueError("oracle_plan rejected its arguments")
    return h.out


def plan_dag(prob, dag, k_max: int | None = None, threads: int | None = None, checks: bool = True) -> dict:
    """Brute-force plan of every request of ``prob`` whose functions have the unit
    structure ``dag`` (unit_off, unit_nb, unit_bend[U,4]; see ffs_oracle.c:
    oracle_plan_dag, R40-R43, R48 for conditional units).  Returns key, status, k, cut_mask (over unit
    boundaries), split_mask (bit s: stage s runs its branches on separate slices),
    e2e_us, bottleneck_us, gpcs, cvq, n_slots, prof[R,8], slice[R,8] and checks[R,3]."""
    k_max = int(prob.k_max if k_max is None else k_max)
    threads = os.cpu_count() if threads is None else threads
    h = _Held(prob, k_max, False)
    R = prob.R
    uo, nb, be = _c(dag.unit_off, np.uint32), _c(dag.unit_nb, np.uint8), _c(dag.unit_bend, np.uint8)
    cond = getattr(dag, "unit_cond", None)
    cd = None if cond is None else _c(cond, np.uint8)  # R48 conditional units (nullable)
    o = {"key": np.zeros(R, np.int64), "status": np.zeros(R, np.int32), "k": np.zeros(R, np.int32),
         "slice": np.zeros((R, 8), np.int32), "cut_mask": np.zeros(R, np.uint32),
         "split_mask": np.zeros(R, np.uint32), "e2e_us": np.zeros(R, np.uint32),
         "bottleneck_us": np.zeros(R, np.uint32), "gpcs": np.zeros(R, np.uint32), "cvq": np.zeros(R, np.uint32),
         "n_slots": np.zeros(R, np.uint32), "prof": np.zeros((R, 8), np.uint8)}
    if checks:
        o["checks"] = np.zeros((R, 3), np.uint64)
    d = _DagArgs(_p(uo), _p(nb), _p(be), _p(cd) if cd is not None else None, _p(o["key"]), _p(o["status"]), _p(o["k"]), _p(o["slice"]),
                 _p(o["cut_mask"]), _p(o["split_mask"]), _p(o["e2e_us"]), _p(o["bottleneck_us"]),
                 _p(o["gpcs"]), _p(o["cvq"]), _p(o["n_slots"]), _p(o["prof"]),
                 _p(o["checks"]) if checks else None)
    rc = lib().oracle_plan_dag(C.byref(h.args), C.byref(d), int(threads))
    if rc != 0:
        raise ValueError("oracle_plan_dag rejected its arguments")
    return o


def plan_any(prob, k_max: int | None = None, threads: int | None = None) -> tuple[dict, np.ndarray]:
    """NEXT-2 any-invoker (cross-node) planning, R39: a request may be served by
    any invoker's node (the controller's load balancer sees every invoker); its
    plan is the argmin over nodes v of the plan against v's free slices (R10 still holds: a
    pipeline never spans nodes); ties in the key prefer the home node, then the lowest node
    id.  Plainly: one full oracle.plan per node with every request moved there, then a
    per-request minimum.  Returns (plans as plan(), node[R]: the serving node or -1)."""
    R = prob.R
    best = None
    node = np.full(R, -1, np.int64)
    home = np.asarray(prob.req["node"], np.int64)
    for v in range(int(prob.n_nodes)):
        req = prob.req.copy()
        req["node"] = v
        o = plan(prob.with_requests(req, prob.slo_us), k_max=k_max, threads=threads, checks=False)
        if best is None:
            best = {k: a.copy() for k, a in o.items()}
            node[:] = v
            continue
        # (key, not home, node id) lexicographic: v > every earlier node id
        cur_home = node == home
        take = (o["key"] < best["key"]) | ((o["key"] == best["key"]) & (home == v) & ~cur_home)
        for k in best:
            best[k][take] = o[k][take]
        node[take] = v
    node[best["status"] != PLAN_OK] = -1
    # an out-of-range function or home node stays a bad request (as in plan())
    bad = np.nonzero((np.asarray(prob.req["func"], np.int64) >= prob.F) | (home >= int(prob.n_nodes)))[0]
    if len(bad):
        o = plan(prob.subset(bad), k_max=k_max, threads=threads, checks=False)
        for k in best:
            best[k][bad] = o[k]
        node[bad] = -1
    return best, node


def plan_ranked(prob, p_ref: int | None = None, k_max: int | None = None, threads: int | None = None) -> dict:
    """NEXT-1: the paper's offline CV ranking + first-fit walk (ffs_oracle.c:
    oracle_plan_ranked).  p_ref = reference profile of the offline CV (default: the
    profile with the most GPCs).  key = position of the chosen partition in the ranked
    list.  Same output fields as plan() (no checks)."""
    k_max = int(prob.k_max if k_max is None else k_max)
    threads = os.cpu_count() if threads is None else threads
    if p_ref is None:
        p_ref = int(np.argmax(np.asarray(prob.gpcs)))
    h = _Held(prob, k_max, False)
    rc = lib().oracle_plan_ranked(C.byref(h.args), int(p_ref), int(threads))
    if rc != 0:
        raise ValueError("oracle_plan_ranked rejected its arguments")
    return h.out


def plan_joint(prob, k_max: int | None = None) -> dict:
    """NEXT-2: joint commit of the batch, node by node in ascending adjusted deadline,
    each plan taking its slices (ffs_oracle.c: oracle_plan_joint).  Single-threaded."""
    h = _Held(prob, int(prob.k_max if k_max is None else k_max), False)
    rc = lib().oracle_plan_joint(C.byref(h.args))
    if rc != 0:
        raise ValueError("oracle_plan_joint rejected its arguments")
    return h.out


def route(prob, inst_func, inst_state, inst_lat, inst_cap) -> np.ndarray:
    """NEXT-2 routing (ffs_oracle.c: oracle_route): instance index per request."""
    h = _Held(prob, prob.k_max, False)
    fu, st = _c(inst_func, np.uint32), _c(inst_state, np.uint8)
    la, ca = _c(inst_lat, np.uint32), _c(inst_cap, np.uint32)
    out = np.full(h.func.shape[0], -1, np.int32)
    lib().oracle_route(C.byref(h.args), C.c_int(int(fu.shape[0])), _p(fu), _p(st), _p(la), _p(ca), _p(out))
    return out


def sim(trace, thr_pct: int = 30, cold_after_us: int = 600_000_000, k_max: int | None = None):
    """NEXT-4 time-sharing simulator with pipeline instances and migration (ffs_oracle.c:
    oracle_sim).  Returns (ctr[N, 12], slice[N, F], state[N, F], last_used[N, F], busy[N, F],
    stages[N, F]).  k_max = pipeline search depth (default the problem's; 0: monolithic
    instances only -- the search then has no candidate)."""
    prob = trace.problem
    h = _Held(prob, int(prob.k_max if k_max is None else k_max), False)
    N, F = int(prob.n_nodes), int(prob.comp_off.shape[0] - 1)
    off, fu, bu = _c(trace.req_off, np.uint32), _c(trace.req_func, np.uint32), _c(trace.req_budget, np.uint32)
    ctr = np.zeros((N, 12), np.uint64)
    fs, fst = np.zeros((N, F), np.int32), np.zeros((N, F), np.uint8)
    fl, fb = np.zeros((N, F), np.uint64), np.zeros((N, F), np.uint32)
    fk = np.zeros((N, F), np.uint8)
    lib().oracle_sim(C.byref(h.args), C.c_int(trace.T), _p(off), _p(fu), _p(bu), C.c_uint64(trace.t0_us),
                     C.c_uint32(trace.tick_us), C.c_uint32(trace.window_ticks), C.c_uint32(thr_pct),
                     C.c_uint64(cold_after_us), _p(ctr), _p(fs), _p(fst), _p(fl), _p(fb), _p(fk))
    return ctr, fs, fst, fl, fb, fk


class Evict(NamedTuple):
    """One snapshot's keep-alive states and LRU order (no packed key): the least recently
    used evictable instance is the one with the largest idle time, ties to the lower index."""
    state: np.ndarray      # uint8 FFS_ST_*
    evictable: np.ndarray  # bool
    idle: np.ndarray       # uint64 now - last_used (0 for a future last use)


def evict(inst: np.ndarray, now_us: int, util_thr_pct: int = 30, window_us: int = 10_000_000,
          cold_after_us: int = 600_000_000) -> Evict:
    """Eviction state + LRU order of one snapshot (ffs_oracle.c: oracle_evict)."""
    n = int(inst.shape[0])
    sl = _c(inst["slice"], np.int32)
    fl = _c(inst["flags"], np.uint8)
    bu = _c(inst["busy_us"], np.uint32)
    lu = _c(inst["last_used_us"], np.uint64)
    state = np.zeros(n, np.uint8)
    ev = np.zeros(n, np.uint8)
    idle = np.zeros(n, np.uint64)
    lib().oracle_evict(C.c_int(n), _p(sl), _p(fl), _p(bu), _p(lu), C.c_uint64(int(now_us)),
                       C.c_uint32(util_thr_pct), C.c_uint32(window_us), C.c_uint64(int(cold_after_us)),
                       _p(state), _p(ev), _p(idle))
    return Evict(state, ev.astype(bool), idle)


def victim(prob, status: np.ndarray, inst: np.ndarray, ev: Evict, k_max: int | None = None) -> np.ndarray:
    """Time-share victim per INFEASIBLE request (ffs_oracle.c: oracle_victim)."""
    h = _Held(prob, int(prob.k_max if k_max is None else k_max), False)
    st = _c(status, np.int32)
    sl = _c(inst["slice"], np.int32)
    e = _c(ev.evictable, np.uint8)
    idle = _c(ev.idle, np.uint64)
    out = np.zeros(h.func.shape[0], np.int32)
    lib().oracle_victim(C.byref(h.args), _p(st), C.c_int(int(inst.shape[0])), _p(sl), _p(e), _p(idle), _p(out))
    return out
