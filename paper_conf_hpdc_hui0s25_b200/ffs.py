"""Thin Python binding of libffs.so (include/ffs.h): argument marshalling only.

Every step of the search runs in the CUDA kernels behind the C ABI; PyTorch provides
device memory, streams and (for multi-GPU) the NCCL process group.  There is no CPU
fallback: importing this module fails if libffs.so is missing, and creating a Planner
fails without an sm_100 device.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

from . import workload as W

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("FFS_LIB") or os.path.join(_PKG, "libffs.so")  # FFS_LIB: experiment builds
if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is not built; run `python -c 'import __graft_entry__ as g; g.build()'`")
_lib = C.CDLL(LIB_PATH)

FFS_OK, FFS_ERR_ARG, FFS_ERR_RANGE, FFS_ERR_CUDA, FFS_ERR_STATE = 0, -1, -2, -3, -4
PLAN_OK, PLAN_INFEASIBLE, PLAN_BAD_REQ = 0, 1, 2
SEARCH_BOUNDED, SEARCH_EXHAUSTIVE = 0, 1
KEY_NONE = np.iinfo(np.int64).max

PLAN_DTYPE = np.dtype([("key", "<i8"), ("status", "<u4"), ("k", "<u4"), ("cut_mask", "<u4"), ("e2e_us", "<u4"),
                       ("bottleneck_us", "<u4"), ("gpcs", "<u4"), ("cvq", "<u4"), ("prof", "u1", (8,)),
                       ("slice", "<i4", (8,)), ("victim", "<i4")])
assert PLAN_DTYPE.itemsize == 80
# ffs_dag_plan (NEXT-1 DAG stages, R40-R43)
DAG_PLAN_DTYPE = np.dtype([("key", "<i8"), ("status", "<u4"), ("k", "<u4"), ("cut_mask", "<u4"), ("split_mask", "<u4"),
                           ("e2e_us", "<u4"), ("bottleneck_us", "<u4"), ("gpcs", "<u4"), ("cvq", "<u4"),
                           ("n_slots", "<u4"), ("pad", "<u4"), ("prof", "u1", (8,)), ("slice", "<i4", (8,))])
assert DAG_PLAN_DTYPE.itemsize == 88


class _Profiles(C.Structure):
    _fields_ = [("n_profiles", C.c_uint32), ("gpcs", C.c_uint32 * 8), ("mem_mib", C.c_uint32 * 8)]


class _Table(C.Structure):
    _fields_ = [("n_funcs", C.c_uint32), ("comp_off", C.c_void_p), ("lat_us", C.c_void_p), ("mem_mib", C.c_void_p),
                ("xfer_us", C.c_void_p), ("load_us", C.c_void_p), ("max_stage_us", C.c_void_p)]


class _Cluster(C.Structure):
    _fields_ = [("n_nodes", C.c_uint32), ("n_slices", C.c_uint32), ("slices", C.c_void_p)]


class _DagTable(C.Structure):
    _fields_ = [("n_funcs", C.c_uint32), ("unit_off", C.c_void_p), ("unit_nb", C.c_void_p), ("unit_bend", C.c_void_p),
                ("unit_cond", C.c_void_p)]


class _EvictParams(C.Structure):
    _fields_ = [("util_thr_pct", C.c_uint32), ("window_us", C.c_uint32), ("cold_after_us", C.c_uint64)]


_vp, _u32, _u64, _i32 = C.c_void_p, C.c_uint32, C.c_uint64, C.c_int
_sig = {
    "ffs_create": ([_i32, C.POINTER(_vp)], _i32),
    "ffs_destroy": ([_vp], None),
    "ffs_last_error": ([_vp], C.c_char_p),
    "ffs_stage_tables": ([_vp, C.POINTER(_Profiles), C.POINTER(_Table), C.POINTER(_Cluster)], _i32),
    "ffs_plan_keys": ([_vp, _vp, _vp, _u32, _u32, _u32, _u32, _vp, _vp, _vp], _i32),
    "ffs_plan_keys_range": ([_vp, _vp, _vp, _u32, _u32, _u32, _u32, _u32, _u32, _vp, _vp, _vp], _i32),
    "ffs_plan_decode": ([_vp, _vp, _vp, _vp, _u32, _u32, _vp, _vp, _u32, _vp, _vp], _i32),
    "ffs_plan_batch": ([_vp, _vp, _vp, _u32, _u32, _vp, _vp], _i32),
    "ffs_plan_batch_host": ([_vp, _vp, _vp, _u32, _u32, _vp, _vp], _i32),
    "ffs_evict_scores": ([_vp, _vp, _u32, _u64, C.POINTER(_EvictParams), _vp, _vp, _vp], _i32),
    "ffs_evict_scores_ticks": ([_vp, _vp, _vp, _vp, _u32, C.POINTER(_EvictParams), _vp, _vp, _vp], _i32),
    "ffs_evict_victims": ([_vp, _vp, _vp, _vp, _u32, _vp, _vp, _vp, _u32, _vp, _vp], _i32),
    "ffs_evict_step": ([_vp, _vp, _vp, _vp, _u32, C.POINTER(_EvictParams), _vp, _vp, _vp, _vp, _vp, _vp, _u32, _vp,
                        _vp], _i32),
    "ffs_plan_joint": ([_vp, _vp, _vp, _u32, _u32, _vp, C.POINTER(C.c_uint32), _vp], _i32),
    "ffs_simulate": ([_vp, _vp, _vp, _vp, _u32, _u64, _u32, _u32, _u32, _u64, _u32, _vp, _vp, _vp, _vp, _vp, _vp, _vp],
                     _i32),
    "ffs_route": ([_vp, _vp, _vp, _u32, _vp, _vp, _vp, _vp, _u32, _vp, _vp], _i32),
    "ffs_frontier_build": ([_vp, _u32, C.POINTER(C.c_uint32), C.POINTER(C.c_uint32), _vp], _i32),
    "ffs_plan_frontier": ([_vp, _vp, _vp, _u32, _vp, _vp], _i32),
    "ffs_plan_frontier_any": ([_vp, _vp, _vp, _u32, _vp, _vp, _vp], _i32),
    "ffs_rank_partitions": ([_vp, _u32, _u32], _i32),
    "ffs_plan_ranked": ([_vp, _vp, _vp, _u32, _vp, _vp], _i32),
    "ffs_dag_stage": ([_vp, C.POINTER(_DagTable), _u32], _i32),
    "ffs_plan_dag": ([_vp, _vp, _vp, _u32, _vp, _vp, _vp], _i32),
    "ffs_bench_int_peak": ([_vp, C.POINTER(C.c_double), C.POINTER(C.c_double)], _i32),
    "ffs_segment_times": ([_vp, C.POINTER(C.c_float)], _i32),
    "ffs_debug_filter_misses": ([_vp, C.POINTER(C.c_uint64)], _i32),
    "ffs_set_search_mode": ([_vp, _u32], _i32),
    "ffs_search_scored": ([_vp, C.POINTER(C.c_uint64)], _i32),
    "ffs_search_live_records": ([_vp, C.POINTER(C.c_uint64)], _i32),
    "ffs_bench_packed_peak": ([_vp, _u32, C.POINTER(C.c_double), C.POINTER(C.c_double)], _i32),
}
for _name, (_args, _res) in _sig.items():
    _f = getattr(_lib, _name)
    _f.argtypes = _args
    _f.restype = _res

EXPORTS = tuple(_sig)


class FFSError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"ffs status {status}: {msg}")
        self.status = status


def _ptr(t) -> int | None:
    """Device pointer of a torch tensor (or None)."""
    if t is None:
        return None
    if not t.is_cuda:
        raise ValueError("expected a CUDA tensor")
    if not t.is_contiguous():
        raise ValueError("expected a contiguous tensor")
    return t.data_ptr()


def _host(a: np.ndarray) -> int:
    return a.ctypes.data


def _stream(stream) -> int | None:
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    return getattr(stream, "cuda_stream", stream)


class Planner:
    """One libffs context on one CUDA device."""

    def __init__(self, device: int = 0):
        h = _vp()
        rc = _lib.ffs_create(int(device), C.byref(h))
        if rc != FFS_OK:
            raise FFSError(rc, f"ffs_create({device}) failed: no sm_100 CUDA device")
        self._h = h
        self.device = int(device)
        self.k_max = None

    def close(self):
        if getattr(self, "_h", None) and _lib is not None:  # (module globals may be gone at exit)
            _lib.ffs_destroy(self._h)
        self._h = None

    __del__ = close

    def _check(self, rc):
        if rc != FFS_OK:
            raise FFSError(rc, _lib.ffs_last_error(self._h).decode())

    # ---- A0 ------------------------------------------------------------------------
    def stage(self, prob) -> None:
        """ffs_stage_tables from a workload.Problem-like object (host numpy arrays)."""
        P = int(prob.gpcs.shape[0])
        pr = _Profiles()
        pr.n_profiles = P
        for p in range(min(P, 8)):
            pr.gpcs[p] = int(prob.gpcs[p])
            pr.mem_mib[p] = int(prob.cap_mib[p])
        keep = [np.ascontiguousarray(prob.comp_off, np.uint32), np.ascontiguousarray(prob.lat_us, np.uint32),
                np.ascontiguousarray(prob.mem_mib, np.uint32), np.ascontiguousarray(prob.xfer_us, np.uint32),
                np.ascontiguousarray(prob.load_us, np.uint32)]
        floor = getattr(prob, "max_stage_us", None)  # R38 throughput floor (optional)
        if floor is not None:
            keep.append(np.ascontiguousarray(floor, np.uint32))
        tb = _Table(int(keep[0].shape[0] - 1), *[_host(a) for a in keep])
        if floor is None:
            tb.max_stage_us = None
        sl = np.ascontiguousarray(prob.slices, dtype=W.SLICE_DTYPE)
        cl = _Cluster(int(prob.n_nodes), int(sl.shape[0]), _host(sl) if sl.shape[0] else None)
        self._check(_lib.ffs_stage_tables(self._h, C.byref(pr), C.byref(tb), C.byref(cl)))

    # ---- A1-A5 ---------------------------------------------------------------------
    def plan_keys(self, req, slo, k_max: int, rank: int = 0, world: int = 1, keys=None, checks=None, stream=None):
        import torch
        n = int(slo.numel())
        if keys is None:
            keys = torch.empty(n, dtype=torch.int64, device=slo.device)
        self._check(_lib.ffs_plan_keys(self._h, _ptr(req), _ptr(slo), n, int(k_max), int(rank), int(world),
                                       _ptr(keys), _ptr(checks), _stream(stream)))
        return keys

    def plan_keys_range(self, req, slo, k_max: int, k_first: int, k_last: int, rank: int = 0, world: int = 1,
                        keys=None, checks=None, stream=None):
        """Segments k_first..k_last; k_first > 1 continues from (and prunes against) `keys`."""
        import torch
        n = int(slo.numel())
        if keys is None:
            keys = torch.empty(n, dtype=torch.int64, device=slo.device)
        self._check(_lib.ffs_plan_keys_range(self._h, _ptr(req), _ptr(slo), n, int(k_max), int(k_first), int(k_last),
                                             int(rank), int(world), _ptr(keys), _ptr(checks), _stream(stream)))
        return keys

    # ---- A6 / A8 -------------------------------------------------------------------
    def plan_decode(self, req, slo, keys, k_max: int, inst=None, scores=None, out=None, stream=None):
        import torch
        n = int(slo.numel())
        if out is None:
            out = torch.empty((n, PLAN_DTYPE.itemsize), dtype=torch.uint8, device=slo.device)
        n_inst = 0 if inst is None else int(inst.numel() // W.INST_DTYPE.itemsize)
        self._check(_lib.ffs_plan_decode(self._h, _ptr(req), _ptr(slo), _ptr(keys), n, int(k_max), _ptr(inst),
                                         _ptr(scores), n_inst, _ptr(out), _stream(stream)))
        return out

    def plan_batch(self, req, slo, k_max: int, out=None, stream=None):
        import torch
        n = int(slo.numel())
        if out is None:
            out = torch.empty((n, PLAN_DTYPE.itemsize), dtype=torch.uint8, device=slo.device)
        self._check(_lib.ffs_plan_batch(self._h, _ptr(req), _ptr(slo), n, int(k_max), _ptr(out), _stream(stream)))
        return out

    def plan_batch_host(self, req: np.ndarray, slo: np.ndarray, k_max: int, out: np.ndarray | None = None,
                        stream=None) -> np.ndarray:
        """End-to-end call with host arrays (pinned recommended): H2D, plan, D2H, sync."""
        n = int(slo.shape[0])
        if out is None:
            out = np.empty(n, dtype=PLAN_DTYPE)
        assert req.dtype == W.REQ_DTYPE and slo.dtype == np.uint32 and out.dtype == PLAN_DTYPE
        self._check(_lib.ffs_plan_batch_host(self._h, _host(req), _host(slo), n, int(k_max), _host(out),
                                             _stream(stream)))
        return out

    # ---- A7 / A8 (eviction) ----------------------------------------------------------
    @staticmethod
    def _params(util_thr_pct=30, window_us=10_000_000, cold_after_us=600_000_000):
        return _EvictParams(int(util_thr_pct), int(window_us), int(cold_after_us))

    def evict_scores(self, inst, now_us: int, score=None, state=None, stream=None, **params):
        import torch
        n = int(inst.numel() // W.INST_DTYPE.itemsize)
        score = torch.empty(n, dtype=torch.int64, device=inst.device) if score is None else score
        state = torch.empty(n, dtype=torch.uint8, device=inst.device) if state is None else state
        prm = self._params(**params)
        self._check(_lib.ffs_evict_scores(self._h, _ptr(inst), n, int(now_us), C.byref(prm), _ptr(score),
                                          _ptr(state), _stream(stream)))
        return score, state

    def evict_scores_ticks(self, inst, tick_off, now_us, score=None, state=None, stream=None, **params):
        import torch
        n = int(inst.numel() // W.INST_DTYPE.itemsize)
        score = torch.empty(n, dtype=torch.int64, device=inst.device) if score is None else score
        state = torch.empty(n, dtype=torch.uint8, device=inst.device) if state is None else state
        prm = self._params(**params)
        self._check(_lib.ffs_evict_scores_ticks(self._h, _ptr(inst), _ptr(tick_off), _ptr(now_us),
                                                int(now_us.numel()), C.byref(prm), _ptr(score), _ptr(state),
                                                _stream(stream)))
        return score, state

    def evict_victims(self, req, slo, req_tick, inst, tick_off, score, victim=None, stream=None):
        import torch
        n = int(slo.numel())
        victim = torch.empty(n, dtype=torch.int32, device=slo.device) if victim is None else victim
        self._check(_lib.ffs_evict_victims(self._h, _ptr(req), _ptr(slo), _ptr(req_tick), n, _ptr(inst),
                                           _ptr(tick_off), _ptr(score), int(tick_off.numel() - 1), _ptr(victim),
                                           _stream(stream)))
        return victim

    def evict_step(self, inst, tick_off, now_us, req, slo, req_tick=None, load_off=None, score=None, state=None,
                   victim=None, stream=None, **params):
        """Scores + states of every tick's instances and the victims of the loads, fused
        (load_off: loads grouped by tick, the victims picked inside the tick's CTA)."""
        import torch
        n = int(inst.numel() // W.INST_DTYPE.itemsize)
        nr = int(slo.numel())
        score = torch.empty(n, dtype=torch.int64, device=inst.device) if score is None else score
        state = torch.empty(n, dtype=torch.uint8, device=inst.device) if state is None else state
        victim = torch.empty(nr, dtype=torch.int32, device=inst.device) if victim is None else victim
        prm = self._params(**params)
        self._check(_lib.ffs_evict_step(self._h, _ptr(inst), _ptr(tick_off), _ptr(now_us), int(now_us.numel()),
                                        C.byref(prm), _ptr(score), _ptr(state), _ptr(req), _ptr(slo), _ptr(req_tick),
                                        _ptr(load_off), nr, _ptr(victim), _stream(stream)))
        return score, state, victim

    # ---- NEXT-2: joint commit -------------------------------------------------
    def plan_joint(self, req, slo, k_max: int, out=None, stream=None):
        """Jointly feasible plans of the batch; returns (plans, rounds).  Synchronous."""
        import torch
        n = int(slo.numel())
        if out is None:
            out = torch.empty((n, PLAN_DTYPE.itemsize), dtype=torch.uint8, device=slo.device)
        rounds = C.c_uint32()
        self._check(_lib.ffs_plan_joint(self._h, _ptr(req), _ptr(slo), n, int(k_max), _ptr(out), C.byref(rounds),
                                        _stream(stream)))
        return out, int(rounds.value)

    # ---- NEXT-4: time-sharing simulator ------------------------------------------
    def simulate(self, trace, thr_pct: int = 30, cold_after_us: int = 600_000_000, k_max: int | None = None,
                 stream=None):
        """Run the simulator on a workload.SimTrace whose problem is staged; k_max = pipeline
        search depth (default the problem's; 0 = monolithic instances only).  Returns device
        tensors (ctr[N, 12], slice[N, F], state[N, F], last_used[N, F], busy[N, F], stages[N, F])."""
        import torch
        prob = trace.problem
        N, F = int(prob.n_nodes), int(prob.comp_off.shape[0] - 1)
        K = int(prob.k_max if k_max is None else k_max)
        dev = torch.device("cuda", self.device)
        t = lambda a: torch.from_numpy(np.ascontiguousarray(a).view(np.int32)).to(dev)
        off, fu, bu = t(trace.req_off), t(trace.req_func), t(trace.req_budget)
        ctr = torch.zeros((N, 12), dtype=torch.int64, device=dev)
        sl = torch.empty((N, F), dtype=torch.int32, device=dev)
        st = torch.empty((N, F), dtype=torch.uint8, device=dev)
        last = torch.empty((N, F), dtype=torch.int64, device=dev)
        busy = torch.empty((N, F), dtype=torch.int32, device=dev)
        stages = torch.empty((N, F), dtype=torch.uint8, device=dev)
        self._check(_lib.ffs_simulate(self._h, _ptr(off), _ptr(fu), _ptr(bu), int(trace.T), int(trace.t0_us),
                                      int(trace.tick_us), int(trace.window_ticks), int(thr_pct), int(cold_after_us),
                                      K, _ptr(ctr), _ptr(sl), _ptr(st), _ptr(last), _ptr(busy), _ptr(stages),
                                      _stream(stream)))
        return ctr, sl, st, last, busy, stages

    # ---- NEXT-2: routing ------------------------------------------------------------
    def route(self, req, slo, inst, state, lat_us, capacity, route=None, stream=None):
        import torch
        n = int(slo.numel())
        n_inst = int(inst.numel() // W.INST_DTYPE.itemsize)
        route = torch.empty(n, dtype=torch.int32, device=slo.device) if route is None else route
        self._check(_lib.ffs_route(self._h, _ptr(req), _ptr(slo), n, _ptr(inst), _ptr(state), _ptr(lat_us),
                                   _ptr(capacity), n_inst, _ptr(route), _stream(stream)))
        return route

    # ---- NEXT-3: frontier precompute ---------------------------------------------------------
    def frontier_build(self, k_max: int, stream=None) -> tuple[int, int]:
        """Build every (function, node free-vector) frontier; returns (groups, rounds)."""
        g, r = C.c_uint32(), C.c_uint32()
        self._check(_lib.ffs_frontier_build(self._h, int(k_max), C.byref(g), C.byref(r), _stream(stream)))
        return int(g.value), int(r.value)

    def plan_frontier(self, req, slo, out=None, stream=None):
        import torch
        n = int(slo.numel())
        if out is None:
            out = torch.empty((n, PLAN_DTYPE.itemsize), dtype=torch.uint8, device=slo.device)
        self._check(_lib.ffs_plan_frontier(self._h, _ptr(req), _ptr(slo), n, _ptr(out), _stream(stream)))
        return out

    def plan_frontier_any(self, req, slo, out=None, node=None, stream=None):
        """NEXT-2 any-invoker planning (R39): (plans, serving node int32 or -1)."""
        import torch
        n = int(slo.numel())
        if out is None:
            out = torch.empty((n, PLAN_DTYPE.itemsize), dtype=torch.uint8, device=slo.device)
        if node is None:
            node = torch.empty(n, dtype=torch.int32, device=slo.device)
        self._check(_lib.ffs_plan_frontier_any(self._h, _ptr(req), _ptr(slo), n, _ptr(out), _ptr(node),
                                               _stream(stream)))
        return out, node

    # ---- NEXT-1: ranked first-fit -----------------------------------------------
    def rank_partitions(self, k_max: int, p_ref: int) -> None:
        self._check(_lib.ffs_rank_partitions(self._h, int(k_max), int(p_ref)))

    def plan_ranked(self, req, slo, out=None, stream=None):
        import torch
        n = int(slo.numel())
        if out is None:
            out = torch.empty((n, PLAN_DTYPE.itemsize), dtype=torch.uint8, device=slo.device)
        self._check(_lib.ffs_plan_ranked(self._h, _ptr(req), _ptr(slo), n, _ptr(out), _stream(stream)))
        return out

    # ---- NEXT-1: DAG stages (R40-R43) ---------------------------------------------------------
    def stage_dag(self, dag, k_max: int) -> None:
        """Stage the unit structure (workload.DagTable: unit_off, unit_nb, unit_bend[U, 4])."""
        uo = np.ascontiguousarray(dag.unit_off, dtype=np.uint32)
        nb = np.ascontiguousarray(dag.unit_nb, dtype=np.uint8)
        be = np.ascontiguousarray(dag.unit_bend, dtype=np.uint8)
        cond = getattr(dag, "unit_cond", None)
        cd = None if cond is None else np.ascontiguousarray(cond, dtype=np.uint8)
        t = _DagTable(int(uo.shape[0] - 1), _host(uo), _host(nb), _host(be), _host(cd) if cd is not None else None)
        self._check(_lib.ffs_dag_stage(self._h, C.byref(t), int(k_max)))

    def plan_dag(self, req, slo, out=None, checks=None, stream=None):
        """Plans of DAG functions: (R, 88) uint8 device tensor of ffs_dag_plan records."""
        import torch
        n = int(slo.numel())
        if out is None:
            out = torch.empty((n, DAG_PLAN_DTYPE.itemsize), dtype=torch.uint8, device=slo.device)
        self._check(_lib.ffs_plan_dag(self._h, _ptr(req), _ptr(slo), n, _ptr(out), _ptr(checks), _stream(stream)))
        return out

    # ---- measurement ---------------------------------------------------------------------
    def int_peak(self) -> tuple[float, float]:
        ops, sec = C.c_double(), C.c_double()
        self._check(_lib.ffs_bench_int_peak(self._h, C.byref(ops), C.byref(sec)))
        return ops.value, sec.value

    def segment_times(self) -> list[float]:
        """Device ms of each search segment (ks = 1..8) of the last plan_keys call."""
        ms = (C.c_float * 8)()
        self._check(_lib.ffs_segment_times(self._h, ms))
        return [float(x) for x in ms]

    def packed_peak(self, mode: int = 1) -> tuple[float, float]:
        """(lane-instructions/s, seconds) of the packed f16x2 microbenchmark (0: HFMA2 only,
        1: HFMA2 interleaved with packed max / LOP3)."""
        v, sec = C.c_double(), C.c_double()
        self._check(_lib.ffs_bench_packed_peak(self._h, int(mode), C.byref(v), C.byref(sec)))
        return v.value, sec.value

    def set_search_mode(self, mode: int) -> None:
        """SEARCH_BOUNDED (default) or SEARCH_EXHAUSTIVE (every candidate scored)."""
        self._check(_lib.ffs_set_search_mode(self._h, int(mode)))

    def live_records(self) -> list[int]:
        """Live (request, mask pair) records of the bounded mode's compaction per ks."""
        v = (C.c_uint64 * 8)()
        self._check(_lib.ffs_search_live_records(self._h, v))
        return [int(x) for x in v]

    def scored(self) -> list[int]:
        """Candidates scored per stage count (ks = 1..8) by the last plan_keys call."""
        v = (C.c_uint64 * 8)()
        self._check(_lib.ffs_search_scored(self._h, v))
        return [int(x) for x in v]

    def filter_misses(self) -> int:
        v = C.c_uint64()
        self._check(_lib.ffs_debug_filter_misses(self._h, C.byref(v)))
        return int(v.value)


def plans_to_numpy(plans) -> np.ndarray:
    """View a (R, 80) uint8 tensor/array of ffs_plan records as a PLAN_DTYPE array."""
    a = plans.cpu().numpy() if hasattr(plans, "cpu") else np.asarray(plans)
    return np.ascontiguousarray(a).view(PLAN_DTYPE).reshape(-1)


def dag_plans_to_numpy(plans) -> np.ndarray:
    """View a (R, 88) uint8 tensor/array of ffs_dag_plan records as a DAG_PLAN_DTYPE array."""
    a = plans.cpu().numpy() if hasattr(plans, "cpu") else np.asarray(plans)
    return np.ascontiguousarray(a).view(DAG_PLAN_DTYPE).reshape(-1)


def to_device(prob, device="cuda"):
    """Requests and budgets of a Problem as device tensors (req: uint8 [R, 8], slo: int32 [R])."""
    import torch
    req = torch.from_numpy(np.ascontiguousarray(prob.req).view(np.uint8).reshape(-1, 8)).to(device)
    slo = torch.from_numpy(np.ascontiguousarray(prob.slo_us).view(np.int32)).to(device)
    return req, slo
