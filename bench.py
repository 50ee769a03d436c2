"""Benchmark of the batched pipeline-construction search (BASELINE.json metric:
candidates scored/s and plans/s at 1/2/4/8 B200, % of the integer roofline).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ffs|reference] [--config 5]
                    [--shard requests|candidates]

One step = the whole hot path over one batch: ffs_plan_keys on this rank's shard (K0
count + scan, K1 search segments KS = 1..4) -> ffs_plan_decode of this rank's slice.
Request shards (default at C5) need no collective; candidate shards all_reduce(keys, MIN)
over NCCL after every segment.  The headline `value` is the EXHAUSTIVE mode (every
candidate of every request scored, device counters prove the count); the production
(bounded) mode -- same keys -- is reported as plans/s under "production".  Inputs are
resident in HBM when the timed region starts; L2 is flushed (256 MiB write) between timed
steps, outside the events.  Each step is timed with CUDA events on the launching stream;
ranks report the max.  The roofline peak is the issue-limited packed rate (unit counts x the SM
clock measured during the timed region); microbenchmarks measured in the same run are reported.
`--impl reference` times the CPU oracle (oracle/, the plain brute force) on a bounded
sample of the same workload on this box's host cores (rank 0 only).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time
from math import comb

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from paper_conf_hpdc_hui0s25_b200 import workload as W  # noqa: E402

ALG_OPS = 5  # hoisted per-candidate ops of A3-A5: add, fma, add (balance), SLO compare, argmin flag
P = 5


def candidates_per_request(prob, k_max):
    n = prob.chain_len()
    S = np.array([sum(comb(int(m) - 1, k - 1) * P ** k for k in range(1, min(int(m), k_max) + 1)) for m in n],
                 dtype=np.int64)
    return S[prob.req["func"]]


def _traffic(kernel):
    """dram read+write bytes per launch of `kernel` from the committed ncu capture, or None."""
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as fh:
            return json.load(fh).get(kernel)
    except OSError:
        return None


def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as fh:
            return json.load(fh)
    except OSError:
        return {}


class Clocks:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""

    def __init__(self, index: int):
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
             "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--id={index}", f"--query-gpu={q}", "--format=csv,noheader,nounits",
                                       "-lms", "100"], stdout=self.f, stderr=subprocess.DEVNULL)
        except OSError:
            self.p = None

    def stop(self):
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.p.terminate()
        self.p.wait()
        self.f.flush()
        rows = [r.split(",") for r in open(self.f.name).read().strip().splitlines() if r.count(",") >= 8]
        os.unlink(self.f.name)
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"]}
        sm = [float(r[1]) for r in rows]
        mx = max(float(r[2]) for r in rows)
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in rows for i in range(4) if r[5 + i].strip() == "Active"})
        loaded = [s for s in sm if s > 0.5 * mx] or sm
        return {"sm_mhz": statistics.median(loaded), "sm_max_mhz": mx, "reasons": reasons, "samples": len(rows)}


def cpu_baseline(prob, k_max, budget_s=30.0):
    """The oracle as it stands, on a bounded sample (every s-th request), all host cores."""
    import oracle
    cores = os.cpu_count() or 1
    S = candidates_per_request(prob, k_max)
    # calibrate on a small strided sample, then size the sample for ~budget_s (the small
    # calibration sample parallelises poorly, so the real sample runs ~3x faster: ~10 s)
    idx = np.arange(0, prob.R, max(1, prob.R // 64))
    t = time.perf_counter()
    oracle.plan(prob.subset(idx), k_max=k_max, threads=cores, checks=False)
    rate = S[idx].sum() / (time.perf_counter() - t)
    want = rate * budget_s
    stride = max(1, int(S.sum() / max(want, 1.0)))
    idx = np.arange(0, prob.R, stride)
    t = time.perf_counter()
    oracle.plan(prob.subset(idx), k_max=k_max, threads=cores, checks=False)
    dt = time.perf_counter() - t
    return {"value": float(S[idx].sum() / dt), "unit": "candidates/s", "cores": cores, "kind": "oracle",
            "sample": f"every {stride}th request of {prob.name} ({len(idx)} requests, {int(S[idx].sum())} "
                      f"candidates) in {dt:.1f} s", "plans_per_s": len(idx) / dt}


def run_reference(args, prob):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import oracle
    cores = os.cpu_count() or 1
    S = candidates_per_request(prob, prob.k_max)
    # per step: a bounded sample sized so the whole run stays within a few minutes
    n_steps = args.steps + args.warmup
    idx0 = np.arange(0, prob.R, max(1, prob.R // 64))
    t = time.perf_counter()
    oracle.plan(prob.subset(idx0), threads=cores, checks=False)
    rate = S[idx0].sum() / (time.perf_counter() - t)
    per_step = min(20.0, 150.0 / max(n_steps, 1))
    stride = max(1, int(S.sum() / (rate * per_step)))
    times, cands, plans = [], 0, 0
    for s in range(n_steps):
        idx = np.arange(s % stride, prob.R, stride)
        t = time.perf_counter()
        oracle.plan(prob.subset(idx), threads=cores, checks=False)
        dt = time.perf_counter() - t
        if s >= args.warmup:
            times.append(dt)
            cands += int(S[idx].sum())
            plans += len(idx)
    tot = sum(times)
    v = cands / tot
    line = {"metric": "candidates_scored_per_s", "value": v, "unit": "candidates/s", "impl": "reference",
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * tot / len(times),
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "exact u64/u128 integers (oracle)",
            "data": "synthetic", "plans_per_s": plans / tot,
            "config": {"workload": prob.meta["workload"], "R": prob.R, "k_max": prob.k_max},
            "cpu_baseline": {"value": v, "unit": "candidates/s", "cores": cores, "kind": "oracle",
                             "sample": f"every {stride}th request (offset by step) of {prob.name}"},
            "e2e": {"value": v, "unit": "candidates/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def run_c4(pl, steps: int, warmup: int, flush, peaks):
    """C4: hotness-aware eviction over T = 4096 tick snapshots of a 32-node
    (256-GPU) cluster, 200 warm functions -- one step = ffs_evict_step: every instance of
    every tick scored (A7) and the victim of every load (A8), fused (one pass over the
    instances builds each tick's (node, profile) minima in shared memory and picks the
    victims of the tick's loads from them: one launch).
    Reported against the HBM roofline: 33 algorithmic bytes per score (24 B record in, 8 B
    score + 1 B state out), for the scoring kernel and for the whole step."""
    import torch
    wl = W.config4()
    prob = wl.problem
    pl.stage(prob)
    inst = torch.from_numpy(wl.inst.view(np.uint8)).cuda()
    toff = torch.from_numpy(wl.tick_off.view(np.int32)).cuda()
    now = torch.from_numpy(wl.now_us.view(np.int64)).cuda()
    req = torch.from_numpy(np.ascontiguousarray(prob.req).view(np.uint8).reshape(-1, 8)).cuda()
    slo = torch.from_numpy(prob.slo_us.view(np.int32)).cuda()
    # the C4 loads arrive tick by tick: grouped (CSR offsets per tick), so the victims are
    # picked inside each tick's CTA
    load_off = torch.from_numpy(np.searchsorted(wl.req_tick, np.arange(len(wl.now_us) + 1)).astype(np.int32)).cuda()
    n = int(wl.inst.shape[0])
    score = torch.empty(n, dtype=torch.int64, device="cuda")
    state = torch.empty(n, dtype=torch.uint8, device="cuda")
    vic = torch.empty(prob.R, dtype=torch.int32, device="cuda")
    stream = torch.cuda.current_stream()

    def step():
        pl.evict_step(inst, toff, now, req, slo, load_off=load_off, score=score, state=state, victim=vic,
                      window_us=wl.window_us)

    for _ in range(warmup):
        step()
    torch.cuda.synchronize()
    ev = [[torch.cuda.Event(enable_timing=True) for _ in range(2)] for _ in range(steps)]
    for i in range(steps):
        flush.fill_(i & 0xFF)
        ev[i][0].record(stream)
        step()
        ev[i][1].record(stream)
    torch.cuda.synchronize()
    t_step = sum(e[0].elapsed_time(e[1]) for e in ev) / steps
    # the scoring pass alone (same kernel without the table), for the kernel-level roofline
    for i in range(steps):
        flush.fill_(i & 0xFF)
        ev[i][0].record(stream)
        pl.evict_scores_ticks(inst, toff, now, score=score, state=state, window_us=wl.window_us)
        ev[i][1].record(stream)
    torch.cuda.synchronize()
    t_sc = sum(e[0].elapsed_time(e[1]) for e in ev) / steps
    peak = float(peaks.get("hbm_gbs", 6650.0))
    achieved = 33.0 * n / (t_sc * 1e-3) / 1e9
    step_gbs = 33.0 * n / (t_step * 1e-3) / 1e9
    return {"metric": "eviction_scores_per_s", "value": n / (t_step * 1e-3), "unit": "scores/s",
            "ms_per_step": t_step, "scores_per_step": n, "loads_per_step": int(prob.R),
            "workload": f"C4: 32 nodes (712 slices), 200 functions, {len(wl.now_us)} ticks x "
                        f"{n // len(wl.now_us)} instances, victims for {prob.R} loads (ffs_evict_step, fused)",
            "kernels_ms": {"k_evict_ticks (scores only)": t_sc},
            "roofline": {"bound": "hbm", "kernel": "k_evict_ticks", "achieved": achieved, "peak": peak,
                         "unit": "GB/s", "frac": achieved / peak, "traffic": _traffic("k_evict_ticks"),
                         "alg_bytes_per_score": 33, "peak_source": "MEASURED_PEAKS.json hbm_gbs (copy)",
                         "step_achieved": step_gbs, "step_frac": step_gbs / peak},
            "l2": "flushed between steps"}


def run_ranked(pl, prob, req, slo, steps: int, warmup: int, flush):
    """NEXT-1 (the paper's literal offline-CV ranked first-fit) on the same batch:
    plans/s of ffs_plan_ranked (the offline ranking is done once, outside the timing)."""
    import torch
    t0 = time.perf_counter()
    pl.rank_partitions(prob.k_max, int(np.argmax(prob.gpcs)))
    rank_s = time.perf_counter() - t0
    out = torch.empty((prob.R, 80), dtype=torch.uint8, device="cuda")
    for _ in range(warmup):
        pl.plan_ranked(req, slo, out=out)
    torch.cuda.synchronize()
    stream = torch.cuda.current_stream()
    ms = 0.0
    for i in range(steps):
        flush.fill_(i & 0xFF)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        pl.plan_ranked(req, slo, out=out)
        b.record(stream)
        torch.cuda.synchronize()
        ms += a.elapsed_time(b)
    from paper_conf_hpdc_hui0s25_b200 import ffs
    p = ffs.plans_to_numpy(out)
    return {"metric": "ranked_first_fit_plans_per_s", "value": prob.R * steps / (ms * 1e-3), "unit": "plans/s",
            "ms_per_step": ms / steps, "offline_rank_s": rank_s,
            "ok_frac": float((p["status"] == 0).mean()), "multi_stage_frac": float(((p["status"] == 0) & (p["k"] > 1)).mean())}


def run_dag(pl, steps: int, warmup: int, flush):
    """NEXT-1 DAG stages (R40-R43) on the CD workload (32 DAG functions on the C3 cluster,
    65,536 requests): candidates/s and plans/s of ffs_plan_dag (one warp per request, exact
    integer scoring).  Stages its own tables; run after the C5 legs."""
    import torch
    from paper_conf_hpdc_hui0s25_b200 import ffs
    prob, dag = W.dag_config()
    pl.stage(prob)
    pl.stage_dag(dag, prob.k_max)
    req, slo = ffs.to_device(prob)
    out = torch.empty((prob.R, ffs.DAG_PLAN_DTYPE.itemsize), dtype=torch.uint8, device="cuda")
    checks = torch.zeros((prob.R, 3), dtype=torch.int64, device="cuda")
    pl.plan_dag(req, slo, out=out, checks=checks)  # candidate count (checksums), untimed
    torch.cuda.synchronize()
    cands = int(checks[:, 0].sum().item())
    for _ in range(warmup):
        pl.plan_dag(req, slo, out=out)
    torch.cuda.synchronize()
    stream = torch.cuda.current_stream()
    ms = 0.0
    for i in range(steps):
        flush.fill_(i & 0xFF)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        pl.plan_dag(req, slo, out=out)
        b.record(stream)
        torch.cuda.synchronize()
        ms += a.elapsed_time(b)
    p = ffs.dag_plans_to_numpy(out)
    return {"metric": "dag_candidates_scored_per_s", "value": cands * steps / (ms * 1e-3), "unit": "candidates/s",
            "plans_per_s": prob.R * steps / (ms * 1e-3), "ms_per_step": ms / steps, "candidates_per_step": cands,
            "workload": "CD: 32 DAG functions (3-8 units, 2-branch blocks p=0.35), C3 cluster, R=65536, K=4",
            "ok_frac": float((p["status"] == 0).mean()), "split_frac": float((p["split_mask"] > 0).mean())}


def run_joint(pl, prob, req, slo):
    """NEXT-2 (joint commit in adjusted-deadline order) on the same batch:
    one call, wall/event time, rounds."""
    import torch
    out = torch.empty((prob.R, 80), dtype=torch.uint8, device="cuda")
    pl.plan_joint(req, slo, prob.k_max, out=out)  # warm-up
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    _, rounds = pl.plan_joint(req, slo, prob.k_max, out=out)
    b.record()
    torch.cuda.synchronize()
    ms = a.elapsed_time(b)
    from paper_conf_hpdc_hui0s25_b200 import ffs
    p = ffs.plans_to_numpy(out)
    return {"metric": "joint_commit_plans_per_s", "value": prob.R / (ms * 1e-3), "unit": "plans/s", "ms": ms,
            "rounds": rounds, "ok_frac": float((p["status"] == 0).mean())}


def run_frontier(pl, prob, req, slo, steps: int, warmup: int, flush):
    """NEXT-3 (frontier precompute): build every (function, node free-vector) frontier once,
    then answer the batch by binary search; plans identical to the argmin path."""
    import torch
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    groups, rounds = pl.frontier_build(prob.k_max)
    build_s = time.perf_counter() - t0
    out = torch.empty((prob.R, 80), dtype=torch.uint8, device="cuda")
    for _ in range(warmup):
        pl.plan_frontier(req, slo, out=out)
    stream = torch.cuda.current_stream()
    ms = 0.0
    for i in range(steps):
        flush.fill_(i & 0xFF)
        a.record(stream)
        pl.plan_frontier(req, slo, out=out)
        b.record(stream)
        torch.cuda.synchronize()
        ms += a.elapsed_time(b)
    # NEXT-2 any-invoker planning (R39) from the same frontiers: every request considers
    # every node of the cluster (one warp per request over the free-vector classes)
    node = torch.empty(prob.R, dtype=torch.int32, device="cuda")
    for _ in range(warmup):
        pl.plan_frontier_any(req, slo, out=out, node=node)
    ms_any = 0.0
    for i in range(steps):
        flush.fill_(i & 0xFF)
        a.record(stream)
        pl.plan_frontier_any(req, slo, out=out, node=node)
        b.record(stream)
        torch.cuda.synchronize()
        ms_any += a.elapsed_time(b)
    st = out.view(-1, 80)[:, 8:12].contiguous().view(torch.int32)
    ok_any = int(torch.count_nonzero(st == 0))
    home = req.view(-1, 8)[:, 4:8].contiguous().view(torch.int32).view(-1)
    away = int(torch.count_nonzero((node >= 0) & (node != home)))
    return {"metric": "frontier_plans_per_s", "value": prob.R * steps / (ms * 1e-3), "unit": "plans/s",
            "query_ms_per_step": ms / steps, "build_s": build_s, "groups": groups, "rounds": rounds,
            "note": "plans identical to the argmin path; candidates are scored once per frontier point and group, "
                    "not per request (not comparable to candidates/s)",
            "any_invoker": {"metric": "any_invoker_plans_per_s", "value": prob.R * steps / (ms_any * 1e-3),
                            "unit": "plans/s", "query_ms_per_step": ms_any / steps, "ok": ok_any,
                            "served_away_from_home": away}}


def run_sim(pl):
    """NEXT-4: the time-sharing simulator on the C4 cluster, 8192 ticks (13.7 simulated
    minutes, so 10-minute cold terminations occur); one kernel, device-timed."""
    import torch
    tr = W.sim_trace(T=8192)
    pl.stage(tr.problem)
    pl.simulate(tr)  # warm-up
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    ctr, *_ = pl.simulate(tr)
    b.record()
    torch.cuda.synchronize()
    ms = a.elapsed_time(b)
    c = ctr.cpu().numpy().sum(axis=0)
    # the same trace with monolithic instances only (no pipelines, R44-R46 off): the
    # FluidFaaS mechanism's effect on the simulated SLO hit rate
    c0 = pl.simulate(tr, k_max=0)[0].cpu().numpy().sum(axis=0)
    return {"metric": "simulated_requests_per_s", "value": float(c[0]) / (ms * 1e-3), "unit": "requests/s",
            "ms": ms, "ticks": tr.T, "nodes": int(tr.problem.n_nodes), "functions": int(tr.problem.F),
            "requests": int(c[0]), "served": int(c[1]), "slo_hit_rate": float(c[2]) / max(1, int(c[0])),
            "reloads": int(c[4]), "evictions": int(c[5]), "cold_terminations": int(c[6]),
            "slice_ticks_occupied": int(c[7]), "pipelines_placed": int(c[8]), "pipeline_migrations": int(c[9]),
            "served_by_pipelines": int(c[10]), "pipeline_slice_ticks": int(c[11]),
            "monolithic_only": {"served": int(c0[1]), "slo_hit_rate": float(c0[2]) / max(1, int(c0[0])),
                                "evictions": int(c0[5])}}


def measure_peaks(pl):
    """Roofline denominators measured on this GPU, in this run: K5 (integer
    IADD3/LOP3/IMAD mix) and the packed f16x2 microbenchmarks (HFMA2 alone = FMA-pipe rate;
    HFMA2 interleaved 1:1 with packed max / LOP3 = issue-limited rate).  Each: ~100 ms of
    warm-up launches (clock ramp from idle), then 16 timed launches."""
    int_ops = pl.int_peak()[0]
    fma = pl.packed_peak(0)[0]
    mix = max(pl.packed_peak(m)[0] for m in (1, 2))
    return {"int32_ops_per_s": int_ops, "hfma2_lane_instr_per_s": fma, "issue_lane_instr_per_s": mix,
            "packed_ops_per_s": 2.0 * max(fma, mix)}


def winner_histogram(p, slo):
    """Winner histogram of one step's plans (printed with every run)."""
    st = p["status"]
    ok = st == 0
    ks = np.bincount(p["k"][ok].astype(np.int64), minlength=9)[1:]
    prof = np.zeros(5, dtype=np.int64)
    for i in range(8):
        sel = ok & (p["k"] > i)
        prof += np.bincount(p["prof"][sel, i].astype(np.int64), minlength=5)[:5]
    n = max(1, len(st))
    return {"requests": int(len(st)), "ok_frac": float(ok.mean()) if len(st) else 0.0,
            "infeasible_frac": float((st == 1).sum() / n), "bad_req_frac": float((st == 2).sum() / n),
            "one_stage_frac": float((ok & (p["k"] == 1)).sum() / n),
            "multi_stage_frac": float((ok & (p["k"] > 1)).sum() / n),
            "k_hist": {str(k + 1): int(v) for k, v in enumerate(ks) if v},
            "stage_profile_hist": dict(zip(["1g", "2g", "3g", "4g", "7g"], map(int, prof)))}


def timed_steps(step, steps, flush, stream, barrier, pl=None):
    """Per-step CUDA events on the launching stream, L2 flushed before each step outside
    the events; returns (total ms, per-segment ms summed over the steps)."""
    import torch
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
    seg_ms = np.zeros(8)
    barrier()
    for i in range(steps):
        flush.fill_(i & 0xFF)
        ev[i][0].record(stream)
        step()
        ev[i][1].record(stream)
        if pl is not None:
            seg_ms += np.array(pl.segment_times())  # waits for this step's search segments
    barrier()
    return sum(a.elapsed_time(b) for a, b in ev), seg_ms


def graph_leg(step, args, flush, stream, barrier, max_over_ranks, keys_now, keys_ref):
    """Production step replayed from a CUDA graph: ms/step and key identity."""
    from paper_conf_hpdc_hui0s25_b200 import dist as D
    try:
        g = D.capture_graph(step)
    except Exception as e:  # noqa: BLE001 -- report, the eager numbers stand
        return {"error": f"{type(e).__name__}: {e}"[:200]}
    keys_now.fill_(0)
    for _ in range(args.warmup):
        g.replay()
    barrier()
    ms, _ = timed_steps(g.replay, args.steps, flush, stream, barrier)
    ms = max_over_ranks(ms)
    import torch
    return {"ms_per_step": ms / args.steps, "keys_identical_to_exhaustive": bool(torch.equal(keys_now, keys_ref))}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ffs", choices=["ffs", "reference"])
    ap.add_argument("--config", type=int, default=5, choices=[2, 3, 5])
    ap.add_argument("--shard", default=None, choices=[None, "requests", "candidates"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-c4", action="store_true", help="skip the C4 eviction and NEXT-row measurements")
    args = ap.parse_args()
    assert args.warmup >= 3 or args.impl == "reference", "timing rules: >= 3 warm-up steps"

    prob = W.CONFIGS[args.config]()
    desc = {2: "C2: 6 functions n in {3,3,5,6,8,12}, 1 Hybrid node (26 slices), R=4096, K=4",
            3: "C3: 20 functions n in U[3,24], 8 nodes = 64 GPUs, R=65536, K=4",
            5: "C5: 64 functions n in U[3,32], 128 nodes = 1024 GPUs, R=1048576, K=4"}
    prob.meta["workload"] = desc[args.config]
    if args.impl == "reference":
        run_reference(args, prob)
        return

    import torch
    import torch.distributed as dist
    from paper_conf_hpdc_hui0s25_b200 import ffs
    from paper_conf_hpdc_hui0s25_b200 import dist as D

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    local = local % torch.cuda.device_count()  # several ranks may share a GPU in smoke runs
    torch.cuda.set_device(local)
    backend = os.environ.get("FFS_DIST_BACKEND", "nccl")  # gloo: multi-rank smoke on one GPU
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    K = prob.k_max
    R = prob.R
    shard = args.shard or D.choose_shard(R, world)
    pl = ffs.Planner(local)
    pl.stage(prob)
    req, slo = ffs.to_device(prob)
    keys = torch.full((R,), np.iinfo(np.int64).max, dtype=torch.int64, device="cuda")
    lo, hi = D.request_slice(R, rank, world)
    plans = torch.empty((hi - lo, 80), dtype=torch.uint8, device="cuda")
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    stream = torch.cuda.current_stream()
    peaks_file = measured_peaks()
    peaks = measure_peaks(pl)  # this GPU, this run

    def step():  # this rank's shard of the batch: keys -> (exchange) -> decode of its slice
        D.plan_step(pl, req, slo, K, rank, world, keys, plans, shard=shard)

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    def max_over_ranks(x):
        if world > 1:
            t = torch.tensor([x], dtype=torch.float64, device="cuda")
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            x = float(t.item())
        return x

    # ---- headline: exhaustive mode, every candidate of every request scored ----
    pl.set_search_mode(ffs.SEARCH_EXHAUSTIVE)
    for _ in range(args.warmup):
        step()
    barrier()
    clocks = Clocks(local)
    ms, seg_ms = timed_steps(step, args.steps, flush, stream, barrier, pl)
    clk = clocks.stop()
    scored_ks = pl.scored()  # device counters of the last (identical) step
    ms = max_over_ranks(ms)
    total_cands = int(candidates_per_request(prob, K).sum())
    scored_all = sum(scored_ks)
    if world > 1:
        t = torch.tensor([sum(scored_ks)], dtype=torch.int64, device="cuda")
        dist.all_reduce(t)
        scored_all = int(t.item())
    value = scored_all * args.steps / (ms * 1e-3)
    # dominant kernel of the exhaustive step on this rank: its scored candidates x the
    # algorithmic ops per candidate over its event-timed launch duration
    top = int(np.argmax(seg_ms)) + 1
    top_ms = seg_ms[top - 1] / args.steps
    top_scored = float(scored_ks[top - 1])
    achieved = top_scored * ALG_OPS / (top_ms * 1e-3)
    traffic = _traffic(f"k_plan_search<{top}>")
    sm_count = torch.cuda.get_device_properties(local).multi_processor_count
    sm_mhz = float(clk.get("sm_mhz") or peaks_file.get("sm_max_mhz", 1965.0))
    # issue-limited peak of the packed datapath: guide unit counts (4 SMSPs
    # per SM, one warp-instruction issued per SMSP per clock, 32 lanes, two 16-bit ops per
    # packed lane-instruction) x the SM count x the SM clock measured during the timed region
    peak = sm_count * 4 * 32 * 2 * sm_mhz * 1e6
    roofline = {"bound": "alu", "kernel": f"k_plan_search<{top}>", "achieved": achieved, "peak": peak,
                "unit": "ops/s (16-bit lane ops; a packed f16x2 lane-instruction = 2)", "frac": achieved / peak,
                "traffic": traffic, "alg_ops_per_candidate": ALG_OPS, "kernel_ms": top_ms,
                "candidates_scored_per_launch": top_scored, "kernel_share_of_step": top_ms / (ms / args.steps),
                "peak_source": f"derived: {sm_count} SMs x 4 SMSP x 1 warp-instr/clk x 32 lanes x 2 ops x "
                               f"{sm_mhz:.0f} MHz (SM clock measured by nvidia-smi during this run's timed region)",
                "microbenchmarks": dict(peaks, note="measured this run (ffs_bench_packed_peak / ffs_bench_int_peak): "
                                        "HFMA2 chains reach the FMA-pipe rate (~half the issue slots); the "
                                        "interleaved mixes stay below what the search kernel itself issues, so "
                                        "they are reported, not used as the ceiling (DESIGN.md §5)"),
                "survey_basis": {"ops_per_candidate": 20, "peak": peaks["int32_ops_per_s"],
                                 "peak_source": "measured this run: K5 IADD3/LOP3/IMAD mix (ffs_bench_int_peak)",
                                 "frac": top_scored * 20 / (top_ms * 1e-3) / peaks["int32_ops_per_s"],
                                 "note": "SURVEY 8(d)'s 20 hoisted scalar int32 ops per candidate; the kernel's "
                                         "group-maximum f16x2 core decides 5 candidates of each of 2 masks with 13 "
                                         "packed instructions, so this basis exceeds 1 (DESIGN.md §5)"}}

    # ---- production: bounded mode, identical keys, plans/s -----------------------------
    pl.set_search_mode(ffs.SEARCH_BOUNDED)
    keys_ex = keys[lo:hi].clone()
    for _ in range(args.warmup):
        step()
    barrier()
    ms_b, seg_b = timed_steps(step, args.steps, flush, stream, barrier, pl)
    ms_b = max_over_ranks(ms_b)
    bounded_scored = sum(pl.scored())
    same = bool(torch.equal(keys_ex, keys[lo:hi]))
    graph = (graph_leg(step, args, flush, stream, barrier, max_over_ranks, keys[lo:hi], keys_ex)
             if shard == "requests" else None)  # (candidate shards: a collective per segment)
    hist = winner_histogram(ffs.plans_to_numpy(plans), None) if rank == 0 else None
    production = {"metric": "plans_per_s", "value": R * args.steps / (ms_b * 1e-3), "unit": "plans/s",
                  "ms_per_step": ms_b / args.steps,
                  "candidates_decided_per_s": total_cands * args.steps / (ms_b * 1e-3),
                  "candidates_scored_per_step_rank0": int(bounded_scored),
                  "segment_ms_rank0": [float(x) / args.steps for x in seg_b[:K]],
                  "keys_identical_to_exhaustive": same,
                  "cuda_graph": graph,
                  "note": "FFS_SEARCH_BOUNDED: exact integer SLO lower bounds prove candidates infeasible "
                          "without scoring them; same keys and plans as the exhaustive headline"}

    # ---- e2e through the public host-buffer API (N = 1: ffs_plan_batch_host) ------------
    e2e = None
    if not args.no_e2e:
        h_req = torch.from_numpy(np.ascontiguousarray(prob.req).view(np.uint8)).pin_memory()
        h_slo = torch.from_numpy(np.ascontiguousarray(prob.slo_us).view(np.uint8)).pin_memory()
        h_out = torch.empty((hi - lo) * 80, dtype=torch.uint8).pin_memory()
        req_np = h_req.numpy().view(W.REQ_DTYPE)
        slo_np = h_slo.numpy().view(np.uint32)
        out_np = h_out.numpy().view(ffs.PLAN_DTYPE)
        d_req = torch.empty_like(req)
        d_slo = torch.empty_like(slo)

        def e2e_step():
            if world == 1:  # the single-GPU public call: ffs_plan_batch_host
                pl.plan_batch_host(req_np, slo_np, K, out=out_np)
            else:
                D.plan_step_host(pl, h_req.view(-1, 8), h_slo.view(torch.int32), d_req, d_slo, K, rank, world,
                                 keys, plans, h_out, shard=shard)

        def e2e_run():
            for _ in range(2):
                e2e_step()
            barrier()
            t0 = time.perf_counter()
            n = max(3, args.steps // 2)
            for _ in range(n):
                e2e_step()
            barrier()
            return n, max_over_ranks(time.perf_counter() - t0)

        pl.set_search_mode(ffs.SEARCH_EXHAUSTIVE)
        n_e2e, dt = e2e_run()
        pl.set_search_mode(ffs.SEARCH_BOUNDED)
        n_b, dt_b = e2e_run()
        e2e = {"value": scored_all * n_e2e / dt, "unit": "candidates/s", "plans_per_s": R * n_e2e / dt,
               "h2d_bytes_per_step": int(D.h2d_bytes(R, rank, world, shard) if world > 1 else R * 12),
               "d2h_bytes_per_step": int((hi - lo) * 80),
               "production_plans_per_s": R * n_b / dt_b,
               "timer": "host wall clock around the blocking call, max over ranks"}

    ranked = joint = frontier = c4 = sim = dagr = None
    if world == 1 and not args.no_c4:
        ranked = run_ranked(pl, prob, req, slo, args.steps, args.warmup, flush)
        joint = run_joint(pl, prob, req, slo)
        frontier = run_frontier(pl, prob, req, slo, args.steps, args.warmup, flush)
        c4 = run_c4(pl, args.steps, args.warmup, flush, peaks_file)
        sim = run_sim(pl)
        dagr = run_dag(pl, args.steps, args.warmup, flush)
    if rank == 0:
        cpu = None
        if world == 1 and not args.no_cpu_baseline:
            cpu = cpu_baseline(prob, K)
        n_seg = min(K, int(prob.chain_len().max()))
        # exhaustive step: count + 3 scan kernels per keys call, the chain-length grouping of
        # the grouped segments (k_group_hist, 3 scan kernels, k_group_tab, k_group_scatter;
        # once per call: KS = 3, 4, and KS = 2 on >= 2^19 requests), a search kernel per
        # segment, decode
        n_rank = (hi - lo) if shard == "requests" else R
        grouped = [k for k in (2, 3, 4) if k <= n_seg and (k != 2 or n_rank >= 1 << 19)]
        if shard == "requests":
            launches_per_step = 1 + 3 + (6 if grouped else 0) + n_seg + 1
        else:
            launches_per_step = K * (1 + 3) + 6 * len(grouped) + n_seg + 1
        line = {
            "metric": "candidates_scored_per_s", "value": value, "unit": "candidates/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms / args.steps,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
            "dtype": "f16x2 pre-filter + exact u32/u64 keys",
            "data": "synthetic", "plans_per_s": R * args.steps / (ms * 1e-3),
            "config": {"workload": prob.meta["workload"], "R": R, "k_max": K, "candidates_per_step": total_cands,
                       "candidates_scored_per_step": scored_all,
                       "scored_counter_equals_sum_S": scored_all == total_cands,
                       "mode": "exhaustive (FFS_SEARCH_EXHAUSTIVE)",
                       "l2": "flushed between steps (256 MiB write, outside the events)",
                       "parallelism": (f"request shards x{world} (no data-path collective)" if shard == "requests"
                                       else f"candidate-range shards x{world} + all_reduce(MIN) over {backend}")
                       if world > 1 else "single GPU"},
            "roofline": roofline,
            "clocks": clk,
            "gpu_launches": launches_per_step * args.steps,
            "e2e": e2e,
            "cpu_baseline": cpu,
            "production": production,
            "winners": hist,
            "eviction_c4": c4,
            "ranked_first_fit": ranked,
            "joint_commit": joint,
            "frontier": frontier,
            "timeshare_sim": sim,
            "dag_stages": dagr,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
