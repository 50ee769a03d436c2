"""Single-GPU emulation of the N-GPU step: every rank's share of the C5
step timed one after another on one B200 with CUDA events (L2 flushed before each).

shard "requests" (dist.plan_step default at C5): rank g plans its contiguous request slice
end to end (count + scan, every segment, decode) -- no collective; the projection is the
max over ranks of those device times.
shard "candidates": for k = 1..K, shard g of segment k continuing from the keys combined
over all shards of the earlier segments (the all_reduce MIN, done here outside the timed
regions), then decode of slice g; the projection adds K all-reduces of the 8 MiB key array
modelled at the guide's measured 8-rank NVLink bus bandwidth (725 GB/s,
B200_PROFILING.md): t = 2 (N-1)/N x bytes / busbw per all-reduce.

Both search modes: exhaustive (the benchmark headline) and bounded (production); the
bounded request shards also replayed from a CUDA graph per rank (dist.capture_graph).
Output: gpurun_out/shard_emulation.json.

    python tools/shard_emulation.py
"""
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_hpdc_hui0s25_b200 import dist, ffs, workload as W  # noqa: E402

BUSBW = 725e9  # B/s, 8-rank NCCL all-reduce bus bandwidth (B200_PROFILING.md)


def main():
    prob = W.config5()
    pl = ffs.Planner(0)
    pl.stage(prob)
    req, slo = ffs.to_device(prob)
    R, K = prob.R, prob.k_max
    keys = torch.empty(R, dtype=torch.int64, device="cuda")
    plans = torch.empty((R, 80), dtype=torch.uint8, device="cuda")
    flush = torch.empty(256 * 2**20, dtype=torch.uint8, device="cuda")
    out = {"workload": "C5", "R": R, "busbw_model_Bps": BUSBW, "runs": {}}

    def timed(fn, it):
        flush.fill_(it)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        return a.elapsed_time(b)

    def median3(fn):  # one warm-up run, then the median of three timed runs
        timed(fn, 0)
        return sorted(timed(fn, it) for it in range(1, 4))[1]

    for mode_name, mode in (("exhaustive", ffs.SEARCH_EXHAUSTIVE), ("bounded", ffs.SEARCH_BOUNDED)):
        pl.set_search_mode(mode)
        for shard in ("requests", "requests+graph", "candidates"):
            if shard != "requests" and mode_name == "exhaustive":
                continue
            res, base = {}, None
            for G in (1, 2, 4, 8):
                times = []
                if shard.startswith("requests") or G == 1:
                    for g in range(G):
                        lo, hi = dist.request_slice(R, g, G)

                        def fn():
                            pl.plan_keys(req[lo:hi], slo[lo:hi], K, keys=keys[lo:hi])
                            pl.plan_decode(req[lo:hi], slo[lo:hi], keys[lo:hi], K, out=plans[lo:hi])
                        if shard == "requests+graph":  # the rank's step replayed from a CUDA graph
                            graph = dist.capture_graph(fn)
                            times.append(median3(graph.replay))
                        else:
                            times.append(median3(fn))
                    coll = 0.0
                else:
                    combs = []  # keys after segments 1..k combined over all shards
                    part = torch.empty((G, R), dtype=torch.int64, device="cuda")
                    for k in range(1, K + 1):
                        for g in range(G):
                            if k > 1:
                                part[g].copy_(combs[-1])
                            pl.plan_keys_range(req, slo, K, k, k, g, G, keys=part[g])
                        combs.append(part.min(dim=0).values)
                    for g in range(G):
                        lo, hi = dist.request_slice(R, g, G)

                        def fn():
                            for k in range(1, K + 1):
                                if k > 1:
                                    keys.copy_(combs[k - 2])  # (copy inside the region: over-counts slightly)
                                pl.plan_keys_range(req, slo, K, k, k, g, G, keys=keys)
                            pl.plan_decode(req[lo:hi], slo[lo:hi], keys[lo:hi], K)
                        times.append(median3(fn))
                    coll = K * 2 * (G - 1) / G * R * 8 / BUSBW * 1e3
                mx = max(times) + coll
                base = base or mx
                res[G] = {"ms_per_rank": times, "modelled_allreduce_ms": coll, "max_ms": mx,
                          "projected_speedup": base / mx, "projected_efficiency": base / mx / G}
                print(mode_name, shard, G, f"max {mx:.3f} ms  speedup {base / mx:.2f}",
                      [f"{t:.3f}" for t in times], flush=True)
            out["runs"][f"{mode_name}/{shard}"] = res
    pl.set_search_mode(ffs.SEARCH_BOUNDED)
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    with open(os.path.join(ROOT, "gpurun_out", "shard_emulation.json"), "w") as fh:
        json.dump(out, fh, indent=1)


if __name__ == "__main__":
    main()
