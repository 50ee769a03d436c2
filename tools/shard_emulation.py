"""Single-GPU emulation of the N-GPU step: every rank's share of the C5
step timed one after another on one B200 with CUDA events (L2 flushed before each).
mode "exchange" (dist.plan_step): for k = 1..K, shard g of segment k continuing from the
keys combined over all shards of the earlier segments (the all_reduce, done here by
torch.minimum outside the timed regions); then decode of slice g.  mode "independent"
(the round-1 first version): shard g of all segments from scratch, then decode.  The
max over g is the device time rank-parallel hardware needs minus the all_reduce(s) of
the 8 MiB key array (not emulated: one GPU).  Output: gpurun_out/shard_emulation.json.

    python tools/shard_emulation.py
"""
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_hpdc_hui0s25_b200 import dist, ffs, workload as W  # noqa: E402


def main():
    prob = W.config5()
    pl = ffs.Planner(0)
    pl.stage(prob)
    req, slo = ffs.to_device(prob)
    keys = torch.empty(prob.R, dtype=torch.int64, device="cuda")
    flush = torch.empty(256 * 2**20, dtype=torch.uint8, device="cuda")
    K = prob.k_max
    out = {"workload": "C5", "R": prob.R, "modes": {}}

    def timed(fn, it):
        flush.fill_(it)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        return a.elapsed_time(b)

    for mode in ("independent", "exchange"):
        res, base = {}, None
        for G in (1, 2, 4, 8):
            combs = []  # keys after segments 1..k combined over all shards
            if mode == "exchange" and G > 1:
                part = torch.empty((G, prob.R), dtype=torch.int64, device="cuda")
                for k in range(1, K + 1):
                    for g in range(G):
                        if k > 1:
                            part[g].copy_(combs[-1])
                        pl.plan_keys_range(req, slo, K, k, k, g, G, keys=part[g])
                    combs.append(part.min(dim=0).values)
            times = []
            for g in range(G):
                lo, hi = dist.request_slice(prob.R, g, G)
                samples = []
                for it in range(4):  # 1 warm-up + 3 timed, keep the median
                    if mode == "exchange" and G > 1:
                        t = 0.0
                        for k in range(1, K + 1):
                            if k > 1:
                                keys.copy_(combs[k - 2])
                            t += timed(lambda: pl.plan_keys_range(req, slo, K, k, k, g, G, keys=keys), it)
                    else:
                        t = timed(lambda: pl.plan_keys(req, slo, K, g, G, keys=keys), it)
                    t += timed(lambda: pl.plan_decode(req[lo:hi], slo[lo:hi], keys[lo:hi], K), it)
                    if it:
                        samples.append(t)
                times.append(sorted(samples)[1])
            mx = max(times)
            base = base or mx
            res[G] = {"ms_per_rank": times, "max_ms": mx, "projected_speedup": base / mx,
                      "projected_efficiency": base / mx / G}
            print(mode, G, f"max {mx:.2f} ms  speedup {base / mx:.2f}", [f"{t:.2f}" for t in times], flush=True)
        out["modes"][mode] = res
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    with open(os.path.join(ROOT, "gpurun_out", "shard_emulation.json"), "w") as fh:
        json.dump(out, fh, indent=1)
    pl.close()


if __name__ == "__main__":
    main()
