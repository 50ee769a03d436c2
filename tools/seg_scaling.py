"""Per-segment device times of the C5 step on request slices of 1/G of the batch (the
request-shard rank's work), bounded and exhaustive modes: which part does not scale."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_hpdc_hui0s25_b200 import ffs, workload as W, dist
prob = W.config5()
pl = ffs.Planner(0); pl.stage(prob)
req, slo = ffs.to_device(prob)
K, R = prob.k_max, prob.R
keys = torch.empty(R, dtype=torch.int64, device="cuda")
for mode in (ffs.SEARCH_BOUNDED, ffs.SEARCH_EXHAUSTIVE):
    pl.set_search_mode(mode)
    for G in (1, 2, 4, 8, 16):
        lo, hi = dist.request_slice(R, 0, G)
        segs = []
        for it in range(4):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            pl.plan_keys(req[lo:hi], slo[lo:hi], K, keys=keys[lo:hi])
            b.record()
            c, d = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            c.record()
            pl.plan_decode(req[lo:hi], slo[lo:hi], keys[lo:hi], K)
            d.record()
            torch.cuda.synchronize()
            if it:
                segs.append([a.elapsed_time(b)] + pl.segment_times()[:K] + [c.elapsed_time(d)])
        m = np.median(np.array(segs), axis=0)
        print("mode", mode, "G", G, "keys %.3f" % m[0], "segs", " ".join("%.3f" % x for x in m[1:K + 1]), "decode %.3f" % m[-1],
              "live", pl.live_records()[:4], flush=True)
