"""Per-stage-count search rates (candidates/s of each k_plan_search<KS> launch) on deep
chains with k_max = 8 (design input for the KS >= 5 path)."""
import os
import sys
from math import comb

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_hpdc_hui0s25_b200 import ffs, workload as W  # noqa: E402

rng = W.SplitMix64(99)
lengths = rng.sub(9).integers(9, 12, 16)
prob = W._problem("deep", rng, lengths, W.NODE_BLOCK, int(sys.argv[1]) if len(sys.argv) > 1 else 256, k_max=8)
pl = ffs.Planner(0)
pl.stage(prob)
req, slo = ffs.to_device(prob)
keys = torch.empty(prob.R, dtype=torch.int64, device="cuda")
for _ in range(2):
    pl.plan_keys(req, slo, 8, keys=keys)
torch.cuda.synchronize()
pl.plan_keys(req, slo, 8, keys=keys)
ms = pl.segment_times()
n = prob.chain_len()[prob.req["func"]]
for ks in range(1, 9):
    cand = sum(comb(int(m) - 1, ks - 1) * 5 ** ks for m in n if m >= ks)
    if ms[ks - 1] > 0:
        print(f"KS={ks}: {cand:.3e} candidates in {ms[ks-1]:8.2f} ms = {cand / (ms[ks-1] * 1e-3):.3e} /s")
