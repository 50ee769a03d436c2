"""Small invocation of every kernel through the C ABI, run under compute-sanitizer by
tests/test_gpu_sanitizer.py (verify mode + production mode + decode + eviction)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_hpdc_hui0s25_b200 import ffs, workload as W  # noqa: E402

pl = ffs.Planner(0)
for prob in (W.config1(), W.config2(R=96)):
    pl.stage(prob)
    req, slo = ffs.to_device(prob)
    checks = torch.zeros((prob.R, 3), dtype=torch.int64, device="cuda")
    keys = pl.plan_keys(req, slo, prob.k_max, checks=checks)
    pl.plan_decode(req, slo, keys, prob.k_max)
    keys2 = pl.plan_keys(req, slo, prob.k_max, rank=1, world=3)
    pl.plan_batch(req, slo, prob.k_max)
wl = W.config4(T=4)
pl.stage(wl.problem)
inst = torch.from_numpy(wl.inst.view(np.uint8)).cuda()
toff = torch.from_numpy(wl.tick_off.view(np.int32)).cuda()
now = torch.from_numpy(wl.now_us.view(np.int64)).cuda()
score, state = pl.evict_scores_ticks(inst, toff, now)
req, slo = ffs.to_device(wl.problem)
pl.evict_victims(req, slo, torch.from_numpy(wl.req_tick.view(np.int32)).cuda(), inst, toff, score)
torch.cuda.synchronize()
print("sanitize-run ok")
