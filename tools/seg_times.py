"""Per-stage-count segment times (ms) of ffs_plan_keys on a config (design input: compare
experiment builds of libffs.so via FFS_LIB).  python tools/seg_times.py [config] [reps]"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_hpdc_hui0s25_b200 import ffs, workload as W  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 5
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
prob = {2: W.config2, 3: W.config3, 5: W.config5}[cfg]()
pl = ffs.Planner(0)
pl.stage(prob)
req, slo = ffs.to_device(prob)
keys = torch.empty(prob.R, dtype=torch.int64, device="cuda")
pl.plan_keys(req, slo, prob.k_max, keys=keys)
torch.cuda.synchronize()
ref = keys.clone()
best = None
for _ in range(reps):
    pl.plan_keys(req, slo, prob.k_max, keys=keys)
    torch.cuda.synchronize()
    ms = pl.segment_times()
    best = ms if best is None else [min(a, b) for a, b in zip(best, ms)]
    assert torch.equal(keys, ref)
if best is None:
    best = pl.segment_times()
lib = os.path.basename(os.environ.get("FFS_LIB", "libffs.so"))
print(f"{lib}: C{cfg} segment ms " + " ".join(f"KS{k + 1}={t:.2f}" for k, t in enumerate(best) if t > 0)
      + f"  total={sum(best):.2f}")
pl.close()
