"""Driver for ncu captures of the search kernels (not a benchmark): stage a config, run
ffs_plan_keys `--calls` times in the given mode.  Example (the KS = 4 launch of the first
call is the 4th k_plan_search launch):

    ncu --set full --import-source on -k regex:k_plan_search --launch-skip 3 --launch-count 1 \
        -o gpurun_out/prof python tools/prof_search.py --mode exhaustive
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from paper_conf_hpdc_hui0s25_b200 import ffs, workload as W  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=5)
ap.add_argument("--mode", default="exhaustive", choices=["exhaustive", "bounded"])
ap.add_argument("--calls", type=int, default=1)
ap.add_argument("--slice", type=int, default=1, help="plan the first 1/SLICE of the requests (a request shard)")
a = ap.parse_args()
prob = W.CONFIGS[a.config]()
pl = ffs.Planner(0)
pl.stage(prob)
pl.set_search_mode(ffs.SEARCH_EXHAUSTIVE if a.mode == "exhaustive" else ffs.SEARCH_BOUNDED)
req, slo = ffs.to_device(prob)
hi = prob.R // a.slice
for _ in range(a.calls):
    keys = pl.plan_keys(req[:hi], slo[:hi], prob.k_max)
torch.cuda.synchronize()
print("segments ms", pl.segment_times()[:prob.k_max], "scored", pl.scored()[:prob.k_max])
