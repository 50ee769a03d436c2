"""C4 step time for libffs builds with different k_evict_ticks CTA shapes (FFS_LIB)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import bench
from paper_conf_hpdc_hui0s25_b200 import ffs
pl = ffs.Planner(0)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
r = bench.run_c4(pl, 20, 5, flush, {"hbm_gbs": 6552.6})
print(os.environ.get("FFS_LIB"), "step_ms", r["ms_per_step"], "score_ms", r["kernels_ms"], "frac", r["roofline"]["frac"],
      "step_frac", r["roofline"]["step_frac"])
