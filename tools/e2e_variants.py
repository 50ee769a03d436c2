"""e2e (ffs_plan_batch_host, pinned buffers) time per step of experiment builds on C5, both
search modes, and a plain 80 MiB pinned device->host copy (design input).
    python tools/e2e_variants.py exp/a.so exp/b.so"""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r"""
import sys, time
sys.path.insert(0, sys.argv[1])
import numpy as np, torch
from paper_conf_hpdc_hui0s25_b200 import ffs, workload as W
prob = W.config5()
pl = ffs.Planner(0)
pl.stage(prob)
h_req = torch.from_numpy(np.ascontiguousarray(prob.req).view(np.uint8)).pin_memory().numpy().view(W.REQ_DTYPE)
h_slo = torch.from_numpy(np.ascontiguousarray(prob.slo_us).view(np.uint8)).pin_memory().numpy().view(np.uint32)
out = torch.empty(prob.R * 80, dtype=torch.uint8).pin_memory().numpy().view(ffs.PLAN_DTYPE)
res = []
for mode in (ffs.SEARCH_EXHAUSTIVE, ffs.SEARCH_BOUNDED):
    pl.set_search_mode(mode)
    for _ in range(2):
        pl.plan_batch_host(h_req, h_slo, prob.k_max, out=out)
    n = 6
    t0 = time.perf_counter()
    for _ in range(n):
        pl.plan_batch_host(h_req, h_slo, prob.k_max, out=out)
    res.append((time.perf_counter() - t0) / n * 1e3)
d = torch.empty(prob.R * 80, dtype=torch.uint8, device="cuda")
torch.cuda.synchronize()
t0 = time.perf_counter()
for _ in range(5):
    torch.from_numpy(out.view(np.uint8)).copy_(d, non_blocking=True)
    torch.cuda.synchronize()
d2h = (time.perf_counter() - t0) / 5
print(f"exhaustive {res[0]:.3f} ms  bounded {res[1]:.3f} ms  (plain 80 MiB D2H {d2h * 1e3:.2f} ms = {80 * 2**20 / d2h / 1e9:.1f} GB/s)")
"""
for lib in sys.argv[1:]:
    for _ in range(2):
        r = subprocess.run([sys.executable, "-c", CHILD, ROOT], env=dict(os.environ, FFS_LIB=lib),
                           capture_output=True, text=True, timeout=900)
        print(os.path.basename(lib), r.stdout.strip() or r.stderr[-1500:], flush=True)
