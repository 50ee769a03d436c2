"""Compare experiment builds of libffs.so (design input, not a benchmark): for every
variant .so given, time ffs_plan_keys on a config in exhaustive and bounded mode (best of
`reps`, per-segment CUDA events) and check its keys against the first variant's.

    python tools/variants.py --config 5 --reps 3 /tmp/v0.so /tmp/v1.so ...

Each variant runs in its own subprocess (FFS_LIB selects the library)."""
import argparse
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = r"""
import json, os, sys
sys.path.insert(0, sys.argv[1])
import torch
from paper_conf_hpdc_hui0s25_b200 import ffs, workload as W
cfg, reps, out = int(sys.argv[2]), int(sys.argv[3]), sys.argv[4]
prob = W.CONFIGS[cfg]()
pl = ffs.Planner(0)
pl.stage(prob)
req, slo = ffs.to_device(prob)
res = {}
for name, mode in (("exhaustive", ffs.SEARCH_EXHAUSTIVE), ("bounded", ffs.SEARCH_BOUNDED)):
    pl.set_search_mode(mode)
    keys = torch.empty(prob.R, dtype=torch.int64, device="cuda")
    best = None
    for _ in range(reps + 1):
        pl.plan_keys(req, slo, prob.k_max, keys=keys)
        torch.cuda.synchronize()
        ms = pl.segment_times()[:prob.k_max]
        best = ms if best is None else [min(a, b) for a, b in zip(best, ms)]
    res[name] = {"seg_ms": best, "total_ms": sum(best), "scored": pl.scored()[:prob.k_max]}
    torch.save(keys.cpu(), out + "." + name + ".pt")
json.dump(res, open(out + ".json", "w"))
"""


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=5)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("libs", nargs="+")
    a = ap.parse_args()
    import torch
    ref = {}
    for i, lib in enumerate(a.libs):
        out = f"/tmp/variant{i}"
        env = dict(os.environ, FFS_LIB=lib)
        r = subprocess.run([sys.executable, "-c", CHILD, ROOT, str(a.config), str(a.reps), out], env=env,
                           capture_output=True, text=True, timeout=1200)
        if r.returncode != 0:
            print(f"{lib}: FAILED\n{r.stderr[-2000:]}", flush=True)
            continue
        res = json.load(open(out + ".json"))
        line = [os.path.basename(lib)]
        for mode in ("exhaustive", "bounded"):
            k = torch.load(out + "." + mode + ".pt")
            if mode not in ref:
                ref[mode] = k
            same = torch.equal(k, ref[mode])
            seg = " ".join(f"{t:.3f}" for t in res[mode]["seg_ms"])
            line.append(f"{mode} {res[mode]['total_ms']:.3f} ms [{seg}] keys {'=' if same else 'DIFFER'}")
        print("  ".join(line), flush=True)


if __name__ == "__main__":
    main()
