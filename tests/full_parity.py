"""Full-batch parity evidence: every request of the given configs planned on the GPU
(production path, the bench launch configuration) and by the CPU oracle, compared field by
field.  Writes gpurun_out/full_parity_<cfg>.json.  One-off evidence run (C5 takes ~40 min of
oracle time on 16 host cores); the sampled versions are in tests/test_gpu_parity.py.

    python tests/full_parity.py 3 5 [--exhaustive]   (test infrastructure: the only place
    besides the test suite that runs the oracle at full size; tools/run_full_parity.sh)
"""
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
from paper_conf_hpdc_hui0s25_b200 import ffs, workload as W  # noqa: E402


def main():
    import torch
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    pl = ffs.Planner(0)
    exhaustive = "--exhaustive" in sys.argv
    if exhaustive:
        pl.set_search_mode(ffs.SEARCH_EXHAUSTIVE)
    for cfg in [int(x) for x in sys.argv[1:] if not x.startswith("--")] or [3]:
        prob = W.CONFIGS[cfg]()
        pl.stage(prob)
        req, slo = ffs.to_device(prob)
        t = time.perf_counter()
        p = ffs.plans_to_numpy(pl.plan_batch(req, slo, prob.k_max))
        torch.cuda.synchronize()
        gpu_s = time.perf_counter() - t
        mism = {}
        t = time.perf_counter()
        chunk = 16384
        for lo in range(0, prob.R, chunk):
            idx = np.arange(lo, min(prob.R, lo + chunk))
            o = oracle.plan(prob.subset(idx), checks=False)
            g = p[idx]
            for a in ("key", "status", "k", "cut_mask", "e2e_us", "bottleneck_us", "gpcs", "cvq"):
                ok = o["status"] == 0 if a not in ("key", "status") else np.ones(len(idx), bool)
                bad = int((g[a][ok] != o[a][ok]).sum())
                mism[a] = mism.get(a, 0) + bad
            mism["prof"] = mism.get("prof", 0) + int((g["prof"] != o["prof"]).any(axis=1).sum())
            mism["slice"] = mism.get("slice", 0) + int((g["slice"] != o["slice"]).any(axis=1).sum())
            print(f"C{cfg}: {lo + len(idx)}/{prob.R} requests checked, mismatches so far {sum(mism.values())}",
                  flush=True)
        cpu_s = time.perf_counter() - t
        st = p["status"]
        res = {"config": f"C{cfg}", "mode": "exhaustive" if exhaustive else "bounded", "requests": prob.R,
               "mismatched_fields": mism,
               "bit_exact": all(v == 0 for v in mism.values()), "gpu_s": gpu_s, "oracle_s": cpu_s,
               "oracle_threads": os.cpu_count(), "ok": int((st == 0).sum()), "infeasible": int((st == 1).sum()),
               "multi_stage": int(((st == 0) & (p["k"] > 1)).sum())}
        print(json.dumps(res), flush=True)
        with open(os.path.join(ROOT, "gpurun_out", f"full_parity_C{cfg}.json"), "w") as fh:
            json.dump(res, fh, indent=1)


if __name__ == "__main__":
    main()
