"""Full-batch parity evidence: every request of the given configs planned on the GPU
(production path, the bench launch configuration) and by the CPU oracle, compared field by
field.  Writes gpurun_out/full_parity_<cfg>.json.  One-off evidence run (C5 takes ~40 min of
oracle time on 16 host cores); the sampled versions are in tests/test_gpu_parity.py.

    python tests/full_parity.py 3 5   (test infrastructure: the only place besides the test
    suite that runs the oracle at full size; tools/run_full_parity.sh; both search modes)
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
    """Both search modes are planned on the GPU and compared against one oracle pass."""
    import torch
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    pl = ffs.Planner(0)
    for cfg in [int(x) for x in sys.argv[1:] if not x.startswith("--")] or [3]:
        prob = W.CONFIGS[cfg]()
        pl.stage(prob)
        req, slo = ffs.to_device(prob)
        plans, gpu_s = {}, {}
        for mode, m in (("bounded", ffs.SEARCH_BOUNDED), ("exhaustive", ffs.SEARCH_EXHAUSTIVE)):
            pl.set_search_mode(m)
            t = time.perf_counter()
            plans[mode] = ffs.plans_to_numpy(pl.plan_batch(req, slo, prob.k_max))
            torch.cuda.synchronize()
            gpu_s[mode] = time.perf_counter() - t
        pl.set_search_mode(ffs.SEARCH_BOUNDED)
        mism = {mode: {} for mode in plans}
        t = time.perf_counter()
        chunk = 16384
        for lo in range(0, prob.R, chunk):
            idx = np.arange(lo, min(prob.R, lo + chunk))
            o = oracle.plan(prob.subset(idx), checks=False)
            for mode, p in plans.items():
                g, mm = p[idx], mism[mode]
                for a in ("key", "status", "k", "cut_mask", "e2e_us", "bottleneck_us", "gpcs", "cvq"):
                    ok = o["status"] == 0 if a not in ("key", "status") else np.ones(len(idx), bool)
                    mm[a] = mm.get(a, 0) + int((g[a][ok] != o[a][ok]).sum())
                mm["prof"] = mm.get("prof", 0) + int((g["prof"] != o["prof"]).any(axis=1).sum())
                mm["slice"] = mm.get("slice", 0) + int((g["slice"] != o["slice"]).any(axis=1).sum())
            print(f"C{cfg}: {lo + len(idx)}/{prob.R} requests checked, mismatches so far "
                  f"{ {m: sum(v.values()) for m, v in mism.items()} }", flush=True)
        cpu_s = time.perf_counter() - t
        st = plans["bounded"]["status"]
        res = {"config": f"C{cfg}", "requests": prob.R, "modes": list(plans), "mismatched_fields": mism,
               "bit_exact": all(v == 0 for mm in mism.values() for v in mm.values()), "gpu_s": gpu_s,
               "oracle_s": cpu_s, "oracle_threads": os.cpu_count(), "ok": int((st == 0).sum()),
               "infeasible": int((st == 1).sum()), "multi_stage": int(((st == 0) & (plans["bounded"]["k"] > 1)).sum())}
        print(json.dumps(res), flush=True)
        with open(os.path.join(ROOT, "gpurun_out", f"full_parity_C{cfg}.json"), "w") as fh:
            json.dump(res, fh, indent=1)


if __name__ == "__main__":
    main()
