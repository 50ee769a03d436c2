"""Driver for ncu captures of the DAG-stage kernel (NEXT-1, not a benchmark): stages the CD
workload and runs ffs_plan_dag `--calls` times.
    ncu --set full -k regex:k_plan_dag --launch-skip 1 --launch-count 1 -o out python tools/prof_dag.py"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from paper_conf_hpdc_hui0s25_b200 import ffs, workload as W  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--calls", type=int, default=2)
a = ap.parse_args()
prob, dag = W.dag_config()
pl = ffs.Planner(0)
pl.stage(prob)
pl.stage_dag(dag, prob.k_max)
req, slo = ffs.to_device(prob)
out = torch.empty((prob.R, ffs.DAG_PLAN_DTYPE.itemsize), dtype=torch.uint8, device="cuda")
for _ in range(a.calls):
    pl.plan_dag(req, slo, out=out)
torch.cuda.synchronize()
print("done")
