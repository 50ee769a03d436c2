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
# NEXT rows on the C2 batch: ranked first-fit (K6), joint commit (K7), frontier (K8),
# routing (K9) and the time-sharing simulator (K10)
prob = W.config2(R=96)
pl.stage(prob)
req, slo = ffs.to_device(prob)
pl.rank_partitions(prob.k_max, int(np.argmax(prob.gpcs)))
pl.plan_ranked(req, slo)
pl.plan_joint(req, slo, prob.k_max)
pl.frontier_build(prob.k_max)
pl.plan_frontier(req, slo)
pl.plan_frontier_any(req, slo)
rng = W.SplitMix64(5)
ni = 12
inst = np.zeros(ni, dtype=W.INST_DTYPE)
inst["func"] = rng.integers(0, prob.F - 1, ni)
inst["slice"] = -1
state = rng.integers(0, 3, ni).astype(np.uint8)
lat = rng.integers(1, 100, ni).astype(np.uint32)
cap = rng.integers(0, 3, ni).astype(np.uint32)
pl.route(req, slo, torch.from_numpy(inst.view(np.uint8)).cuda(), torch.from_numpy(state).cuda(),
         torch.from_numpy(lat.view(np.int32)).cuda(), torch.from_numpy(cap.view(np.int32)).cuda())
tr = W.sim_trace(seed=101, T=64, n_funcs=6, nodes=[W.PART_P1, W.PART_HYBRID], rate_scale=8.0)
pl.stage(tr.problem)
pl.simulate(tr)
torch.cuda.synchronize()
# NEXT-1 DAG stages (K11): a small DAG batch with split-capable blocks, with checksums
dprob, dag = W.dag_config(R=64, F=6)
pl.stage(dprob)
pl.stage_dag(dag, dprob.k_max)
dreq, dslo = ffs.to_device(dprob)
dchecks = torch.zeros((dprob.R, 3), dtype=torch.int64, device="cuda")
pl.plan_dag(dreq, dslo, checks=dchecks)
pl.plan_dag(dreq, dslo)
torch.cuda.synchronize()
print("sanitize-run ok")
