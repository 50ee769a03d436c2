"""Debug: bounded (list) vs exhaustive vs bounded-with-fallback keys on a config."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_hpdc_hui0s25_b200 import ffs, workload as W
cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 5
prob = W.CONFIGS[cfg]()
pl = ffs.Planner(0); pl.stage(prob)
req, slo = ffs.to_device(prob)
K = prob.k_max
kb = pl.plan_keys(req, slo, K).cpu().numpy(); live = pl.live_records(); sb = pl.scored()
pl.set_search_mode(ffs.SEARCH_EXHAUSTIVE)
ke = pl.plan_keys(req, slo, K).cpu().numpy()
pl.set_search_mode(ffs.SEARCH_BOUNDED)
os.environ["FFS_LIST_CAP"] = "0"
p2 = ffs.Planner(0); p2.stage(prob)
kf = p2.plan_keys(req, slo, K).cpu().numpy()
print("live", live[:4], "scored", sb[:4])
print("bounded-list vs exhaustive mismatches:", int((kb != ke).sum()), " fallback vs exhaustive:", int((kf != ke).sum()))
bad = np.flatnonzero(kb != ke)[:20]
n = prob.chain_len()[prob.req["func"]]
def dec(k):
    if k == np.iinfo(np.int64).max: return "NONE"
    k = int(k); return f"cvq={k>>50} k={((k>>47)&7)+1} g={(k>>41)&63} idx={k & ((1<<41)-1)}"
for r in bad:
    print(r, "n", n[r], "func", prob.req["func"][r], "node", prob.req["node"][r], "B", prob.slo_us[r], "| list", dec(kb[r]), "| exh", dec(ke[r]))
