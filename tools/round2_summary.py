"""Collect one GPU evidence run (tools/gpu_evidence_r2.sh -> gpurun_out/ev2) into
profiles/round2/: the bench JSON lines, the ncu launch-list shares, ncu --set full
summaries of the profiled kernels, the shard emulation, segment scaling and the issue
microbenchmark.  Also refreshes profiles/traffic.json (DRAM bytes per launch).

    python tools/round2_summary.py [gpurun_out/ev2]
"""
import collections
import csv
import io
import json
import os
import shutil
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "gpurun_out", "ev2")
DST = os.path.join(ROOT, "profiles", "round2")
os.makedirs(DST, exist_ok=True)


def last_json(path):
    try:
        lines = [x for x in open(path) if x.startswith("{")]
    except OSError:
        return None
    return json.loads(lines[-1]) if lines else None


def ncu_raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    return rows[0], rows[1], rows[2:]


for name, src in (("bench_c5.json", "bench.log"), ("bench_reference.json", "bench_reference.log")):
    d = last_json(os.path.join(SRC, src))
    if d:
        json.dump(d, open(os.path.join(DST, name), "w"), indent=1)

# launch list: share of the exhaustive and the bounded step per kernel (bench --steps 3)
lp = os.path.join(SRC, "launches_c5.csv")
if os.path.exists(lp):
    shutil.copy(lp, os.path.join(DST, "launches_c5.csv"))
    rows = [r for r in csv.reader(open(lp)) if len(r) > 10]
    h = rows[0]
    iN, iV = h.index("Kernel Name"), h.index("Metric Value")
    agg = collections.defaultdict(lambda: [0, 0.0])
    for r in rows[1:]:
        k = r[iN].split("(")[0].replace("void ", "")
        agg[k][0] += 1
        agg[k][1] += float(r[iV].replace(",", ""))
    search = {k: v for k, v in agg.items() if "peak" not in k}
    tot = sum(v[1] for v in search.values())
    with open(os.path.join(DST, "launches_c5_summary.txt"), "w") as fh:
        fh.write("ncu --metrics gpu__time_duration.sum --clock-control none, bench.py --steps 3 --warmup 3\n"
                 "(3+3 exhaustive and 3+3 bounded steps; peak microbenchmarks excluded from the shares)\n")
        for k, (n, ns) in sorted(search.items(), key=lambda x: -x[1][1]):
            fh.write(f"{k:48s} launches {n:4d}  {ns / 1e6:10.3f} ms  {100 * ns / tot:6.2f} %\n")

traffic = {}
for rep in ("prof_ks4_exh", "prof_ks4_bnd", "prof_c4"):
    p = os.path.join(SRC, rep + ".ncu-rep")
    if not os.path.exists(p):
        continue
    shutil.copy(p, os.path.join(DST, rep + ".ncu-rep"))
    h, units, vs = ncu_raw(p)
    with open(os.path.join(DST, rep + "_summary.txt"), "w") as fh:
        for v in vs:
            for w in ("Kernel Name", "gpu__time_duration.sum", "launch__registers_per_thread", "launch__block_size",
                      "launch__grid_size", "smsp__issue_active.avg.pct_of_peak_sustained_active",
                      "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
                      "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
                      "smsp__inst_executed.sum", "smsp__thread_inst_executed_per_inst_executed.ratio",
                      "dram__bytes_read.sum", "dram__bytes_write.sum",
                      "dram__throughput.avg.pct_of_peak_sustained_elapsed",
                      "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "local_load"):
                if w in h:
                    fh.write(f"{w:60s} {v[h.index(w)]}\n")
            fh.write("\n")
            name = v[h.index("Kernel Name")]
            traffic[f"{rep}: {name}"] = {w: v[h.index(w)] + " " + units[h.index(w)]
                                         for w in ("dram__bytes_read.sum", "dram__bytes_write.sum") if w in h}
    if rep == "prof_ks4_exh":
        lines = subprocess.run([sys.executable, os.path.join(ROOT, "tools", "ncu_lines.py"), p, "30"],
                               capture_output=True, text=True).stdout
        open(os.path.join(DST, rep + "_lines.txt"), "w").write(lines)

for f in ("shard_emulation.json", "seg_scaling.log", "issue_bench.log", "smoke.log", "gpu_tests.log"):
    p = os.path.join(SRC, f)
    if os.path.exists(p):
        shutil.copy(p, os.path.join(DST, {"shard_emulation.json": "shard_emulation_c5.json"}.get(f, f)))
json.dump(traffic, open(os.path.join(DST, "dram_per_launch_raw.json"), "w"), indent=1)


def _bytes(x):  # "25.004032 Mbyte" -> bytes
    v, u = x.split()
    return int(round(float(v) * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}[u]))


# profiles/traffic.json: the bench's roofline.traffic (DRAM read + write per launch)
tj = os.path.join(ROOT, "profiles", "traffic.json")
tr = json.load(open(tj)) if os.path.exists(tj) else {}
for key, d in traffic.items():
    rep, name = key.split(": ", 1)
    tot = sum(_bytes(x) for x in d.values())
    if rep == "prof_ks4_exh" and "k_plan_search<4" in name:
        tr["k_plan_search<4>"] = tot
        tr["_source"] = (f"profiles/round2/prof_ks4_exh.ncu-rep (ncu --set full, exhaustive mode, C5): "
                         f"{d.get('dram__bytes_read.sum')} read + {d.get('dram__bytes_write.sum')} written for one "
                         f"launch of {name.split('(')[0].replace('void ', '')}")
    if rep == "prof_c4" and "k_evict_ticks" in name:
        tr["k_evict_ticks"] = tot
        tr["_source_k_evict_ticks"] = (f"profiles/round2/prof_c4.ncu-rep (ncu --set full, ffs_evict_step on C4): "
                                       f"{d.get('dram__bytes_read.sum')} read + {d.get('dram__bytes_write.sum')} "
                                       f"written per launch")
json.dump(tr, open(tj, "w"), indent=1)
print("wrote", sorted(os.listdir(DST)))
