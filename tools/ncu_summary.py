"""Summarise an ncu --set full report of a search kernel: time, issue/pipe utilisation,
stall reasons, executed lane-instructions per candidate by opcode (design input)."""
import collections
import csv
import io
import re
import subprocess
import sys

rep, cands = sys.argv[1], float(sys.argv[2])
flt = ["-k", "regex:" + sys.argv[3]] if len(sys.argv) > 3 else []  # kernel filter
raw = subprocess.run(["ncu", "-i", rep, *flt, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
h, v = rows[0], rows[2]
for w in ["Kernel Name", "gpu__time_duration.sum", "launch__registers_per_thread", "launch__block_size",
          "smsp__issue_active.avg.pct_of_peak_sustained_active",
          "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
          "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
          "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
          "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
          "smsp__inst_executed.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
          "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum"]:
    if w in h:
        print(f"{w:60s} {v[h.index(w)]}")
st = sorted(((float(v[i]), n) for i, n in enumerate(h)
             if "pcsamp_warps_issue_stalled" in n and not n.endswith("not_issued") and v[i] not in ("", "n/a")),
            reverse=True)
tot = sum(x for x, _ in st)
print("stall samples:", ", ".join(f"{n.split('stalled_')[1]} {x / tot:.2f}" for x, n in st[:8]))
src = subprocess.run(["ncu", "-i", rep, *flt, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(src)))
h = rows[1]
iA, iE = h.index("Source"), h.index("Instructions Executed")
ops = collections.Counter()
tot = 0
for r in rows[2:]:
    if len(r) <= max(iA, iE) or not r[iE].isdigit():
        continue
    e = int(r[iE])
    m = re.match(r"(@!?U?P\w+\s+)?([A-Z0-9_]+)", r[iA].strip())
    ops[m.group(2) if m else "?"] += e
    tot += e
print(f"lane-instructions per candidate: {tot * 32 / cands:.3f}")
print("  " + ", ".join(f"{o} {c * 32 / cands:.3f}" for o, c in ops.most_common(14)))
