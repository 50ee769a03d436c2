"""Per-source-line executed instructions of an ncu report (--page source, cuda+sass):
prints the top lines by warp-instructions executed and the share per function region."""
import csv
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
flt = []
if len(sys.argv) > 3:  # a kernel-name regex, or the index of the launch in the report
    a = sys.argv[3]
    flt = ["--launch-skip", a, "--launch-count", "1"] if a.isdigit() else ["-k", "regex:" + a]
out = subprocess.run(["ncu", "-i", rep, *flt, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
hdr = next(i for i, r in enumerate(rows) if r and r[0] == "Line No")
h = rows[hdr]
iE = h.index("Instructions Executed")
per_line, src = {}, {}
cur = None
for r in rows[hdr + 1:]:
    if not r:
        continue
    if r[0] and r[0].isdigit():
        cur = int(r[0])
        src[cur] = r[1]
    try:
        v = float(r[iE] or 0)
    except (ValueError, IndexError):
        continue
    if cur is not None and r[2]:  # a SASS row under source line `cur`
        per_line[cur] = per_line.get(cur, 0.0) + v
tot = sum(per_line.values())
print(f"total warp-instructions {tot:.4g}")
for ln, v in sorted(per_line.items(), key=lambda x: -x[1])[:top]:
    print(f"{ln:5d} {v / tot * 100:6.2f}%  {src.get(ln, '').strip()[:110]}")
