"""Attribute ncu per-instruction counts (sass source page) of one kernel to CUDA source lines.
usage: sass_lines.py REPORT.ncu-rep CUBIN KERNEL_SUBSTRING [top]"""
import csv, re, subprocess, sys
from collections import defaultdict
rep, cubin, kname = sys.argv[1:4]
top = int(sys.argv[4]) if len(sys.argv) > 4 else 30
dis = subprocess.run(["nvdisasm", "-g", "-c", cubin], capture_output=True, text=True).stdout
# per-function list of (offset, file:line)
cur, line_of, inside = None, {}, False
for ln in dis.splitlines():
    if ln.startswith(".text.") and ln.rstrip().endswith(":"):
        inside = kname in ln
        continue
    if not inside:
        continue
    m = re.search(r'//## File "([^"]+)", line (\d+)', ln)
    if m:
        cur = f"{m.group(1).split('/')[-1]}:{m.group(2)}"
        continue
    m = re.match(r"\s*/\*([0-9a-f]{4,})\*/", ln)
    if m:
        line_of[int(m.group(1), 16)] = cur
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True,
                     text=True).stdout
rows = list(csv.reader(src.splitlines()))
h = rows[0] if "Address" in rows[0] else rows[1]
data = [r for r in rows[rows.index(h) + 1:] if len(r) == len(h)]
ia, ie, isamp = h.index("Address"), h.index("Instructions Executed"), h.index("Warp Stall Sampling (All Samples)")
addrs = [int(r[ia], 16) for r in data]
base = min(addrs)
agg_i, agg_s = defaultdict(int), defaultdict(int)
for r, a in zip(data, addrs):
    l = line_of.get(a - base, "?")
    agg_i[l] += int(r[ie] or 0)
    agg_s[l] += int(r[isamp] or 0)
ti, ts = sum(agg_i.values()), sum(agg_s.values())
print(f"total inst {ti}  samples {ts}")
for l, v in sorted(agg_i.items(), key=lambda x: -x[1])[:top]:
    print(f"  {l:22s} inst {v:11d} {100*v/ti:5.1f}%   samples {agg_s[l]:6d} {100*agg_s[l]/max(ts,1):5.1f}%")
if len(sys.argv) > 5:  # range summary: comma-separated "name:lo-hi" over check.cu lines
    for spec in sys.argv[5].split(","):
        nm, rg = spec.split(":")
        lo, hi = map(int, rg.split("-"))
        s = sum(v for l, v in agg_i.items() if l and l.startswith(sys.argv[6] if len(sys.argv) > 6 else "check.cu:")
                and lo <= int(l.split(":")[1]) <= hi)
        print(f"  range {nm:12s} {lo}-{hi}: {s:11d} {100*s/ti:5.1f}%")
