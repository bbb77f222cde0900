"""Aggregate an ncu launch-list CSV (gpu__time_duration.sum [+ dram bytes]) per kernel for the last bc_detect."""
import csv, sys
f = sys.argv[1]
rows = [r for r in csv.reader(open(f)) if len(r) > 10]
h = rows[0]
ik, iv, im, iid = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Name"), h.index("ID")
d = {}
for r in rows[1:]:
    d.setdefault(int(r[iid]), {"k": r[ik].split("(")[0][:40]})[r[im]] = float(r[iv].replace(",", ""))
ids = sorted(d)
starts = [i for i in ids if d[i]["k"].endswith("k_header")]
last = starts[-1] if starts else ids[0]
agg, tot = {}, 0.0
for i in ids:
    if i < last:
        continue
    k = d[i]["k"]; t = d[i].get("gpu__time_duration.sum", 0)
    a = agg.setdefault(k, [0, 0.0, 0.0]); a[0] += 1; a[1] += t
    a[2] += d[i].get("dram__bytes_read.sum", 0) + d[i].get("dram__bytes_write.sum", 0)
    tot += t
print(f"{f}: {sum(a[0] for a in agg.values())} launches in the last detect, {tot/1000:.1f} us serialised")
for k, (n, t, b) in sorted(agg.items(), key=lambda x: -x[1][1]):
    print(f"  {k:40s} n={n:3d} {t/1000:9.1f} us {100*t/tot:5.1f}%  dram {b/1e6:9.1f} MB")
