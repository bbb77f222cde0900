"""Per-source-line stall samples of an .ncu-rep (cuda,sass view): top lines and their hottest SASS."""
import csv, subprocess, sys
rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
hdr = None; f = None; line = None; src = None; agg = {}
for r in rows:
    if len(r) == 2 and r[0] in ("File Path", "Function Name"):
        if r[0] == "File Path": f = r[1].split("/")[-1]
        continue
    if r and r[0] == "Line No":
        hdr = r; i_s = hdr.index("Warp Stall Sampling (All Samples)"); continue
    if not hdr or len(r) < len(hdr): continue
    if r[0].strip():
        line = r[0]; src = r[1]
    v = r[i_s]
    if v and v.replace('.', '').isdigit():
        a = agg.setdefault((f, line), [0, src, []]); a[0] += int(float(v)); a[2].append((int(float(v)), r[3][:50]))
tot = sum(a[0] for a in agg.values())
print("samples", tot)
for (f, l), (v, s, ins) in sorted(agg.items(), key=lambda x: -x[1][0])[:top]:
    ins.sort(reverse=True)
    print(f"{v:8d} {100*v/max(tot,1):5.1f}% {f}:{l:5s} {s.strip()[:80]}  | {ins[0][1]}")
