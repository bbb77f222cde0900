#!/bin/bash
# C5: launch list of K7's kernels per window, then ncu --set full of K7b and K7a2 on window 1
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv -k regex:"k_blk|k_check|k_range|k_shadow|k_expand|k_rs_down" --log-file $O/launches_c5_k7.csv python tools/prof_one.py c5 > $O/l5.log 2>&1; echo l5=$?
python tools/launches.py $O/launches_c5_k7.csv > $O/launches_c5_k7.txt 2>&1; head -30 $O/launches_c5_k7.txt
python - <<'PY'
import csv
rows=[r for r in csv.reader(open('gpurun_out/launches_c5_k7.csv')) if len(r)>10]
h=rows[0]; ik,iv,im,iid=h.index("Kernel Name"),h.index("Metric Value"),h.index("Metric Name"),h.index("ID")
d={}
for r in rows[1:]:
    d.setdefault(int(r[iid]),{"k":r[ik].split("(")[0][-24:]})[r[im]]=float(r[iv].replace(",",""))
for i in sorted(d):
    x=d[i]; print(i, x["k"], round(x.get("gpu__time_duration.sum",0)/1e3,1),"us", round((x.get("dram__bytes_read.sum",0)+x.get("dram__bytes_write.sum",0))/1e6,1),"MB")
PY
for k in k_check_tile k_blk_units; do
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:$k --launch-skip 1 -c 1 -o $O/prof_${k}_c5 python tools/prof_one.py c5 > $O/ncu_c5_$k.log 2>&1; echo ncu=$?
python tools/ncu_summary.py $O/prof_${k}_c5.ncu-rep 24 > $O/ncu_${k}_c5.txt 2>&1
head -45 $O/ncu_${k}_c5.txt
done
