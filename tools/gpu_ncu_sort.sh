#!/bin/bash
# one ncu --set full capture of the K5 downsweep (first k_rs_down<10> launch of the item sort, C2)
O=gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_rs_down --launch-skip 1 -c 1 -o $O/prof_rs_down_c2 python tools/prof_one.py c2 > $O/ncu_rs_down.log 2>&1; echo f=$?
python tools/ncu_summary.py $O/prof_rs_down_c2.ncu-rep 12 > $O/ncu_rs_down_c2.txt 2>&1; echo s=$?
head -60 $O/ncu_rs_down_c2.txt
