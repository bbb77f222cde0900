#!/bin/bash
# one ncu --set full capture per top kernel of a C4 detect (first launch of each), summaries
O=gpurun_out
CFG=${CFG:-c4}
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || exit 1
for k in ${KERNELS:-k_expand k_rs_down k_header k_replay k_check_tile}; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$k -c 1 -o $O/prof_${k}_$CFG python tools/prof_one.py $CFG > $O/ncu_$k.log 2>&1; echo $k=$?
  python tools/ncu_summary.py $O/prof_${k}_$CFG.ncu-rep 14 > $O/ncu_${k}_$CFG.txt 2>&1
  head -32 $O/ncu_${k}_$CFG.txt
done
