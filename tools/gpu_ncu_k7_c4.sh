#!/bin/bash
# ncu --set full of K7's kernels on C4 (one launch each), per-line stall summaries
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
for k in ${KERNELS:-k_blk_sum k_check_tile k_blk_units}; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$k -c 1 -o $O/prof_${k}_${CFG:-c4} python tools/prof_one.py ${CFG:-c4} > $O/ncu_$k.log 2>&1; echo $k=$?
  python tools/ncu_summary.py $O/prof_${k}_${CFG:-c4}.ncu-rep 6 > $O/ncu_${k}_${CFG:-c4}.txt 2>&1
  python tools/ncu_lines.py $O/prof_${k}_${CFG:-c4}.ncu-rep 14 >> $O/ncu_${k}_${CFG:-c4}.txt 2>&1
  cat $O/ncu_${k}_${CFG:-c4}.txt
done
