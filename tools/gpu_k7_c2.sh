#!/bin/bash
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
for c in c2 c3 c4; do
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none --csv -k regex:"k_blk|k_check|k_shadow" --log-file $O/launches_${c}_k7.csv python tools/prof_one.py $c > /dev/null 2>&1; echo l=$?
python tools/launches.py $O/launches_${c}_k7.csv
done
CFG=c2 KERNELS="k_blk_sum k_check_tile" bash tools/gpu_ncu_k7_c4.sh 2>&1 | grep -v "^k_"
CFG=c4 KERNELS="k_check_tile" bash tools/gpu_ncu_k7_c4.sh 2>&1 | grep -v "^k_"
