#!/bin/bash
# K7 iteration: window / shard / stream GPU tests, C4 + C5 bench, C5 K7 launch list, ncu of K7b (SH) on C5 window 1
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 1500 python -m pytest tests -q -m gpu -p no:cacheprovider --timeout 900 -x ${PTK:+-k "$PTK"} > $O/pytest_k7.log 2>&1; echo pytest=$?
tail -3 $O/pytest_k7.log
timeout 900 python bench.py --steps 5 --no-cpu-baseline > $O/bench_c4.json 2> $O/bench_c4.err; echo c4=$?
timeout 1200 python bench.py --config c5 --steps 3 --no-cpu-baseline --no-ncu > $O/bench_c5.json 2> $O/bench_c5.err; echo c5=$?
for c in c4 c5; do timeout 20 python -c "
import json; d=json.load(open('$O/bench_$c.json')); print('$c', round(d['value']/1e9,3), 'Gev/s', round(d['ms_per_step'],4), 'ms', 'K7', round(d['roofline']['frac'],4), d['roofline']['kernel_ms'], d['roofline']['traffic'], d.get('phases_ms'), d['config']['windows'])"; done
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv -k regex:"k_blk|k_check|k_range|k_shadow" --log-file $O/launches_c4_k7.csv python tools/prof_one.py c4 > $O/l4.log 2>&1; echo l4=$?
python tools/launches.py $O/launches_c4_k7.csv > $O/launches_c4_k7.txt 2>&1; cat $O/launches_c4_k7.txt
if [ -z "$NO_NCU" ]; then
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv -k regex:"k_blk|k_check|k_range|k_shadow" --log-file $O/launches_c5_k7.csv python tools/prof_one.py c5 > $O/l5.log 2>&1; echo l5=$?
python tools/launches.py $O/launches_c5_k7.csv > $O/launches_c5_k7.txt 2>&1; cat $O/launches_c5_k7.txt
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_check_tile --launch-skip 1 -c 1 -o $O/prof_k_check_tile_c5 python tools/prof_one.py c5 > $O/ncu_c5_kct.log 2>&1; echo ncu=$?
python tools/ncu_summary.py $O/prof_k_check_tile_c5.ncu-rep 10 > $O/ncu_k_check_tile_c5.txt 2>&1
head -25 $O/ncu_k_check_tile_c5.txt
fi
