#!/bin/bash
# C5 (several windows): window-related GPU tests, bench, one ncu capture of K7b on a carrying window
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 1500 python -m pytest tests -q -m gpu -p no:cacheprovider --timeout 900 -x -k "window or stream or shard or c5 or overwrite" > $O/pytest_win.log 2>&1; echo pytest=$?
tail -3 $O/pytest_win.log
timeout 1200 python bench.py --config c5 --steps 3 --no-cpu-baseline --no-ncu > $O/bench_c5.json 2> $O/bench_c5.err; echo c5=$?
timeout 20 python -c "
import json; d=json.load(open('$O/bench_c5.json')); print('c5', round(d['value']/1e9,3), 'Gev/s', round(d['ms_per_step'],4), 'ms', 'K7', round(d['roofline']['frac'],4), d.get('phases_ms'), d['config']['windows'])"
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:k_check_tile --launch-skip 3 -c 1 -o $O/prof_k_check_tile_c5 python tools/prof_one.py c5 > $O/ncu_c5.log 2>&1; echo ncu=$?
python tools/ncu_summary.py $O/prof_k_check_tile_c5.ncu-rep 20 > $O/ncu_k_check_tile_c5.txt 2>&1
head -40 $O/ncu_k_check_tile_c5.txt
