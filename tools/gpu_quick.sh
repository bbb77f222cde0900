#!/bin/bash
# quick check: build, parity subset, C4 bench, launch times of the named kernels on C4
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 1500 python -m pytest tests -q -m gpu -p no:cacheprovider --timeout 600 -x -k "${PTK:-c1 or litmus or random or window or stream or shard or c4 or infeasible}" > $O/pytest_q.log 2>&1; echo pytest=$?
tail -2 $O/pytest_q.log
timeout 900 python bench.py --steps 5 --no-cpu-baseline --no-ncu 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('c4', round(d['value']/1e9,3), round(d['ms_per_step'],4), d['phases_ms'])"
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv -k regex:"${KRE:-k_expand|k_blk|k_check}" --log-file $O/lq.csv python tools/prof_one.py c4 > /dev/null 2>&1; python tools/launches.py $O/lq.csv
