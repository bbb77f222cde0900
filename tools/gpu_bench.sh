#!/bin/bash
# build, bench (default C4 line with ncu traffic), extra configs, reference arm, launch lists
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 900 python bench.py > $O/bench_c4.json 2> $O/bench_c4.err; echo c4=$?
for c in ${EXTRA:-c2 c3}; do timeout 600 python bench.py --config $c --steps 10 --no-cpu-baseline --no-ncu > $O/bench_$c.json 2> $O/bench_$c.err; echo $c=$?; done
for c in ${LAUNCH:-c4}; do
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $O/launches_$c.csv python tools/prof_one.py $c > /dev/null 2>&1; echo n_$c=$?
python tools/launches.py $O/launches_$c.csv > $O/launches_$c.txt 2>&1
head -14 $O/launches_$c.txt
done
for c in c4 ${EXTRA:-c2 c3}; do timeout 20 python -c "
import json; d=json.load(open('$O/bench_$c.json')); print('$c', round(d['value']/1e9,3), 'Gev/s', round(d['ms_per_step'],4), 'ms', 'e2e', round(d['e2e']['value']/1e9,3), 'K7', round(d['roofline']['frac'],4), d['roofline']['traffic'], 'pipe', round(d['roofline_pipeline']['frac'],4), 'sort', round(d['roofline_sort']['frac'],4), d['phases_ms'], d['clocks'], d.get('cpu_baseline'))"; done
