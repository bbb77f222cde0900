#!/bin/bash
# build, smoke, full GPU parity, bench C2 (+CPU baseline) / C3 / C4 / reference arm, ncu launch lists C2 / C3 / C4
O=gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo smoke=$?
timeout 900 python -m pytest tests -q -m gpu -p no:cacheprovider --timeout 600 > $O/pytest_gpu.log 2>&1; echo pytest=$?
tail -1 $O/pytest_gpu.log
timeout 600 python bench.py > $O/bench_c2.json 2> $O/bench_c2.err; echo c2=$?
for c in c3 c4; do timeout 600 python bench.py --config $c --steps 10 --no-cpu-baseline > $O/bench_$c.json 2> $O/bench_$c.err; echo $c=$?; done
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 > $O/bench_ref.json 2> $O/bench_ref.err; echo ref=$?
for c in c2 c3 c4; do timeout 20 python -c "
import json; d=json.load(open('$O/bench_$c.json')); print('$c', round(d['value']/1e9,3), 'Gev/s', round(d['ms_per_step'],4), 'ms', 'e2e', round(d['e2e']['value']/1e9,3), 'K7', round(d['roofline']['frac'],4), 'sort', round(d['roofline_sort']['frac'],4), d['phases_ms'], d['clocks'])"; done
for c in c2 c3 c4; do
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $O/launches_$c.csv python tools/prof_one.py $c > /dev/null 2>&1; echo n_$c=$?
python tools/launches.py $O/launches_$c.csv > $O/launches_$c.txt 2>&1
done
head -8 $O/launches_c2.txt
