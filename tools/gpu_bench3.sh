#!/bin/bash
# bench lines C2 (with the CPU baseline) + C3 / C4, each with roofline (K7) and roofline_sort (K5)
O=gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 600 python bench.py > $O/bench_c2.json 2> $O/bench_c2.err; echo c2=$?
for c in c3 c4; do timeout 600 python bench.py --config $c --steps 5 --no-cpu-baseline > $O/bench_$c.json 2> $O/bench_$c.err; echo $c=$?; done
for c in c2 c3 c4; do timeout 20 python -c "
import json; d=json.load(open('$O/bench_$c.json')); print('$c', round(d['value']/1e9,3), 'Gev/s', round(d['ms_per_step'],3), 'ms', 'K7', round(d['roofline']['frac'],4), 'sort', round(d['roofline_sort']['frac'],4), d['clocks'])"; done
