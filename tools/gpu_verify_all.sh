#!/bin/bash
# full GPU parity + bench lines C4 (with in-job ncu) / C2 / C3 / C5 + K7 launch split
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo smoke=$?
timeout 2000 python -m pytest tests -q -m gpu -p no:cacheprovider --timeout 900 > $O/pytest_gpu.log 2>&1; echo pytest=$?
tail -3 $O/pytest_gpu.log
timeout 900 python bench.py ${C4ARGS:---no-cpu-baseline} > $O/bench_c4.json 2> $O/bench_c4.err; echo c4=$?
for c in c2 c3; do timeout 600 python bench.py --config $c --steps 10 --no-cpu-baseline --no-ncu > $O/bench_$c.json 2> $O/bench_$c.err; echo $c=$?; done
timeout 1200 python bench.py --config c5 --steps 3 --no-cpu-baseline --no-ncu > $O/bench_c5.json 2> $O/bench_c5.err; echo c5=$?
for c in c4 c2 c3 c5; do timeout 20 python -c "
import json; d=json.load(open('$O/bench_$c.json')); print('$c', round(d['value']/1e9,3), 'Gev/s', round(d['ms_per_step'],4), 'ms e2e', round(d['e2e']['value']/1e9,3), 'K7', round(d['roofline']['frac'],4), round(d['roofline']['kernel_ms'],4), d['roofline']['traffic'], 'pipe', round(d['roofline_pipeline']['frac'],4), d['phases_ms'])"; done
for c in c2 c4; do
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv -k regex:"k_blk|k_check" --log-file $O/l7_$c.csv python tools/prof_one.py $c > /dev/null 2>&1; echo "$c"; python tools/launches.py $O/l7_$c.csv | tail -2
done
