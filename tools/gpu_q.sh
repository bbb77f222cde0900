#!/bin/bash
# quick iteration: build, a parity subset, bench C2/C3/C4 (default variant), launch list of C2 and C4
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -m "gpu" -p no:cacheprovider --timeout 300 -x -k "k7_variants or configs_reduced or random_traces_granules or hot_granule or c3_64 or c4_64" > gpurun_out/pytest_q.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_q.log
for c in c2 c3 c4; do
timeout 300 python bench.py --config $c --steps 5 --no-cpu-baseline > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err
timeout 20 python -c "
import json; d=json.load(open('gpurun_out/bench_$c.json')); print('$c', round(d['value']/1e9,3), 'Gev/s', round(d['ms_per_step'],3), 'ms', 'roof', round(d['roofline']['frac'],4), d['phases_ms'])"
done
for c in c2 c4; do
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_$c.csv python tools/prof_one.py $c > /dev/null 2>&1
python tools/launches.py gpurun_out/launches_$c.csv 2>/dev/null | head -14
done
