#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -m "gpu" -p no:cacheprovider --timeout 300 -k "c6" > gpurun_out/pytest_c6.log 2>&1; echo pytest=$?
tail -5 gpurun_out/pytest_c6.log; grep -E "Error|assert" gpurun_out/pytest_c6.log | head
for c in c6 c2; do
timeout 300 python bench.py --config $c --steps 5 > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; tail -3 gpurun_out/bench_$c.err
timeout 20 python -c "
import json; d=json.load(open('gpurun_out/bench_$c.json')); print('$c', round(d['value']/1e9,3), 'Gev/s', round(d['ms_per_step'],3), 'ms', 'roof', d['roofline'], d['phases_ms'], d.get('cpu_baseline'))"
done
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_c6.csv python tools/prof_one.py c6 > /dev/null 2>&1
python tools/launches.py gpurun_out/launches_c6.csv 2>/dev/null | head -14
