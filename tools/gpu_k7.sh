#!/bin/bash
# K7 iteration: build, GPU parity suite, bench C2/C3/C4 (default K7 and ballot), launch list C2
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python -m pytest tests -q -m "gpu" -p no:cacheprovider --timeout 300 -x > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_gpu.log
grep -E "FAILED|Error|assert" gpurun_out/pytest_gpu.log | head -20
for c in c2 c3 c4; do timeout 300 python bench.py --config $c --steps 5 --no-cpu-baseline > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; echo $c=$?; tail -2 gpurun_out/bench_$c.err; timeout 20 python -c "
import json; d=json.load(open('gpurun_out/bench_$c.json')); print('$c', round(d['value']/1e9,3), 'Gev/s', round(d['ms_per_step'],3), 'ms', 'e2e', round(d['e2e']['value']/1e9,3), 'roof', round(d['roofline']['frac'],4), d['phases_ms'])"; done
for c in c2 c4; do BC_K7=ballot timeout 300 python bench.py --config $c --steps 5 --no-cpu-baseline > gpurun_out/bench_${c}_ballot.json 2>/dev/null; timeout 20 python -c "
import json; d=json.load(open('gpurun_out/bench_${c}_ballot.json')); print('$c ballot', round(d['ms_per_step'],3), 'ms k_check', d['phases_ms']['k_check'])"; done
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_c2.csv python tools/prof_one.py c2 > /dev/null 2>&1; echo n0=$?
python tools/launches.py gpurun_out/launches_c2.csv | head -8
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_check -c 1 -o gpurun_out/prof_check_c2 python tools/prof_one.py c2 > gpurun_out/ncu_chk_c2.log 2>&1; echo n2=$?
