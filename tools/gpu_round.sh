#!/bin/bash
# One GPU call: build, GPU parity suite, bench lines, ncu launch list + full capture of k_check.
python -c "import __graft_entry__ as g; g.build()" || exit 1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/nvsmi.txt
cat MEASURED_PEAKS.json > gpurun_out/peaks.json 2>/dev/null
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout 900 python -m pytest tests -q -m "gpu" -p no:cacheprovider --timeout 300 > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
tail -2 gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; echo bench=$?
timeout 300 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err; echo ref=$?
for c in c3 c4; do timeout 300 python bench.py --config $c --steps 5 --no-cpu-baseline > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; echo $c=$?; done
BC_K7=seq timeout 300 python bench.py --config c4 --steps 5 --no-cpu-baseline > gpurun_out/bench_c4_seq.json 2> gpurun_out/bench_c4_seq.err; echo c4seq=$?
BC_K7=seq timeout 300 python bench.py --config c2 --steps 5 --no-cpu-baseline > gpurun_out/bench_c2_seq.json 2> gpurun_out/bench_c2_seq.err; echo c2seq=$?
for f in bench_default bench_c3 bench_c4 bench_c4_seq bench_c2_seq; do timeout 20 python -c "
import json; d=json.load(open('gpurun_out/$f.json')); print('$f', d['config']['workload'], round(d['value']/1e9,3), 'Gev/s', round(d['ms_per_step'],3), 'ms', 'e2e', round(d['e2e']['value']/1e9,3), 'roof', round(d['roofline']['frac'],4), d['phases_ms'], d.get('cpu_baseline',{}).get('value'))"; done
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_c2.csv python tools/prof_one.py c2 > /dev/null 2>&1; echo n0=$?
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_c4.csv python tools/prof_one.py c4 > /dev/null 2>&1; echo n1=$?
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_check -c 1 -o gpurun_out/prof_check_c2 python tools/prof_one.py c2 > gpurun_out/ncu_chk_c2.log 2>&1; echo n2=$?
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_check -c 1 -o gpurun_out/prof_check_c4 python tools/prof_one.py c4 > gpurun_out/ncu_chk_c4.log 2>&1; echo n3=$?
