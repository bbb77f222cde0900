#!/bin/bash
# Round evidence in one GPU call: build, smoke, full GPU parity suite, bench lines (C2 default with
# the CPU baseline, the reference arm, C1/C3/C4/C6, the ballot K7 variant), ncu launch lists and a
# full capture of the K7 kernel (C2, C4) from which the roofline `traffic` is taken.
O=gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/nvsmi.txt
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo smoke=$?
timeout 1200 python -m pytest tests -q -m "gpu" -p no:cacheprovider --timeout 600 > $O/pytest_gpu.log 2>&1; echo pytest=$?
tail -2 $O/pytest_gpu.log
timeout 600 python bench.py > $O/bench_c2.json 2> $O/bench_c2.err; echo bench=$?
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 > $O/bench_ref.json 2> $O/bench_ref.err; echo ref=$?
for c in c1 c3 c4 c6; do timeout 600 python bench.py --config $c --steps 5 --no-cpu-baseline > $O/bench_$c.json 2> $O/bench_$c.err; echo $c=$?; done
for c in c2 c4; do BC_K7=ballot timeout 600 python bench.py --config $c --steps 5 --no-cpu-baseline > $O/bench_${c}_ballot.json 2>/dev/null; done
for f in bench_c2 bench_c1 bench_c3 bench_c4 bench_c6 bench_c2_ballot bench_c4_ballot; do timeout 20 python -c "
import json; d=json.load(open('$O/$f.json')); print('$f', d['config']['workload'], round(d['value']/1e9,3), 'Gev/s', round(d['ms_per_step'],3), 'ms', 'e2e', round(d['e2e']['value']/1e9,3), 'roof', round(d['roofline']['frac'],4), d['phases_ms'], d.get('cpu_baseline',{}).get('value'))"; done
for c in c2 c4 c6; do
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $O/launches_$c.csv python tools/prof_one.py $c > /dev/null 2>&1; echo n_$c=$?
python tools/launches.py $O/launches_$c.csv > $O/launches_$c.txt 2>&1
done
for c in c2 c4; do
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_check -c 1 -o $O/prof_check_$c python tools/prof_one.py $c > $O/ncu_chk_$c.log 2>&1; echo f_$c=$?
python tools/ncu_summary.py $O/prof_check_$c.ncu-rep 12 > $O/ncu_check_$c.txt 2>&1
done
