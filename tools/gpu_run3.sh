python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 1500 python -m pytest tests -q -m "gpu and not slow" -p no:cacheprovider --timeout 900 -x > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_gpu.log
for c in c2 c3 c4; do timeout 900 python bench.py --config $c --steps 5 --no-cpu-baseline > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; echo $c=$?; python -c "
import json; d=json.load(open('gpurun_out/bench_$c.json')); print('$c', round(d['value']/1e9,2), 'Gev/s', round(d['ms_per_step'],3), 'ms', 'e2e', round(d['e2e']['value']/1e9,2), 'roof', round(d['roofline']['frac'],4), d['phases_ms'])"; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_check -s 3 -c 1 -o gpurun_out/prof_check_c2 python bench.py --steps 1 --no-cpu-baseline > gpurun_out/ncu_full_c2.log 2>&1; echo n2=$?
