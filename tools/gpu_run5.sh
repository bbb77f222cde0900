python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python -m pytest tests -q -m "gpu" -p no:cacheprovider --timeout 300 -x > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
tail -2 gpurun_out/pytest_gpu.log
for c in c2 c3 c4; do timeout 300 python bench.py --config $c --steps 5 --no-cpu-baseline > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; echo $c=$?; timeout 20 python -c "
import json; d=json.load(open('gpurun_out/bench_$c.json')); print('$c', round(d['value']/1e9,2), 'Gev/s', round(d['ms_per_step'],3), 'ms', 'e2e', round(d['e2e']['value']/1e9,2), 'roof', round(d['roofline']['frac'],4), d['phases_ms'])"; done
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_rs_onesweep -s 8 -c 1 -o gpurun_out/prof_sort_c4 python bench.py --config c4 --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_sort_c4.log 2>&1; echo n1=$?
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_check -s 3 -c 1 -o gpurun_out/prof_check_c4 python bench.py --config c4 --steps 1 --no-cpu-baseline > gpurun_out/ncu_chk_c4.log 2>&1; echo n2=$?
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_check -s 3 -c 1 -o gpurun_out/prof_check_c2 python bench.py --config c2 --steps 1 --no-cpu-baseline > gpurun_out/ncu_chk_c2.log 2>&1; echo n3=$?
