#!/bin/bash
# quick K7 iteration: build, K7-variant parity tests, bench C2/C4 for both K7 variants, ncu of K7 on C2
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -m "gpu" -p no:cacheprovider --timeout 300 -x -k "k7_variants or configs_reduced or random_traces_granules" > gpurun_out/pytest_k7.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_k7.log
for v in tile ballot; do for c in c2 c3 c4; do
BC_K7=$v timeout 300 python bench.py --config $c --steps 5 --no-cpu-baseline > gpurun_out/bench_${c}_$v.json 2> gpurun_out/bench_$c.err
timeout 20 python -c "
import json; d=json.load(open('gpurun_out/bench_${c}_$v.json')); print('$v $c', round(d['value']/1e9,3), 'Gev/s', round(d['ms_per_step'],3), 'ms', 'roof', round(d['roofline']['frac'],4), 'k_check', d['phases_ms']['k_check'])"
done; done
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_check -c 1 -o gpurun_out/prof_check_c2 python tools/prof_one.py c2 > gpurun_out/ncu_chk_c2.log 2>&1; echo n2=$?
