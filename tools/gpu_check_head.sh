#!/bin/bash
# re-verify HEAD: build, smoke, full GPU parity, bench C4 (default) and C5
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > $O/nvsmi.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo smoke=$?
timeout 2400 python -m pytest tests -q -m gpu -p no:cacheprovider --timeout 900 > $O/pytest_gpu.log 2>&1; echo pytest=$?
tail -15 $O/pytest_gpu.log
timeout 900 python bench.py --no-ncu > $O/bench_c4.json 2> $O/bench_c4.err; echo c4=$?
timeout 1200 python bench.py --config c5 --steps 5 --no-cpu-baseline --no-ncu > $O/bench_c5.json 2> $O/bench_c5.err; echo c5=$?
for c in c4 c5; do timeout 20 python -c "
import json; d=json.load(open('$O/bench_$c.json')); print('$c', round(d['value']/1e9,3), 'Gev/s', round(d['ms_per_step'],4), 'ms', 'e2e', round(d['e2e']['value']/1e9,3), 'K7', round(d['roofline']['frac'],4), 'pipe', round(d['roofline_pipeline']['frac'],4), d.get('phases_ms'), d['clocks'])"; done
