#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
for c in c2 c3 c4; do python bench.py --config $c --steps 5 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('$c', round(d['ms_per_step'],4), d['phases_ms']['sort'], d['phases_ms']['partition'])"; done
timeout 300 python -m pytest tests/test_gpu_parity.py -q -m gpu -p no:cacheprovider -x -k "random_traces or configs_reduced or hot_granule" 2>&1 | tail -1
