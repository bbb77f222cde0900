#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
timeout 800 python -m pytest tests/test_gpu_parity.py tests/test_shard.py -q -m gpu -p no:cacheprovider --timeout 300 -x 2>&1 | tail -2
for c in c1 c3 c6 c2; do python bench.py --config $c --steps 5 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('$c', round(d['ms_per_step'],4), d['phases_ms']['sync'], d['phases_ms']['partition'])"; done
