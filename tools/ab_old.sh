#!/bin/bash
for h in v1 v2; do
(cd old_tree/$h && python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1; for c in c2 c4; do python bench.py --config $c --steps 5 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('$h $c', round(d['ms_per_step'],4), d['phases_ms']['k_check'], d['roofline']['clock_gathers'])"; done)
done
