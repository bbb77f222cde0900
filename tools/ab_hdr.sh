#!/bin/bash
for v in "-DHDR_ROWS=8" "-DHDR_ROWS=16" "-DHDR_ROWS=4"; do
rm -f paper_conf_pldi_eizenbergppmd17_b200/lib/*.o paper_conf_pldi_eizenbergppmd17_b200/lib/libbc.so
BC_NVCC_FLAGS="$v" python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
for c in c2 c4; do python bench.py --config $c --steps 5 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('$v $c', round(d['ms_per_step'],4), d['phases_ms']['header'], d['phases_ms']['replay'])"; done
done
