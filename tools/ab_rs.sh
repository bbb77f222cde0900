#!/bin/bash
# A/B of the radix tile (keys per thread) and downsweep staging on C2 / C4
for v in "-DRS_ITEMS_=28 -DRS_DSTAGES_=2" "-DRS_ITEMS_=32 -DRS_DSTAGES_=2" "-DRS_ITEMS_=32 -DRS_DSTAGES_=1"; do
rm -f paper_conf_pldi_eizenbergppmd17_b200/lib/*.o paper_conf_pldi_eizenbergppmd17_b200/lib/libbc.so
BC_NVCC_FLAGS="$v" python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
for c in c2 c4; do python bench.py --config $c --steps 5 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('$v $c', round(d['ms_per_step'],4), d['phases_ms']['sort'], d['phases_ms']['partition'])"; done
done
