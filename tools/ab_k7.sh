#!/bin/bash
# A/B of K7 tile build variants (compile-time macros) on C2 / C3 / C4
for v in "-DKT_IPL_=16 -DKT_NWARPS=16" "-DKT_IPL_=8 -DKT_NWARPS=20" "-DKT_IPL_=12 -DKT_NWARPS=16" "-DKT_IPL_=32 -DKT_NWARPS=8"; do
rm -f paper_conf_pldi_eizenbergppmd17_b200/lib/*.o paper_conf_pldi_eizenbergppmd17_b200/lib/libbc.so
BC_NVCC_FLAGS="$v" python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
for c in c2 c3 c4; do python bench.py --config $c --steps 5 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('$v $c', round(d['ms_per_step'],4), d['phases_ms']['k_check'])"; done
done
