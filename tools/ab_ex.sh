#!/bin/bash
# A/B of k_expand chunking (records per chunk x stages in flight) on C2 / C4
for v in "-DEX_REC_=64 -DEX_STAGES_=2" "-DEX_REC_=128 -DEX_STAGES_=2" "-DEX_REC_=128 -DEX_STAGES_=3" "-DEX_REC_=256 -DEX_STAGES_=2"; do
rm -f paper_conf_pldi_eizenbergppmd17_b200/lib/*.o paper_conf_pldi_eizenbergppmd17_b200/lib/libbc.so
BC_NVCC_FLAGS="$v" python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
for c in c2 c4; do python bench.py --config $c --steps 5 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('$v $c', round(d['ms_per_step'],4), d['phases_ms']['k_expand'])"; done
done
