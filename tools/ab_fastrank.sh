#!/bin/bash
# A/B: shuffle + vote fast paths before MATCH.ANY in the radix downsweep (RS_FASTRANK=1) vs MATCH.ANY only
O=gpurun_out
for v in "-DRS_FASTRANK=1" "-DRS_FASTRANK=0" "-DRS_FASTRANK=1"; do
rm -f paper_conf_pldi_eizenbergppmd17_b200/lib/*.o paper_conf_pldi_eizenbergppmd17_b200/lib/libbc.so
BC_NVCC_FLAGS="$v" python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1 || { echo build_fail; exit 1; }
for c in c2 c3 c4; do timeout 300 python bench.py --config $c --steps 10 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('$v $c', round(d['ms_per_step'],4), 'sort', d['phases_ms']['sort'], 'part', d['phases_ms']['partition'], 'sync', d['phases_ms']['sync'])"; done
done
timeout 900 python -m pytest tests -q -m gpu -p no:cacheprovider --timeout 600 -x > $O/pytest_gpu.log 2>&1; echo pytest=$?
tail -1 $O/pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo smoke=$?
