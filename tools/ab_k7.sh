#!/bin/bash
# A/B of K7 variants on C2: HEAD, STK/VIS reverted, same_value/gat reverted
run() { python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1; for i in 1 2; do python bench.py --config c2 --steps 10 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('$1', round(d['ms_per_step'],4), d['phases_ms']['k_check'])"; done; }
run A
sed -i 's/constexpr int STK = 256, VIS = 256;/constexpr int STK = 96, VIS = 160;/' paper_conf_pldi_eizenbergppmd17_b200/csrc/common.cuh
run B
sed -i 's/constexpr int STK = 96, VIS = 160;/constexpr int STK = 256, VIS = 256;/' paper_conf_pldi_eizenbergppmd17_b200/csrc/common.cuh
sed -i 's/same_value(a, we, e);  \/\/ P:L577-581/(we >> 5) == (e >> 5);  \/\/ P:L577-581/; s/          ++gat;$//' paper_conf_pldi_eizenbergppmd17_b200/csrc/check.cu
run C
