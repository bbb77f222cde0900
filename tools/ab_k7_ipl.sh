#!/bin/bash
# k_expand parity subset on the default build, then A/B of the K7 block size (KT_IPL) on C2 / C3 / C4
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 1200 python -m pytest tests -q -m gpu -p no:cacheprovider --timeout 600 -x -k "c1 or litmus or random or window or infeasible or c4 or stream" > $O/pytest_ex.log 2>&1; echo pytest=$?
tail -2 $O/pytest_ex.log
for c in c4 c2 c3; do timeout 600 python bench.py --config $c --steps 5 --no-cpu-baseline --no-ncu 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('default $c', round(d['ms_per_step'],4), d['phases_ms'])"; done
for v in "-DKT_IPL_=8" "-DKT_IPL_=4"; do
rm -f paper_conf_pldi_eizenbergppmd17_b200/lib/*.o paper_conf_pldi_eizenbergppmd17_b200/lib/libbc.so
BC_NVCC_FLAGS="$v" python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1 || echo buildfail $v
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -p no:cacheprovider --timeout 600 -x -k "litmus or random or hot or long" > $O/pytest_ipl.log 2>&1; echo "pytest $v"=$?; tail -1 $O/pytest_ipl.log
for c in c4 c2 c3; do timeout 600 python bench.py --config $c --steps 5 --no-cpu-baseline --no-ncu 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('$v $c', round(d['ms_per_step'],4), d['phases_ms']['k_check'], d['roofline']['frac'])"; done
done
rm -f paper_conf_pldi_eizenbergppmd17_b200/lib/*.o paper_conf_pldi_eizenbergppmd17_b200/lib/libbc.so
