#!/bin/bash
O=gpurun_out
mkdir -p $O
for v in "" "-DKT_NWARPS=8" "-DKT_NWARPS=12"; do
rm -f paper_conf_pldi_eizenbergppmd17_b200/lib/*.o paper_conf_pldi_eizenbergppmd17_b200/lib/libbc.so
BC_NVCC_FLAGS="$v" python -c "import __graft_entry__ as g; g.build()" > $O/build_ab.log 2>&1 || { echo buildfail $v; tail -5 $O/build_ab.log; }
grep -A3 "k_check_tileILb0" $O/build_ab.log | grep -E "spill|Used" | head -2
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -p no:cacheprovider --timeout 600 -x -k "litmus or random or hot or long or c2 or c3" > $O/pytest_ab.log 2>&1; echo "pytest [$v]"=$?; tail -1 $O/pytest_ab.log
for c in c2 c3 c4; do
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv -k regex:"k_check_tile" --log-file $O/lab.csv python tools/prof_one.py $c > /dev/null 2>&1; echo "[$v] $c"; python tools/launches.py $O/lab.csv | tail -1
done
done
rm -f paper_conf_pldi_eizenbergppmd17_b200/lib/*.o paper_conf_pldi_eizenbergppmd17_b200/lib/libbc.so
