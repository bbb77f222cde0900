#!/bin/bash
# A/B: K7a stages / tile unroll, k_expand residency (C4 launch times), parity subset per variant
O=gpurun_out
mkdir -p $O
for v in "" "-DKB_STAGES_=3" "-DKB_STAGES_=3 -DKA_UNROLL=2" "-DKB_STAGES_=4 -DKA_UNROLL=2" "-DEX_MINB=4"; do
rm -f paper_conf_pldi_eizenbergppmd17_b200/lib/*.o paper_conf_pldi_eizenbergppmd17_b200/lib/libbc.so
BC_NVCC_FLAGS="$v" python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1 || echo buildfail $v
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -p no:cacheprovider --timeout 600 -x -k "litmus or random or hot or long or c4 or window" > $O/pytest_ab.log 2>&1; echo "pytest [$v]"=$?; tail -1 $O/pytest_ab.log
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv -k regex:"k_blk|k_check|k_expand" --log-file $O/lab.csv python tools/prof_one.py c4 > /dev/null 2>&1; echo "[$v] c4"; python tools/launches.py $O/lab.csv | tail -3
done
rm -f paper_conf_pldi_eizenbergppmd17_b200/lib/*.o paper_conf_pldi_eizenbergppmd17_b200/lib/libbc.so
