#!/bin/bash
# new k_expand: parity subset + C4/C5 bench; K7 split (K7a / K7b) at KT_IPL 16 and 8 on C2 / C4
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 1500 python -m pytest tests -q -m gpu -p no:cacheprovider --timeout 600 -x > $O/pytest_ex.log 2>&1; echo pytest=$?
tail -2 $O/pytest_ex.log
for c in c4 c5; do timeout 900 python bench.py --config $c --steps 3 --no-cpu-baseline --no-ncu 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('default $c', round(d['ms_per_step'],4), d['phases_ms'])"; done
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv -k regex:"k_expand" --log-file $O/l_ex.csv python tools/prof_one.py c4 > /dev/null 2>&1; python tools/launches.py $O/l_ex.csv
for v in "" "-DKT_IPL_=8"; do
rm -f paper_conf_pldi_eizenbergppmd17_b200/lib/*.o paper_conf_pldi_eizenbergppmd17_b200/lib/libbc.so
BC_NVCC_FLAGS="$v" python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1 || echo buildfail $v
for c in c2 c4 c3; do
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv -k regex:"k_blk|k_check" --log-file $O/l_$c.csv python tools/prof_one.py $c > /dev/null 2>&1; echo "$v $c"; python tools/launches.py $O/l_$c.csv | tail -2
done
done
rm -f paper_conf_pldi_eizenbergppmd17_b200/lib/*.o paper_conf_pldi_eizenbergppmd17_b200/lib/libbc.so
