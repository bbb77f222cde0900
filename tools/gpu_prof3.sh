#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_rs_down -s 2 -c 1 -o gpurun_out/prof_down_c2 python tools/prof_one.py c2 > gpurun_out/ncu_down_c2.log 2>&1; echo n1=$?
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_replay -c 1 -o gpurun_out/prof_replay_c4 python tools/prof_one.py c4 > gpurun_out/ncu_replay_c4.log 2>&1; echo n2=$?
