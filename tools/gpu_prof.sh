python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_expand -c 1 -o gpurun_out/prof_expand_c4 python tools/prof_one.py c4 > /dev/null 2>&1; echo n1=$?
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_rs_downsweep -s 2 -c 1 -o gpurun_out/prof_down_c4 python tools/prof_one.py c4 > /dev/null 2>&1; echo n2=$?
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_header -c 1 -o gpurun_out/prof_header_c4 python tools/prof_one.py c4 > /dev/null 2>&1; echo n3=$?
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_replay -c 1 -o gpurun_out/prof_replay_c4 python tools/prof_one.py c4 > /dev/null 2>&1; echo n4=$?
