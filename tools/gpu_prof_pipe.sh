#!/bin/bash
# ncu full captures of the pipeline kernels other than K7: radix downsweep (C2, item sort),
# k_expand / k_replay / k_header (C4)
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_rs_down -s 2 -c 1 -o gpurun_out/prof_down_c2 python tools/prof_one.py c2 > gpurun_out/ncu_down_c2.log 2>&1; echo d=$?
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_rs_up -s 2 -c 1 -o gpurun_out/prof_up_c2 python tools/prof_one.py c2 > gpurun_out/ncu_up_c2.log 2>&1; echo u=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_expand|k_replay|k_header" -c 3 -o gpurun_out/prof_pipe_c4 python tools/prof_one.py c4 > gpurun_out/ncu_pipe_c4.log 2>&1; echo p=$?
