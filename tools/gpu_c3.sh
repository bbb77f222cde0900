#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 300 python bench.py --config c3 --steps 5 --no-cpu-baseline > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err; echo c3=$?
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c3.csv python tools/prof_one.py c3 > /dev/null 2>&1; echo n0=$?
python tools/launches.py gpurun_out/launches_c3.csv
