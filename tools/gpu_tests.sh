#!/bin/bash
# build + smoke + GPU parity tests (args: extra pytest args, e.g. -k windows)
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > $O/nvsmi.txt; free -g >> $O/nvsmi.txt; nproc >> $O/nvsmi.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo smoke=$?
timeout ${PT_TIMEOUT:-1500} python -m pytest tests -q -m gpu -p no:cacheprovider --timeout 900 -x "$@" > $O/pytest_gpu.log 2>&1; echo pytest=$?
tail -30 $O/pytest_gpu.log
