set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout 900 python -m pytest tests -q -m "gpu and not slow" -p no:cacheprovider --timeout 300 -x -k "c1 or fig or litmus" > gpurun_out/pytest1.log 2>&1; echo p1=$?
timeout 900 python -m pytest tests -q -m "gpu and not slow" -p no:cacheprovider --timeout 300 > gpurun_out/pytest2.log 2>&1; echo p2=$?
tail -30 gpurun_out/pytest2.log
