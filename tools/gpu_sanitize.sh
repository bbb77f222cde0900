#!/bin/bash
O=gpurun_out
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || exit 1
for t in memcheck racecheck synccheck initcheck; do
  timeout 1500 compute-sanitizer --tool $t --launch-timeout 0 --print-limit 50 python tools/sanitize_one.py > $O/sanitize_$t.log 2>&1; echo $t=$?
  tail -4 $O/sanitize_$t.log
done
