set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 1500 python -m pytest tests -q -m gpu -p no:cacheprovider --timeout 900 > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err; echo b2=$?
timeout 900 python bench.py --config c4 --steps 5 > gpurun_out/bench_c4.json 2> gpurun_out/bench_c4.err; echo b4=$?
timeout 600 python bench.py --config c3 --steps 5 > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err; echo b3=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2.csv python bench.py --steps 1 --no-cpu-baseline > /dev/null 2>&1; echo n1=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_check -s 3 -c 1 -o gpurun_out/prof_check_c2 python bench.py --steps 1 --no-cpu-baseline > gpurun_out/ncu_full_c2.log 2>&1; echo n2=$?
cat gpurun_out/bench_c2.json gpurun_out/bench_c4.json gpurun_out/bench_c3.json
tail -3 gpurun_out/bench_c4.err
