python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python -m pytest tests -q -m "gpu" -p no:cacheprovider --timeout 300 > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_gpu.log
timeout 300 python bench.py --config c4 --steps 5 --no-cpu-baseline > gpurun_out/bench_c4.json 2> gpurun_out/bench_c4.err; echo c4=$?
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_expand -s 3 -c 1 -o gpurun_out/prof_expand_c4 python bench.py --config c4 --steps 1 --no-cpu-baseline > gpurun_out/ncu_exp_c4.log 2>&1; echo n1=$?
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_check -s 3 -c 1 -o gpurun_out/prof_check_c3 python bench.py --config c3 --steps 1 --no-cpu-baseline > gpurun_out/ncu_chk_c3.log 2>&1; echo n2=$?
