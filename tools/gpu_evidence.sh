#!/bin/bash
# round evidence: build, smoke, full GPU parity, bench lines (C4 default + others), reference arm,
# launch lists, ncu --set full captures of the top C4 kernels and K7
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > $O/nvsmi.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo smoke=$?
timeout 2000 python -m pytest tests -q -m gpu -p no:cacheprovider --timeout 900 > $O/pytest_gpu.log 2>&1; echo pytest=$?
tail -2 $O/pytest_gpu.log
timeout 900 python bench.py > $O/bench_c4.json 2> $O/bench_c4.err; echo c4=$?
for c in c2 c3 c6 c6f; do timeout 600 python bench.py --config $c --steps 10 --no-cpu-baseline --no-ncu > $O/bench_$c.json 2> $O/bench_$c.err; echo $c=$?; done
timeout 1200 python bench.py --config c5 --steps 3 --no-cpu-baseline --no-ncu > $O/bench_c5.json 2> $O/bench_c5.err; echo c5=$?
timeout 900 python bench.py --impl reference --steps 2 --warmup 3 > $O/bench_ref.json 2> $O/bench_ref.err; echo ref=$?
for c in c4 c2 c3 c6 c6f c5; do timeout 20 python -c "
import json; d=json.load(open('$O/bench_$c.json')); print('$c', round(d['value']/1e9,3), 'Gev/s', round(d['ms_per_step'],4), 'ms', 'e2e', round(d['e2e']['value']/1e9,3), 'K7', round(d['roofline']['frac'],4), round(d['roofline']['kernel_ms'],4), d['roofline']['traffic'], 'pipe', round(d['roofline_pipeline']['frac'],4), 'win', d['config']['windows'], d['clocks'])"; done
for c in c4 c2 c3; do
  timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $O/launches_$c.csv python tools/prof_one.py $c > /dev/null 2>&1; echo n_$c=$?
  python tools/launches.py $O/launches_$c.csv > $O/launches_$c.txt 2>&1
  head -12 $O/launches_$c.txt
done
CFG=c4 KERNELS="k_expand k_rs_down k_header k_replay k_blk_sum k_check_tile" bash tools/gpu_ncu_k7_c4.sh > $O/ncu_all.log 2>&1; echo ncu=$?
