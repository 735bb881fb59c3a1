#!/bin/bash
# graph-replay headline: full GPU suite + default bench + the other workloads
O=gpurun_out/exp72; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 1500 python -m pytest tests -m gpu -q > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
TTLG_BENCH_CASES=1 timeout 900 python bench.py --steps 10 --warmup 3 > $O/bench.json 2> $O/bench.err
for w in ccsdt smallfvi; do TTLG_BENCH_CASES=1 timeout 900 python bench.py --workload $w --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/bench_$w.json 2> $O/bench_$w.err; done
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
  -k regex:k_ -s 171 -c 57 --csv --log-file $O/launches.csv \
  python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline --tune 0 > /dev/null 2>&1
