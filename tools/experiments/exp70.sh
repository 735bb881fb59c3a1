#!/bin/bash
# final round check s4h + launch lists for CCSD(T) / small-FVI + full captures of every kernel family
NCU_KERNELS="quad direct pipe" bash tools/round_check.sh s4h
O=gpurun_out/s4h
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
timeout 900 ncu --metrics $M --clock-control none -k regex:k_ -s 75 -c 25 --csv --log-file $O/launches_smallfvi.csv \
  python bench.py --workload smallfvi --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline --tune 0 > /dev/null 2>&1
timeout 900 ncu --metrics $M --clock-control none -k regex:k_ -s 120 -c 40 --csv --log-file $O/launches_ccsdt.csv \
  python bench.py --workload ccsdt --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline --tune 0 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_deint -s 10 -c 1 -o $O/prof_deint \
  python bench.py --workload smallfvi --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline --tune 0 > /dev/null 2>&1
timeout 900 python tools/suite.py --groups c3 --out $O/suite_c3.jsonl > $O/suite_c3.log 2>&1
timeout 600 python bench.py --workload sharded --steps 5 --warmup 3 > $O/bench_sharded.json 2> $O/bench_sharded.err
