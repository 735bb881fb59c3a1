#!/bin/bash
# round check (s4c) + config-3 single/repeated-use suite + sharded bench + plan time on the box CPU
bash tools/round_check.sh s4c
O=gpurun_out/s4c
timeout 900 python tools/suite.py --groups c3 --out $O/suite_c3.jsonl > $O/suite_c3.log 2>&1
timeout 600 python bench.py --workload sharded --steps 5 --warmup 3 > $O/bench_sharded.json 2> $O/bench_sharded.err
g++ -O2 -std=c++17 -I include tools/plantime.cpp -L paper_conf_ipps_veduradasskhpkn18_b200 -lttlg -Wl,-rpath,$PWD/paper_conf_ipps_veduradasskhpkn18_b200 -o /tmp/plantime && \
printf "8 6 16 16 16 16 16 16 0 2 5 1 4 3\n8 6 16 16 16 16 16 16 4 1 2 5 3 0\n8 6 16 16 16 16 16 16 5 4 3 2 1 0\n8 6 16 16 16 16 16 16 2 1 0 5 4 3\n8 2 5120 5120 1 0\n4 3 3 4096 4096 0 2 1\n" | /tmp/plantime > $O/plantime.txt 2>&1
