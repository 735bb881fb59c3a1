#!/bin/bash
# round check on the recalibrated model + plan-time and single/repeated-use on the box CPU
bash tools/round_check.sh s3d
O=gpurun_out/s3d
g++ -O2 -std=c++17 -I include tools/plantime.cpp -L paper_conf_ipps_veduradasskhpkn18_b200 -lttlg \
  -Wl,-rpath,$PWD/paper_conf_ipps_veduradasskhpkn18_b200 -o /tmp/plantime 2>/dev/null
for c in "8 6 16 16 16 16 16 16 4 1 2 5 3 0" "8 2 5120 5120 1 0" "8 5 32 32 25 32 32 2 0 4 1 3" "4 3 4 4096 4096 1 2 0" "8 6 24 24 24 24 24 24 5 4 3 2 1 0"; do
  echo "$c" | /tmp/plantime >> $O/plantime.txt 2>&1
done
lscpu | head -20 > $O/cpu.txt
timeout 1200 python tools/suite.py --groups c1,c3,c5 --out $O/suite.jsonl > $O/suite.log 2>&1
