#!/bin/bash
# round 2, call 21: ncu --set full of every remaining case below 0.9 of the same-size D2D copy
mkdir -p gpurun_out/r2e21
prof() {  # tag workload case-id
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_ -s 2 -c 1 \
    -o /tmp/prof_$1 python tools/one_case.py $2 $3 3 > gpurun_out/r2e21/prof_$1.log 2>&1
  python tools/ncu_summary.py /tmp/prof_$1.ncu-rep > gpurun_out/r2e21/sum_$1.txt 2>&1
  head -1 gpurun_out/r2e21/sum_$1.txt
}
prof c2_2057_543210 c2 2057
prof c2_2053_325104 c2 2053
prof c3_3008_102435 c3 3008
prof c3_3012_412530 c3 3012
prof c3_3014_543210 c3 3014
prof c4_4002_210n2 c4 4002
prof c4_4005_201n2 c4 4005
prof c4_4007_210n3 c4 4007
prof c4_4008_deint3 c4 4008
prof c4_4011_021n4 c4 4011
prof s16_6128_103425 720-16 6128
prof s16_6096_051234 720-16 6096
