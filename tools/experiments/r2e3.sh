#!/bin/bash
# round 2, call 3b: GPU tests after the batched-launch + generalized k_quad changes;
# ncu full captures of the weak cases (summarised on the box, reports not kept)
mkdir -p gpurun_out/r2e3
timeout 1500 python -m pytest tests -m gpu -x -q -k "not fullsize" > gpurun_out/r2e3/gputest.log 2>&1
echo "gputest rc=$?"; tail -30 gpurun_out/r2e3/gputest.log
prof() {  # workload case-id tag
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_ -s 2 -c 1 \
    -o /tmp/prof_$3 python tools/one_case.py $1 $2 3 > gpurun_out/r2e3/prof_$3.log 2>&1
  python tools/ncu_summary.py /tmp/prof_$3.ncu-rep > gpurun_out/r2e3/sum_$3.txt 2>&1
  ncu -i /tmp/prof_$3.ncu-rep --page raw --csv > gpurun_out/r2e3/raw_$3.csv 2>/dev/null
  ncu -i /tmp/prof_$3.ncu-rep --page source --csv > gpurun_out/r2e3/src_$3.csv 2>/dev/null
  gzip -f gpurun_out/r2e3/src_$3.csv
}
prof c2 2053 c2_325104
prof c4 4006 c4_fms3
prof c4 4007 c4_210n3
prof c3 3014 c3_543210_24
prof 720-16 6120 s16_102345
prof 720-17 6585 s17_451230
prof c4 4011 c4_fms4
du -sh gpurun_out/r2e3
