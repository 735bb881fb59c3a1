#!/bin/bash
# round 2, call 3: GPU tests after the batched-launch signature change; per-case
# tables with the cudaMemcpyAsync D2D denominator; ncu full captures of the weak cases
mkdir -p gpurun_out/r2e3
timeout 1500 python -m pytest tests -m gpu -x -q -k "not fullsize" > gpurun_out/r2e3/gputest.log 2>&1
echo "gputest rc=$?"; tail -3 gpurun_out/r2e3/gputest.log
for w in 720-15 720-17 fig13 c1 c4; do
  python tools/cases.py --workload $w --out gpurun_out/r2e3/cases_$w.json > gpurun_out/r2e3/cases_$w.log 2>&1
  tail -1 gpurun_out/r2e3/cases_$w.log | cut -c1-300
done
prof() {  # workload case-id tag
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_ -s 2 -c 1 \
    -o gpurun_out/r2e3/prof_$3 python tools/one_case.py $1 $2 3 > gpurun_out/r2e3/prof_$3.log 2>&1
}
prof c2 2053 c2_325104
prof c4 4006 c4_fms3
prof c4 4007 c4_210n3
prof c3 3014 c3_543210_24
prof 720-16 6120 s16_102345
prof 720-17 6585 s17_451230
prof c4 4011 c4_fms4
ls -la gpurun_out/r2e3/
