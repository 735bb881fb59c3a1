#!/bin/bash
# round 2, call 10: model recalibrated (cal33: k_vec in the automatic choice);
# per-case tables for every workload, default bench, GPU tests
mkdir -p gpurun_out/r2e10
timeout 900 python -m pytest tests -m gpu -x -q -k "not fullsize" > gpurun_out/r2e10/gputest.log 2>&1
echo "gputest rc=$?"; tail -3 gpurun_out/r2e10/gputest.log
for w in c2 c3 c4 c1 fig13 720-15 720-16 720-17; do
  timeout 600 python tools/cases.py --workload $w --out gpurun_out/r2e10/cases_$w.json > gpurun_out/r2e10/cases_$w.log 2>&1
  tail -1 gpurun_out/r2e10/cases_$w.log | cut -c1-330
done
timeout 900 python bench.py > gpurun_out/r2e10/bench.json 2> gpurun_out/r2e10/bench.err
tail -c 1500 gpurun_out/r2e10/bench.json
