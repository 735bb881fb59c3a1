#!/bin/bash
# round 2, call 12: two-tree-set ranking (round-1 trees + k_vec challenge under the cal33 trees)
mkdir -p gpurun_out/r2e12
timeout 900 python -m pytest tests -m gpu -x -q -k "not fullsize" > gpurun_out/r2e12/gputest.log 2>&1
echo "gputest rc=$?"; tail -2 gpurun_out/r2e12/gputest.log
for w in c2 c3 c4 c1 fig13 720-15 720-16 720-17; do
  timeout 600 python tools/cases.py --workload $w --out gpurun_out/r2e12/cases_$w.json > gpurun_out/r2e12/cases_$w.log 2>&1
  tail -1 gpurun_out/r2e12/cases_$w.log | cut -c1-300
done
timeout 900 python bench.py > gpurun_out/r2e12/bench.json 2> gpurun_out/r2e12/bench.err
tail -c 1200 gpurun_out/r2e12/bench.json
