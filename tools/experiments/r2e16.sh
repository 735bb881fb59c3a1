#!/bin/bash
# round 2, call 16: second opinion (cal33 trees re-rank the short list when the winner is
# predicted below 0.8 of copy speed) -- per-case tables A/B against r2e14/r2e15
mkdir -p gpurun_out/r2e16
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "scaled or variants or odd or rank6 or 720" > gpurun_out/r2e16/gputest.log 2>&1
echo "gputest rc=$?"; tail -1 gpurun_out/r2e16/gputest.log
for w in c2 c3 c4 720-15 720-16 720-17; do
  timeout 600 python tools/cases.py --workload $w --out gpurun_out/r2e16/cases_$w.json > gpurun_out/r2e16/cases_$w.log 2>&1
  tail -1 gpurun_out/r2e16/cases_$w.log | cut -c1-250
done
