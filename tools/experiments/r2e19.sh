#!/bin/bash
# round 2, call 19: small tensors ranked by the second tree set (its data include 0.25-32 MB)
mkdir -p gpurun_out/r2e19
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "config1 or rank1 or rank15 or extent_one or single_use or odd" > gpurun_out/r2e19/gputest.log 2>&1
echo "gputest rc=$?"; tail -1 gpurun_out/r2e19/gputest.log
for w in c1 fig13; do
  timeout 600 python tools/cases.py --workload $w --out gpurun_out/r2e19/cases_$w.json > gpurun_out/r2e19/cases_$w.log 2>&1
  tail -1 gpurun_out/r2e19/cases_$w.log | cut -c1-250
  timeout 900 python bench.py --workload $w --tune 0 > gpurun_out/r2e19/bench_$w.json 2> gpurun_out/r2e19/bench_$w.err
done
