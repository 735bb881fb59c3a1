#!/bin/bash
# round 2, call 4: k_bulk (TMA bulk row loads + mbarrier ring) parity, then
# per-case timing of the auto slices run by k_bulk vs the auto plans
mkdir -p gpurun_out/r2e4
timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "bulk or variants_forced or execute_batch" > gpurun_out/r2e4/gputest.log 2>&1
rc=$?; echo "bulk tests rc=$rc"; tail -15 gpurun_out/r2e4/gputest.log
if [ $rc -ne 0 ]; then exit 1; fi
for w in c2 c3 c4; do
  timeout 300 python tools/cases.py --workload $w --bulk --out gpurun_out/r2e4/bulk_$w.json > gpurun_out/r2e4/bulk_$w.log 2>&1
  tail -1 gpurun_out/r2e4/bulk_$w.log | cut -c1-400
  timeout 300 python tools/cases.py --workload $w --out gpurun_out/r2e4/auto_$w.json > gpurun_out/r2e4/auto_$w.log 2>&1
  tail -1 gpurun_out/r2e4/auto_$w.log | cut -c1-400
done
