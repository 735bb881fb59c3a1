#!/bin/bash
# round 2, call 5: k_bulk with cp.async row chunks (short rows) vs TMA rows
mkdir -p gpurun_out/r2e5
for m in 0 1; do
TTLG_BULK_TMA=$m timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "bulk or variants_forced or execute_batch" > gpurun_out/r2e5/gputest_$m.log 2>&1
rc=$?; echo "bulk tests tma=$m rc=$rc"; tail -3 gpurun_out/r2e5/gputest_$m.log
if [ $rc -ne 0 ]; then exit 1; fi
done
for w in c2 c3 c4; do
  TTLG_BULK_TMA=0 timeout 300 python tools/cases.py --workload $w --bulk --out gpurun_out/r2e5/bulk0_$w.json > gpurun_out/r2e5/bulk0_$w.log 2>&1
  tail -1 gpurun_out/r2e5/bulk0_$w.log | cut -c1-300
  timeout 300 python tools/cases.py --workload $w --bulk --out gpurun_out/r2e5/bulkA_$w.json > gpurun_out/r2e5/bulkA_$w.log 2>&1
  tail -1 gpurun_out/r2e5/bulkA_$w.log | cut -c1-300
done
