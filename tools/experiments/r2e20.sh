#!/bin/bash
# round 2, call 20: k_rows (16-byte FML rows with head/tail) -- parity, A/B against k_direct
mkdir -p gpurun_out/r2e20
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "rows or odd or config1 or rank6 or 720 or scaled or misaligned or direct or strided" > gpurun_out/r2e20/gputest.log 2>&1
rc=$?; echo "gputest rc=$rc"; tail -3 gpurun_out/r2e20/gputest.log; [ $rc -ne 0 ] && exit 1
timeout 900 python -m pytest tests/test_strided.py tests/test_sharded.py -x -q -m gpu > gpurun_out/r2e20/gputest2.log 2>&1; echo "strided rc=$?"; tail -1 gpurun_out/r2e20/gputest2.log
for w in fig13 720-15 720-17; do
  for m in 0 1; do
    TTLG_ROWS=$m timeout 600 python tools/cases.py --workload $w --out gpurun_out/r2e20/cases_${w}_rows$m.json > gpurun_out/r2e20/cases_${w}_$m.log 2>&1
    tail -1 gpurun_out/r2e20/cases_${w}_$m.log | cut -c1-200
  done
done
