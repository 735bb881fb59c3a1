#!/bin/bash
# round 2, call 13: k_vec with the gather-conflict padding; small closed-block deep tiles
mkdir -p gpurun_out/r2e13
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "bulk or variants_forced or closed or all_720" > gpurun_out/r2e13/gputest.log 2>&1
echo "gputest rc=$?"; tail -2 gpurun_out/r2e13/gputest.log
timeout 900 python tools/bulk_sweep.py --workload c4 --variants 7 --max-cand 80 --only 4006,4016,4007,4002 > gpurun_out/r2e13/vec_c4.jsonl 2> gpurun_out/r2e13/vec_c4.err
grep summary gpurun_out/r2e13/vec_c4.jsonl | cut -c1-300
for w in c4 c3 720-16; do
  timeout 600 python tools/cases.py --workload $w --out gpurun_out/r2e13/cases_$w.json > gpurun_out/r2e13/cases_$w.log 2>&1
  tail -1 gpurun_out/r2e13/cases_$w.log | cut -c1-300
done
gzip -f gpurun_out/r2e13/*.jsonl
