#!/bin/bash
# round 2, call 7: every k_bulk candidate vs the auto plan (graph timing), configs 2-4
mkdir -p gpurun_out/r2e7
timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "bulk" > gpurun_out/r2e7/gputest.log 2>&1 || { tail -20 gpurun_out/r2e7/gputest.log; exit 1; }
for w in c2 c3 c4; do
  timeout 900 python tools/bulk_sweep.py --workload $w --max-cand 80 > gpurun_out/r2e7/sweep_$w.jsonl 2> gpurun_out/r2e7/sweep_$w.err
  grep summary gpurun_out/r2e7/sweep_$w.jsonl | wc -l
done
gzip -f gpurun_out/r2e7/sweep_*.jsonl
