#!/bin/bash
# round 2, call 9: calibration sweep cal33 (every kernel incl. k_vec / k_bulk; small sizes)
mkdir -p gpurun_out/r2e9
export TTLG_VEC=1 TTLG_BULK=1
run() { timeout 1200 python tools/calib_sweep.py "$@" ; }
run --group c2 --max-cand 60 > gpurun_out/r2e9/cal33_c2.jsonl 2> gpurun_out/r2e9/c2.err
run --group c3 --max-cand 60 > gpurun_out/r2e9/cal33_c3.jsonl 2> gpurun_out/r2e9/c3.err
run --group c4 --max-cand 80 > gpurun_out/r2e9/cal33_c4.jsonl 2> gpurun_out/r2e9/c4.err
run --group c1 --max-cand 40 > gpurun_out/r2e9/cal33_c1.jsonl 2> gpurun_out/r2e9/c1.err
run --recipe 120 --seed 11 --max-cand 48 > gpurun_out/r2e9/cal33_recipe.jsonl 2> gpurun_out/r2e9/recipe.err
run --recipe 100 --seed 12 --lo-mb 0.25 --hi-mb 32 --log-size --max-cand 40 > gpurun_out/r2e9/cal33_small.jsonl 2> gpurun_out/r2e9/small.err
run --group c2 --max-cand 24 --top > gpurun_out/r2e9/cal33_c2top.jsonl 2> gpurun_out/r2e9/c2top.err
run --group c4 --max-cand 24 --top > gpurun_out/r2e9/cal33_c4top.jsonl 2> gpurun_out/r2e9/c4top.err
wc -l gpurun_out/r2e9/*.jsonl
tail -3 gpurun_out/r2e9/*.err
gzip -f gpurun_out/r2e9/*.jsonl
