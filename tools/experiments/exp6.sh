#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 600 python tools/sweep.py --case 26214400:0:8 --case 52428800:0:4 --d2d --reps 10 --hints '{}' --hints '{"threads":512}' --hints '{"threads":1024}' --hints '{"in_block":1048576}' --hints '{"in_block":4096}' --hints '{"in_block":16384}' --hints '{"in_block":16384,"threads":512}' > gpurun_out/sweep6_copy.jsonl 2>&1
timeout 1500 python tools/calib_sweep.py --group c2 --max-cand 40 --threads 256,512 > gpurun_out/calib6_c2.jsonl 2> gpurun_out/calib6_c2.err
