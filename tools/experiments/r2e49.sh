#!/bin/bash
# round 2, call 49: every k_quad (3), k_tile (1), k_pipe (2) slice of the three weakest TTC cases
O=gpurun_out/r2e49
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1500 python tools/bulk_sweep.py --workload c2 --only 2047,2053,2057 --variants 3,1,2 --max-cand 400 --reps 5 > $O/sweep_ttc_weak.jsonl 2> $O/sweep_ttc_weak.err
