#!/bin/bash
# round 2, call 45: every candidate of the FML cases on k_direct -- Fig. 13 127^4 / 63^4 / 31^4
# `0 2 1 3` and six 17^6 FML perms -- to find what separates the fast and slow k_direct tiles
O=gpurun_out/r2e45
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1200 python tools/bulk_sweep.py --workload fig13 --only 7006,7004,7002 --variants 0 --max-cand 300 --reps 5 > $O/sweep_fig13.jsonl 2> $O/sweep_fig13.err
timeout 1200 python tools/bulk_sweep.py --workload 720-17 --only 6001,6005,6009,6013,6017,6021 --variants 0 --max-cand 150 --reps 5 > $O/sweep_17fml.jsonl 2> $O/sweep_17fml.err
