#!/bin/bash
# 1 0 2 4 3 5 family (CCSD(T)): input runs beyond 4 KB (tile [n0, n1, k, ...], output run = i1) vs the auto plan
O=gpurun_out/exp51; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for c in 24,24,24,24,24,24:1,0,2,4,3,5:8 16,16,16,16,16,16:1,0,2,4,3,5:8 32,32,32,16,16,16:1,0,2,4,3,5:8; do
  python tools/sweep.py --case $c --reps 10 >> $O/sweep.jsonl 2>> $O/sweep.err
  for k in 2 3 4 6 8; do for v in 1 2; do
    python tools/sweep.py --case $c --reps 10 --hints "{\"in_dim\": 2, \"in_block\": $k, \"out_dim\": 0, \"variant\": $v}" >> $O/sweep.jsonl 2>> $O/sweep.err
  done; done
done
