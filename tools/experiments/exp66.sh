#!/bin/bash
# staged k_deint at n0 = 7, 8 vs the auto plan (k_quad / k_pipe)
O=gpurun_out/exp66; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for n0 in 7 8; do for p in 1,0,2 1,2,0; do
  python tools/sweep.py --case $n0,4096,4096:$p:4 --reps 10 >> $O/auto.jsonl 2>> $O/err
  python tools/sweep.py --case $n0,4096,4096:$p:4 --reps 10 --hints '{"variant": 4}' >> $O/deint.jsonl 2>> $O/err
done; done
for n0 in 7 8; do
  python tools/sweep.py --case 4,4096,4096:1,0,2:8 --reps 10 >> $O/auto64.jsonl 2>> $O/err
  python tools/sweep.py --case 4,4096,4096:1,0,2:8 --reps 10 --hints '{"variant": 4}' >> $O/deint64.jsonl 2>> $O/err
done
