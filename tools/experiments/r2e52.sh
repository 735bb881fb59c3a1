#!/bin/bash
# round 2, call 52: A/B the tree pre-screen as challengers with a 5 % margin (TTLG_TREE_SCREEN=0/2):
# every workload's per-case table (graph timing), same box, back to back
O=gpurun_out/r2e52
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for w in c2 c3 c4 fig13 720-16 720-15 720-17 c1; do
  for c in 0 2; do
    TTLG_TREE_SCREEN=$c timeout 900 python tools/cases.py --workload $w --out $O/cases_${w}_ts$c.json > /dev/null 2> $O/cases_${w}_ts$c.err
  done
done
TTLG_TREE_SCREEN=2 timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "config1 or scaled or odd or rank6 or 720" > $O/t_sel.log 2>&1; tail -1 $O/t_sel.log
