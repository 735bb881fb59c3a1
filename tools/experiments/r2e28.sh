#!/bin/bash
# round 2, call 28: the closed 16x16 / 24x24 leading-block family (`1 0 ...`): hinted slices
O=gpurun_out/r2e28
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
i=0
for h in '{}' \
  '{"variant": 7, "in_dim": 2, "in_block": 8, "out_dim": 1, "out_block": 16}' \
  '{"variant": 7, "in_dim": 2, "in_block": 4, "out_dim": 1, "out_block": 16}' \
  '{"variant": 7, "in_dim": 2, "in_block": 2, "out_dim": 1, "out_block": 16}' \
  '{"variant": 7, "in_dim": 2, "in_block": 16, "out_dim": 1, "out_block": 16}' \
  '{"variant": 1, "in_dim": 2, "in_block": 8, "out_dim": 1, "out_block": 16}' \
  '{"variant": 1, "in_dim": 2, "in_block": 4, "out_dim": 1, "out_block": 16}' \
  '{"variant": 2, "in_dim": 2, "in_block": 8, "out_dim": 1, "out_block": 16}' \
  '{"variant": 7, "in_dim": 2, "in_block": 8, "out_dim": 1, "out_block": 16, "threads": 512}' \
  '{"variant": 6, "in_dim": 2, "in_block": 8, "out_dim": 1, "out_block": 16}' ; do
  timeout 300 python tools/cases.py --workload 720-16 --only 6120,6122,6126,6129 --hints "$h" --out $O/s16_$i.json > /dev/null 2> $O/s16_$i.err
  echo "$i $h" >> $O/hints.txt
  i=$((i+1))
done
i=0
for h in '{}' \
  '{"variant": 7, "in_dim": 2, "in_block": 4, "out_dim": 1, "out_block": 24}' \
  '{"variant": 7, "in_dim": 2, "in_block": 2, "out_dim": 1, "out_block": 24}' \
  '{"variant": 7, "in_dim": 2, "in_block": 8, "out_dim": 1, "out_block": 24}' \
  '{"variant": 1, "in_dim": 2, "in_block": 4, "out_dim": 1, "out_block": 24}' \
  '{"variant": 1, "in_dim": 2, "in_block": 2, "out_dim": 1, "out_block": 24}'; do
  timeout 300 python tools/cases.py --workload c3 --only 3016 --hints "$h" --out $O/c3_$i.json > /dev/null 2> $O/c3_$i.err
  echo "c3 $i $h" >> $O/hints.txt
  i=$((i+1))
done
