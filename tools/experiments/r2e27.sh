#!/bin/bash
# round 2, call 27: k_direct tiles capped at ~1.3 load rounds per thread at 4/8-byte access
O=gpurun_out/r2e27
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for w in fig13 fmlrows 720-15 720-17 720-16 c2 c3 c1; do
  timeout 600 python tools/cases.py --workload $w --out $O/cases_$w.json > /dev/null 2>&1
done
