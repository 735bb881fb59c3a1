#!/bin/bash
# A/B: the bench step as a CUDA-graph replay vs direct launches
O=gpurun_out/exp71; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for r in 1 2; do for g in 0 1; do for w in ttc57 ccsdt smallfvi c1; do
  if [ $g = 1 ]; then G=--graph; else G=; fi
  timeout 600 python bench.py --workload $w --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --tune 0 $G > $O/bench_${w}_g${g}_r$r.json 2> $O/bench_${w}_g${g}_r$r.err
done; done; done
