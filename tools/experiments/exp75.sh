#!/bin/bash
# N3 workloads and config 1 with the graph-replayed step
O=gpurun_out/exp75; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for w in 720-15 720-16 720-17 fig13 c1; do
  TTLG_BENCH_CASES=1 timeout 900 python bench.py --workload $w --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline --tune 0 > $O/bench_$w.json 2> $O/bench_$w.err
done
