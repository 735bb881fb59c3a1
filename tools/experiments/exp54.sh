#!/bin/bash
# N3: the paper's second workloads (720 perms of 15^6/16^6/17^6, Fig. 13 sizes) + config 1 + sharded config 5
O=gpurun_out/exp54; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for w in 720-15 720-16 720-17 fig13 c1; do
  TTLG_BENCH_CASES=1 timeout 900 python bench.py --workload $w --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline --tune 0 > $O/bench_$w.json 2> $O/bench_$w.err
done
timeout 600 python bench.py --workload sharded --steps 5 --warmup 3 > $O/bench_sharded.json 2> $O/bench_sharded.err
