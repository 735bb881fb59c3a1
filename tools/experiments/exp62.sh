#!/bin/bash
# model regret on the 720-perm sweeps (measure mode beside the model) + bench smoke of the e2e change
O=gpurun_out/exp62; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for w in 720-15 720-17; do
  timeout 900 python bench.py --workload $w --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline --tune 8 > $O/bench_$w.json 2> $O/bench_$w.err
done
timeout 900 python bench.py --steps 3 --warmup 3 --e2e-steps 2 --no-cpu-baseline --tune 0 > $O/bench.json 2> $O/bench.err
