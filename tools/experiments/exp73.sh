#!/bin/bash
# bench with per-kernel graphs for the roofline pass (default run as the driver does it)
O=gpurun_out/exp73; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python bench.py > $O/bench.json 2> $O/bench.err
timeout 600 python bench.py --impl reference > $O/bench_ref.json 2> $O/bench_ref.err
for w in ccsdt smallfvi; do timeout 900 python bench.py --workload $w --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/bench_$w.json 2> $O/bench_$w.err; done
