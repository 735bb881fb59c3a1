#!/bin/bash
# graph replay with / without programmatic dependent launch on the kernel nodes
O=gpurun_out/exp74; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for r in 1 2; do for p in 0 1; do for w in ttc57 smallfvi ccsdt; do
  TTLG_PDL=$p timeout 600 python bench.py --workload $w --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --tune 0 > $O/bench_${w}_p${p}_r$r.json 2> $O/bench_${w}_p${p}_r$r.err
done; done; done
