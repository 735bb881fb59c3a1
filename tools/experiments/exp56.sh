#!/bin/bash
# A/B/C/D: PDL x max shared-memory carveout on the mixed suites
O=gpurun_out/exp56; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for rep in 1 2; do
  for cfg in 00 01 10 11; do
    p=${cfg:0:1}; c=${cfg:1:1}
    for w in ttc57 smallfvi; do
      TTLG_PDL=$p TTLG_CARVE=$c timeout 600 python bench.py --workload $w --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --tune 0 > $O/bench_${w}_p${p}c${c}_r$rep.json 2> $O/bench_${w}_p${p}c${c}_r$rep.err
    done
  done
done
