#!/bin/bash
# A/B: programmatic dependent launch (TTLG_PDL=1, default) vs plain stream serialisation (0)
O=gpurun_out/exp55; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
for rep in 1 2; do
  for v in 0 1; do
    for w in ttc57 ccsdt smallfvi c1; do
      TTLG_PDL=$v TTLG_BENCH_CASES=1 timeout 600 python bench.py --workload $w --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --tune 0 > $O/bench_${w}_v${v}_r$rep.json 2> $O/bench_${w}_v${v}_r$rep.err
    done
  done
done
